// cost.cpp -- the paper's cost model (§IV, Eqs. (1)-(9))
// for this engine: calibration of the per-element kernel costs K_i on the
// GPU, and the host-side evaluation that predicts one exec's latency under
// each execution strategy (nested loop / index, with or without caching)
// and picks the fastest -- "a cost model to guide subquery processing by
// selecting the most effective execution path".
//
// Calibration ("One method to estimate Ki is actually running the
// query once and reusing this value for all predictions"): each kernel
// family of the hot path runs once on synthetic data in the scratch pool,
// timed with CUDA events after a warm-up; K_i = (time - launches * C) / D_i.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstring>
#include <vector>

#include "../../include/nestgpu.h"
#include "internal.h"

namespace {

struct Timer {
    cudaEvent_t a, b;
    cudaStream_t st;
    explicit Timer(cudaStream_t s) : st(s)
    {
        cudaEventCreate(&a);
        cudaEventCreate(&b);
    }
    ~Timer()
    {
        cudaEventDestroy(a);
        cudaEventDestroy(b);
    }
    // median of 3 timed runs after one warm-up; fn returns cudaError_t
    template <typename F>
    cudaError_t ms(F fn, double *out)
    {
        cudaError_t e = fn();
        if (e != cudaSuccess) return e;
        double t[3];
        for (int r = 0; r < 3; r++) {
            cudaEventRecord(a, st);
            if ((e = fn()) != cudaSuccess) return e;
            cudaEventRecord(b, st);
            if ((e = cudaEventSynchronize(b)) != cudaSuccess) return e;
            float f = 0.f;
            cudaEventElapsedTime(&f, a, b);
            t[r] = f;
        }
        std::sort(t, t + 3);
        *out = t[1];
        return cudaSuccess;
    }
};

inline double pos(double x) { return x > 0 ? x : 0; }

}  // namespace

extern "C" {

nestgpu_status nestgpu_cost_calibrate(nestgpu_ctx *c, int64_t n_rows, nestgpu_cost_params *out)
{
    if (!c || !out) return ng::ctx_fail(c, NESTGPU_ERR_INVALID, "cost_calibrate: null argument");
    cudaSetDevice(ng::ctx_device(c));
    memset(out, 0, sizeof *out);
    const cudaStream_t st = ng::ctx_stream(c);
    long long *L = ng::ctx_launches(c);
    const int sms = ng::ctx_num_sms(c);
    long long n = n_rows > 0 ? n_rows : (16ll << 20);
    n = std::min<long long>(n, 1ll << 28);

    // ------------------------------------------------------------ buffers
    char *kraw = nullptr, *vraw = nullptr, *ids = nullptr, *k1 = nullptr, *v1 = nullptr, *k2 = nullptr,
         *v2 = nullptr, *acc = nullptr, *cnt = nullptr, *oid = nullptr, *oval = nullptr, *oflag = nullptr,
         *fscr = nullptr, *sscr = nullptr, *small = nullptr, *hist = nullptr, *dbase = nullptr, *pre = nullptr,
         *suf = nullptr, *rscr = nullptr, *bscr = nullptr, *gscr = nullptr, *uk = nullptr, *map = nullptr;
    for (;; n /= 2) {
        ng::ctx_scratch_reset(c);
        if (n < (1 << 16)) return ng::ctx_fail(c, NESTGPU_ERR_OOM, "cost_calibrate: arena too small");
        auto A = [&](size_t b) { return (char *)ng::ctx_scratch_alloc(c, b); };
        kraw = A(n * 4); vraw = A(n * 4); ids = A(n * 4); k1 = A(n * 4); v1 = A(n * 4); k2 = A(n * 4);
        v2 = A(n * 4); acc = A(n * 8); cnt = A(n * 8); oid = A(n * 8); oval = A(n * 8); oflag = A(n * 2);
        fscr = A(ng::filter_scratch_bytes(n)); sscr = A(ng::sort_scratch_bytes(n)); small = A(256);
        hist = A(ng::hist_bytes()); dbase = A(8 * 256 * 4); pre = A((n + 1) * 8); suf = A((n + 1) * 8);
        rscr = A(ng::range_scratch_bytes(n)); bscr = A(ng::bnl_scratch_bytes(n)); gscr = A(ng::group_scratch_bytes(n));
        uk = A(n * 4); map = A(n * 4);
        if (kraw && vraw && ids && k1 && v1 && k2 && v2 && acc && cnt && oid && oval && oflag && fscr && sscr &&
            small && hist && dbase && pre && suf && rscr && bscr && gscr && uk && map)
            break;
    }
    long long *d_small = (long long *)small;   // [0] n  [1] n_bnl_r  [2] n_bnl_s  [3] out count  [4..5] extreme
    unsigned *extreme = (unsigned *)(d_small + 4);
#define CC(expr)                                                                            \
    do {                                                                                    \
        cudaError_t e_ = (expr);                                                            \
        if (e_ != cudaSuccess) return ng::ctx_fail(c, NESTGPU_ERR_CUDA, cudaGetErrorString(e_)); \
    } while (0)
    CC(ng::launch_fill_hash(kraw, 4, n, 1, 1ull << 30, 0, st, L));
    CC(ng::launch_fill_hash(vraw, 4, n, 2, 1000, 0, st, L));
    CC(cudaMemsetAsync(small, 0, 256, st));
    CC(cudaStreamSynchronize(st));
    Timer T(st);
    double t;

    // C: a kernel with a tiny input (20 back-to-back launches)
    CC(T.ms([&] {
        cudaError_t e = cudaSuccess;
        for (int i = 0; i < 20 && e == cudaSuccess; i++) e = ng::launch_init_partials(1, d_small, ng::MIN,
                                                                                     (long long *)acc, (long long *)cnt, st, L);
        return e;
    }, &t));
    const double C = t / 20;
    out->launch_ms = C;

    // selection: R' filter (ordered ids + encoded keys), 1 predicate (k >= 0, all pass)
    ng::PredSet ps;
    memset(&ps, 0, sizeof ps);
    ps.n = 1;
    ps.p[0].col = kraw;
    ps.p[0].w = 4;
    ps.p[0].op = ng::GE;
    ps.p[0].lit = 0;
    ng::KeySrc ks;
    memset(&ks, 0, sizeof ks);
    ks.c0 = kraw;
    ks.w0 = 4;
    ks.n_key = 1;
    ng::ValSrc none{nullptr, nullptr, 0};
    CC(T.ms([&] {
        return ng::launch_filter(n, ps, ks, 4, none, 0, 0, 0, (int *)ids, k1, nullptr, nullptr, nullptr, nullptr, fscr,
                                 d_small + 3, st, L);
    }, &t));
    out->filter_ms_per_row = pos(t - 3 * C) / n;

    // index build: digit histogram (3 digits) + one radix pass of (u32 key, u32 payload)
    ng::ValSrc vs{vraw, nullptr, 4};
    CC(ng::launch_filter(n, ps, ks, 4, vs, 4, 1, 1, nullptr, k1, nullptr, v1, nullptr, nullptr, fscr, d_small + 3, st,
                         L));
    const int shifts[3] = {0, 8, 16};
    CC(T.ms([&] { return ng::launch_digit_hist(4, k1, n, shifts, 3, (unsigned *)hist, (unsigned *)dbase, sms, st, L); },
            &t));
    out->hist_ms_per_key_digit = pos(t - 3 * C) / (3.0 * n);
    double t8;
    CC(T.ms([&] {
        return ng::launch_radix_pass(4, 4, k1, k2, v1, v2, n, 0, (const unsigned *)dbase, sscr, st, L);
    }, &t8));
    // (8-byte key, 8-byte payload) pass over the same count: per-key + per-byte split
    CC(ng::launch_fill_hash(acc, 8, n, 7, 1ull << 62, 0, st, L));
    CC(ng::launch_fill_hash(cnt, 8, n, 8, 1000, 0, st, L));
    const int shift8[1] = {8};   // digit offsets of THESE keys (a pass scatters by them)
    CC(ng::launch_digit_hist(8, acc, n, shift8, 1, (unsigned *)hist, (unsigned *)dbase, sms, st, L));
    double t16;
    CC(T.ms([&] {
        return ng::launch_radix_pass(8, 8, acc, oid, cnt, oval, n, 8, (const unsigned *)dbase, sscr, st, L);
    }, &t16));
    out->sort_ms_per_byte = pos(t16 - t8) / (8.0 * n);
    out->sort_ms_per_key = pos(t8 - 2 * C - out->sort_ms_per_byte * 8.0 * n) / n;

    // binary search: '=' COUNT of n/4 probes over n sorted keys in runs of 4
    const long long np = n / 4;
    memcpy(ng::ctx_pinned(c), &np, 8);
    CC(cudaMemcpyAsync(d_small, ng::ctx_pinned(c), 8, cudaMemcpyHostToDevice, st));
    CC(ng::launch_fill_runs(k2, 4, n, 4, 0, st, L));
    CC(ng::launch_fill_hash(k1, 4, np, 3, (unsigned long long)(n / 4), 0, st, L));
    const double steps = std::ceil(std::log2((double)n + 1));
    CC(T.ms([&] {
        return ng::launch_range_agg(4, 4, ng::EQ, ng::COUNT, np, d_small, k1, k2, v1, n, nullptr, nullptr,
                                    (long long *)acc, (long long *)cnt, rscr, st, L);
    }, &t));
    out->probe_ms_per_step = pos(t - 2 * C) / (np * 2.0 * steps);
    // fold: '=' MIN over runs of 16 (the short, thread-per-tuple path)
    CC(ng::launch_fill_runs(k2, 4, n, 16, 0, st, L));
    CC(ng::launch_fill_hash(k1, 4, np, 4, (unsigned long long)(n / 16), 0, st, L));
    CC(T.ms([&] {
        return ng::launch_range_agg(4, 4, ng::EQ, ng::MIN, np, d_small, k1, k2, v1, n, nullptr, nullptr,
                                    (long long *)acc, (long long *)cnt, rscr, st, L);
    }, &t));
    out->range_ms_per_elem = pos(t - 2 * C - out->probe_ms_per_step * np * 2.0 * steps) / (np * 16.0);

    // prefix / suffix aggregates of an index payload
    CC(T.ms([&] { return ng::launch_index_aux(ng::MIN, 4, v1, n, (long long *)pre, (long long *)suf, rscr, st, L); },
            &t));
    out->aux_ms_per_elem = pos(t - 6 * C) / n;

    // nested loop: |R'| x |S'| pairs per aggregate class ('>' correlation)
    // (full R blocks: |R'| a multiple of 2048 tuples and enough units for every CTA)
    const long long nbr = std::max<long long>(2048, std::min<long long>(32768, n / 8)) / 2048 * 2048;
    const long long nbs = std::min<long long>(n / 2, 262144);
    long long nn2[2] = {nbr, nbs};
    memcpy(ng::ctx_pinned(c), nn2, 16);
    CC(cudaMemcpyAsync(d_small + 1, ng::ctx_pinned(c), 16, cudaMemcpyHostToDevice, st));
    const int cls_agg[4] = {ng::MIN, ng::COUNT, ng::SUM, ng::EXISTS};
    for (int kw = 0; kw < 2; kw++) {
        const int kbw = kw ? 8 : 4;
        CC(ng::launch_fill_hash(k1, kbw, nbr, 5, kw ? (1ull << 62) : (1ull << 32), 0, st, L));
        CC(ng::launch_fill_hash(k2, kbw, nbs, 6, kw ? (1ull << 62) : (1ull << 32), 0, st, L));
        for (int k = 0; k < 4; k++) {
            if (cls_agg[k] == ng::EXISTS) CC(cudaMemsetAsync(k1, 0, nbr * kbw, st));   // r.key = 0: no s < r
            CC(T.ms([&] {
                cudaError_t e = ng::launch_init_partials(nbr, d_small + 1, cls_agg[k], (long long *)acc, (long long *)cnt,
                                                         st, L);
                if (e != cudaSuccess) return e;
                return ng::launch_bnl(kbw, cls_agg[k] == ng::COUNT || cls_agg[k] == ng::EXISTS ? 0 : 4, ng::GT,
                                      cls_agg[k], nbr, d_small + 1, k1, nbs, d_small + 2, k2, v1, extreme,
                                      (long long *)acc, (long long *)cnt, bscr, sms, 1, st, L);
            }, &t));
            out->bnl_ms_per_pair[kw][k] = pos(t - 2 * C) / ((double)nbr * nbs);
        }
    }

    // finalize (+ compaction): nothing passes vs everything emitted
    ng::FinalizeArgs fa{};
    fa.n_rp_max = n;
    fa.d_nrp = d_small;
    fa.ids = (const int *)ids;
    fa.acc = (const long long *)acc;
    fa.cnt = (const long long *)cnt;
    fa.x_col = kraw;
    fa.x_w = 4;
    fa.agg = ng::MIN;
    fa.outer_op = ng::EQ;
    fa.a = fa.b = 1;
    fa.out_ids = (long long *)oid;
    fa.out_vals = (long long *)oval;
    fa.out_valid = (uint8_t *)oflag;
    fa.out_passed = (uint8_t *)oflag + n;
    fa.out_count = d_small + 3;
    fa.scratch = fscr;
    memcpy(ng::ctx_pinned(c), &n, 8);
    CC(cudaMemcpyAsync(d_small, ng::ctx_pinned(c), 8, cudaMemcpyHostToDevice, st));
    CC(ng::launch_init_partials(n, d_small, ng::MIN, (long long *)acc, (long long *)cnt, st, L));
    CC(ng::launch_fill_runs(ids, 4, n, 1, 0, st, L));
    double t_none, t_all;
    fa.emit_all = 0;
    CC(T.ms([&] { return ng::launch_finalize(fa, st, L); }, &t_none));
    fa.emit_all = 1;
    CC(T.ms([&] { return ng::launch_finalize(fa, st, L); }, &t_all));
    out->final_ms_per_row = pos(t_none - C) / n;
    out->materialize_ms_per_byte = pos(t_all - t_none) / (18.0 * n);

    // caching: grouping of sorted keys (runs of 4)
    CC(ng::launch_fill_runs(k2, 4, n, 4, 0, st, L));
    CC(ng::launch_iota((int *)v2, n, st, L));
    CC(T.ms([&] {
        return ng::launch_group(4, k2, (const int *)v2, n, uk, (int *)map, d_small + 3, gscr, st, L);
    }, &t));
    out->group_ms_per_key = pos(t - C) / n;

    // host round trip: small D2H + stream synchronisation (20 in a row)
    {
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        float f = 0.f;
        for (int rep = 0; rep < 2; rep++) {   // first round warms up
            cudaEventRecord(a, st);
            for (int i = 0; i < 20; i++) {
                CC(cudaMemcpyAsync(ng::ctx_pinned(c), d_small, 8, cudaMemcpyDeviceToHost, st));
                CC(cudaStreamSynchronize(st));
            }
            cudaEventRecord(b, st);
            CC(cudaEventSynchronize(b));
            cudaEventElapsedTime(&f, a, b);
        }
        cudaEventDestroy(a);
        cudaEventDestroy(b);
        out->sync_ms = f / 20.0;
    }
#undef CC
    ng::ctx_scratch_reset(c);

    // Fixed host-side overheads: tiny plans through the public API, wall
    // clock, minus what the model already charges for them.
    {
        uint64_t mark;
        nestgpu_status s = nestgpu_mark(c, &mark);
        if (s) return s;
        const int m = 256;
        std::vector<int32_t> k(m), v(m);
        for (int i = 0; i < m; i++) { k[i] = (i * 37) % 64; v[i] = (i * 11) % 16; }
        int32_t rk, rv, sk, sv;
        if ((s = nestgpu_load_column(c, NG_INT32, 0, k.data(), nullptr, m, &rk)) ||
            (s = nestgpu_load_column(c, NG_INT32, 0, v.data(), nullptr, m, &rv)) ||
            (s = nestgpu_load_column(c, NG_INT32, 0, k.data(), nullptr, m, &sk)) ||
            (s = nestgpu_load_column(c, NG_INT32, 0, v.data(), nullptr, m, &sv)))
            return s;
        nestgpu_plan P;
        memset(&P, 0, sizeof P);
        P.outer_key_cols[0] = rk;
        P.inner_key_cols[0] = sk;
        P.n_key_cols = 1;
        P.corr_op = NG_EQ;
        P.agg = NG_MIN;
        P.agg_col = sv;
        P.outer_cmp_col = rv;
        P.outer_op = NG_EQ;
        P.lhs_mult = P.rhs_mult = 1;
        P.index = -1;
        nestgpu_result res;
        auto wall = [&](auto fn, double *ms) -> nestgpu_status {
            double t[7];
            for (int r = 0; r < 8; r++) {
                const auto a = std::chrono::steady_clock::now();
                nestgpu_status e = fn();
                if (e) return e;
                cudaStreamSynchronize(st);
                const auto b = std::chrono::steady_clock::now();
                if (r) t[r - 1] = std::chrono::duration<double, std::milli>(b - a).count();
            }
            std::sort(t, t + 7);
            *ms = t[3];
            return NESTGPU_OK;
        };
        nestgpu_cost_input in;
        memset(&in, 0, sizeof in);
        in.n_r = in.n_s = in.n_rp = in.n_sp = m;
        in.n_distinct = 64;
        in.sum_k = (int64_t)m * 4;
        in.key_bytes = 4;
        in.payload_bytes = 4;
        in.sort_passes = 1;
        in.dedup_passes = 1;
        in.corr_op = NG_EQ;
        in.agg = NG_MIN;
        nestgpu_cost_estimate est;
        double t_exec, t_dedup, t_build;
        if ((s = wall([&] { return nestgpu_exec_correlated(c, &P, &res); }, &t_exec))) return s;
        P.dedup = 1;
        if ((s = wall([&] { return nestgpu_exec_correlated(c, &P, &res); }, &t_dedup))) return s;
        P.dedup = 0;
        int32_t ix = -1;
        const int32_t keyc[1] = {sk};
        if ((s = wall([&] {
                if (ix >= 0) nestgpu_drop_index(c, ix);
                return nestgpu_build_index(c, keyc, 1, sv, nullptr, 0, &ix);
            }, &t_build)))
            return s;
        nestgpu_cost_estimate_plan(out, &in, &est);
        out->exec_overhead_ms = pos(t_exec - est.ms[NESTGPU_STRATEGY_NESTED_LOOP]);
        out->dedup_overhead_ms = pos(t_dedup - t_exec - (est.ms[NESTGPU_STRATEGY_NESTED_LOOP_CACHED] -
                                                         est.ms[NESTGPU_STRATEGY_NESTED_LOOP]));
        out->build_overhead_ms = pos(t_build - est.index_build_ms);
        if ((s = nestgpu_release(c, mark))) return s;
    }
    return NESTGPU_OK;
}

nestgpu_status nestgpu_cost_estimate_plan(const nestgpu_cost_params *p, const nestgpu_cost_input *in,
                                          nestgpu_cost_estimate *out)
{
    if (!p || !in || !out) return NESTGPU_ERR_INVALID;
    memset(out, 0, sizeof *out);
    if (in->n_r < 0 || in->n_s < 0 || in->n_rp < 0 || in->n_sp < 0 || in->n_distinct < 0 || in->sum_k < 0 ||
        in->survivors < 0 || in->n_rp > in->n_r || in->n_sp > in->n_s || in->n_distinct > in->n_rp ||
        (in->key_bytes != 4 && in->key_bytes != 8) ||
        (in->payload_bytes != 0 && in->payload_bytes != 4 && in->payload_bytes != 8) || in->sort_passes < 0 ||
        in->sort_passes > 8 || in->dedup_passes < 0 || in->dedup_passes > 8 || in->corr_op < NG_EQ ||
        in->corr_op > NG_GE || in->agg < NG_MIN || in->agg > NG_NOT_EXISTS)
        return NESTGPU_ERR_INVALID;
    const double C = p->launch_ms;
    const double nR = (double)in->n_r, nS = (double)in->n_s, nRp = (double)in->n_rp, nSp = (double)in->n_sp;
    const double kb = in->key_bytes, vb = in->payload_bytes;
    const bool minmax = in->agg == NG_MIN || in->agg == NG_MAX;
    const bool sumavg = in->agg == NG_SUM || in->agg == NG_AVG;
    const bool value_agg = minmax || sumavg;
    const int cls = minmax ? 0 : (in->agg == NG_COUNT ? 1 : (sumavg ? 2 : 3));
    // launch counts follow api.cpp: one fill kernel per exec / index build
    // zeroes every scratch region, a filter is one launch
    auto selection = [&](double rows) { return C + p->filter_ms_per_row * rows; };   // Eq. (1)

    // U, Eq. (8): outer selection, then finalize + compaction (M * D_r * sum Rs)
    const double rs = 18.0 + (in->agg == NG_AVG ? 16.0 : 0.0);   // id + value + valid + passed (+ sum, nn)
    const double U = selection(nR) + 2 * C + p->final_ms_per_row * nRp +
                     p->materialize_ms_per_byte * (double)in->survivors * rs + p->sync_ms + p->exec_overhead_ms;
    out->outer_ms = U;

    // bytes per key moved by the passes: (key in + key out) / 2 + payload;
    // narrowed 8-byte keys are 4 bytes wide between the first and last pass
    auto pass_bytes = [&](double passes) {
        if (passes <= 0) return 0.0;
        if (!(in->narrow_keys && kb == 8 && passes >= 2)) return passes * (kb + vb);
        return 2 * (6 + vb) + (passes - 2) * (4 + vb);
    };
    // caching: S - Ch evaluations after sorting / grouping the R' keys
    const double dp = in->dedup_passes;
    const double dedup = 2 * C + p->hist_ms_per_key_digit * nRp * dp +
                         dp * (2 * C + p->sort_ms_per_key * nRp) +
                         p->sort_ms_per_byte * nRp * (pass_bytes(dp) - dp * vb + dp * 4) + C +
                         p->group_ms_per_key * nRp +
                         2 * p->sync_ms + p->dedup_overhead_ms;

    // index build (invariant, once): S' selection + histogram + radix passes;
    // plus the payload prefix aggregates when the plan reads them (NEXT 3)
    const double sp = in->sort_passes;
    double build = C + selection(nS) + p->sync_ms + p->build_overhead_ms +
                   (sp > 0 ? 2 * C + p->hist_ms_per_key_digit * nSp * sp : 0) +
                   sp * (C + p->sort_ms_per_key * nSp) + p->sort_ms_per_byte * nSp * pass_bytes(sp);
    if (value_agg && (in->corr_op != NG_EQ || sumavg)) build += (minmax ? 6 : 3) * C + p->aux_ms_per_elem * nSp;
    out->index_build_ms = build;

    const double steps = std::ceil(std::log2(nSp + 1));
    const double searches = (in->corr_op == NG_EQ || in->corr_op == NG_NE) ? 2 : 1;
    const bool scans = in->corr_op == NG_EQ && minmax;   // the only ranges folded element by element
    auto nested_index = [&](double ev) {
        const double share = nRp > 0 ? ev / nRp : 0;
        return 2 * C + p->probe_ms_per_step * ev * steps * searches +
               (scans ? p->range_ms_per_elem * (double)in->sum_k * share : 0);
    };
    // nested loop: S' selection (invariant) + init + |evaluations| x |S'| pairs
    auto nested_loop = [&](double ev) {
        return selection(nS) + 2 * C + p->bnl_ms_per_pair[in->key_bytes == 8][cls] * ev * nSp;
    };
    const double nd = (double)in->n_distinct;
    out->nested_ms[NESTGPU_STRATEGY_NESTED_LOOP] = nested_loop(nRp);
    out->nested_ms[NESTGPU_STRATEGY_INDEX] = nested_index(nRp);
    out->nested_ms[NESTGPU_STRATEGY_NESTED_LOOP_CACHED] = dedup + nested_loop(nd);
    out->nested_ms[NESTGPU_STRATEGY_INDEX_CACHED] = dedup + nested_index(nd);
    // Eq. (9): Q = N + Nmem + U  (Nmem = 0: preloaded columns, pooled scratch)
    for (int s = 0; s < 4; s++) {
        const bool idx = s == NESTGPU_STRATEGY_INDEX || s == NESTGPU_STRATEGY_INDEX_CACHED;
        out->ms[s] = U + out->nested_ms[s] + (idx ? build : 0);
    }
    int best = 0;
    for (int s = 1; s < 4; s++)
        if (out->ms[s] < out->ms[best]) best = s;
    out->best = best;
    return NESTGPU_OK;
}

}  // extern "C"
