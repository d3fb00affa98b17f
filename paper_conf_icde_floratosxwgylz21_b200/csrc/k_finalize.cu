// k_finalize.cu -- a8 (aggregate finalize + outer comparison) and a9
// (ordered compaction of the survivors), plus the partial-aggregate init and
// the column min/max used by the SUM/AVG overflow pre-check.
//
// PAPER.md P:183 (§III-B, Fig. 4): after the subquery loop fills Res[i], the
// drive program runs "Selection(=, R.col1, Res)" and materialises the result
// (0-1 vector -> prefix sum -> materialize).  Here one kernel computes
// Res[i] from the per-tuple partial aggregates with the SQL empty-set rules
// (readings R1, R2), evaluates a*x OP b*v exactly in int128 (R6, R7) and
// compacts the survivors in row order with a decoupled look-back.
#include <climits>

#include "internal.h"
#include "scan.cuh"

namespace ng {

constexpr int F_THREADS = 256;
constexpr int F_WARPS = F_THREADS / 32;
#ifndef NG_F_ITEMS
#define NG_F_ITEMS 2   // rows per thread per batch (loads of all of them in flight, then evaluated)
#endif
constexpr int F_ITEMS = NG_F_ITEMS;
constexpr int F_TILE = F_THREADS * F_ITEMS;
constexpr int F_STAGE_ROWS = 8192;   // compaction: rows per chunk kept in shared memory (9 B each)

size_t finalize_scratch_bytes(long long n)
{
    // barrier word, per-CTA counts (<= 2048), ballot words (n / 8 bytes)
    return 1024 + 16384 + (size_t)(n / 32 + 2) * 4 + 256;
}

// ------------------------------------------------------------------ a8 + a9
// round_half_away_from_zero(num / den), den > 0 (reading R6).
__device__ __forceinline__ long long div_round_half_away(__int128 num, long long den)
{
    __int128 mag = num < 0 ? -num : num;
    __int128 q = (2 * mag + den) / (2 * (__int128)den);
    return (long long)(num < 0 ? -q : q);
}

// AVG as a scaled integer: round_half_away(acc * 10^6 / c), c > 0.  The
// int128 quotient is a slow software routine (~67 us for SF1 Q17's 6.3k R'
// rows at 16 rows per thread); split it instead: |acc| = q0 c + r0, so
// |acc| 10^6 / c = q0 10^6 + r0 10^6 / c with r0 10^6 < c 10^6 < 2^53 --
// identical result in 64-bit arithmetic whenever q0 10^6 fits.
__device__ __forceinline__ long long avg_scaled(long long acc, long long c)
{
    const unsigned long long mag = acc < 0 ? 0ull - (unsigned long long)acc : (unsigned long long)acc;
    const unsigned long long uc = (unsigned long long)c;
    const unsigned long long q0 = mag / uc, r0 = mag - q0 * uc;
    if (uc < (1ull << 32) && q0 < 9223372036854ull) {   // q0 10^6 + 10^6 <= INT64_MAX
        const unsigned long long t = r0 * 1000000ull;
        const unsigned long long q = q0 * 1000000ull + (2 * t + uc) / (2 * uc);
        return acc < 0 ? -(long long)q : (long long)q;
    }
    return div_round_half_away((__int128)acc * 1000000, c);
}

// ---- one R' row: inputs, then Res[i] + the outer comparison (R1, R2, R6, R7)
struct FinIn {
    long long acc, cnt, x, g;
    int row;
    bool kval, xv;
};

__device__ __forceinline__ void fin_load(const FinalizeArgs &A, long long i, FinIn &r)
{
    r.kval = A.kvalid ? A.kvalid[i] != 0 : true;
    r.g = A.map ? (long long)A.map[i] : i;   // cached result slot
    r.cnt = A.cnt[r.g];
    r.acc = A.acc[r.g];
    r.row = A.ids[i];
    r.x = 0;
    r.xv = false;
}

__device__ __forceinline__ void fin_load_x(const FinalizeArgs &A, FinIn &r)
{
    if (A.agg != EXISTS && A.agg != NOT_EXISTS) {
        r.xv = !(A.x_valid && !A.x_valid[r.row]);
        r.x = load_w(A.x_col, A.x_w, r.row);
    }
}

// value (0 when NULL), valid, passed.  Inlined (a call would put the kernel
// parameters and the row in local memory); callers unroll over at most
// F_EVAL rows (round 1: 16 unrolled rows made a ~175 KB kernel whose
// instruction-cache misses dominated small R').
__device__ __forceinline__ void fin_eval(const FinalizeArgs &A, const FinIn &r, long long &value, bool &valid,
                                      bool &passed)
{
    const long long c = r.kval ? r.cnt : 0;   // NULL key: empty subquery (R2)
    long long acc = r.acc;
    bool vv = true;
    if (A.acc_hi && c > 0) {   // split SUM: hi * 2^32 + lo, exact (reading R5)
        const __int128 t = (__int128)A.acc_hi[r.g] * 4294967296ll + (__int128)(unsigned long long)acc;
        if (t > (__int128)LLONG_MAX || t < (__int128)LLONG_MIN) {
            atomicOr(A.overflow, 1ull);
            acc = 0;
        } else {
            acc = (long long)t;
        }
    }
    long long v = 0;
    switch (A.agg) {
    case MIN: case MAX: case SUM: vv = c > 0; v = acc; break;
    case COUNT: v = c; break;
    case AVG: vv = c > 0; if (vv) v = avg_scaled(acc, c); break;
    case EXISTS: v = c > 0; break;
    default: v = c == 0; break;
    }
    bool p;
    if (A.agg == EXISTS || A.agg == NOT_EXISTS) {
        p = v != 0;
    } else {
        p = false;
        if (vv && r.xv) {
            if (A.a == 1 && A.b == 1 && A.agg != AVG) {   // no scaling: a plain 64-bit compare (uniform branch)
                p = cmp_rt<long long>(r.x, A.outer_op, v);
            } else {
                const __int128 x = r.x;
                if (A.agg == AVG)
                    p = cmp_rt<__int128>((__int128)A.a * x * c, A.outer_op, (__int128)A.b * acc);
                else
                    p = cmp_rt<__int128>((__int128)A.a * x, A.outer_op, (__int128)A.b * v);
            }
        }
    }
    value = vv ? v : 0;
    valid = vv;
    passed = p;
}

__device__ __forceinline__ void fin_write(const FinalizeArgs &A, const FinIn &r, long long pos, long long value,
                                          bool valid, bool passed)
{
    A.out_ids[pos] = A.row_id_base + r.row;
    A.out_vals[pos] = value;
    A.out_valid[pos] = valid ? 1 : 0;
    A.out_passed[pos] = passed ? 1 : 0;
    if (A.out_sum) {
        long long sum = r.kval ? r.acc : 0;
        if (A.acc_hi && r.kval)
            sum = (long long)((__int128)A.acc_hi[r.g] * 4294967296ll + (__int128)(unsigned long long)sum);
        A.out_sum[pos] = sum;
        A.out_cnt[pos] = r.kval ? r.cnt : 0;
    }
}

// emit_all: every R' tuple at its own position (no compaction, no scan)
__global__ void __launch_bounds__(F_THREADS) finalize_all_kernel(FinalizeArgs A)
{
    const long long n = *A.d_nrp;
    const long long t0 = blockIdx.x * (long long)F_THREADS + threadIdx.x, nt = (long long)gridDim.x * F_THREADS;
    for (long long b = t0; b < n; b += nt * F_ITEMS) {
        FinIn r[F_ITEMS];
#pragma unroll
        for (int j = 0; j < F_ITEMS; j++)
            if (b + j * nt < n) fin_load(A, b + j * nt, r[j]);
#pragma unroll
        for (int j = 0; j < F_ITEMS; j++)
            if (b + j * nt < n) fin_load_x(A, r[j]);
#pragma unroll
        for (int j = 0; j < F_ITEMS; j++) {
            if (b + j * nt < n) {
                long long v;
                bool vv, p;
                fin_eval(A, r[j], v, vv, p);
                fin_write(A, r[j], b + j * nt, v, vv, p);
            }
        }
    }
    if (t0 == 0) *A.out_count = n;
}

// Survivors only: the ordered compaction as one cooperative launch (P:235's
// 0-1 vector -> prefix sum -> materialize, like the R' filter, §8): a chunk
// per CTA; phase 1 evaluates every row of the chunk into ballot words (the
// 0-1 vector, n / 8 bytes) + the chunk count; one grid barrier; phase 2 walks
// the survivors 32 at a time and re-evaluates each from its inputs to write
// it (the round-1 kernel's decoupled look-back over ~16k tiles serialised on
// L2 round trips: 0.44 ms for C5's 16M R').
__global__ void __launch_bounds__(F_THREADS, 2)
finalize_compact_kernel(FinalizeArgs A, long long chunk, unsigned *__restrict__ bits,
                        unsigned long long *__restrict__ counts, unsigned *__restrict__ barrier)
{
    extern __shared__ __align__(16) unsigned char f_smem[];
    __shared__ unsigned long long s_red[F_WARPS];
    __shared__ unsigned s_wtot[F_WARPS];
    __shared__ unsigned long long s_base;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const long long n = *A.d_nrp;
    // chunks from the ACTUAL |R'| (the host sized the grid by its upper
    // bound): whole 32-row words, every CTA a share
    (void)chunk;
    const long long chunk_d = ((n + gridDim.x - 1) / gridDim.x + 31) / 32 * 32;
    const long long c0 = min(n, blockIdx.x * chunk_d);
    const long long c1 = min(n, c0 + chunk_d);
    // chunks that fit shared memory keep every row's (value, valid|passed)
    // from phase 1, so phase 2 writes survivors without re-evaluating them
    // (dense survivors, e.g. SF10 Q4's 92 %); larger chunks re-evaluate
    const bool staged = chunk_d <= F_STAGE_ROWS && !A.out_sum;
    long long *s_v = (long long *)f_smem;
    uint8_t *s_f = f_smem + F_STAGE_ROWS * 8;
    // ---- phase 1: passed bits of every row of the chunk
    unsigned long long mycount = 0;
    const long long w0 = c0 / 32, w1 = c1 > c0 ? (c1 + 31) / 32 : w0;
    for (long long wb = w0 + warp; wb < w1; wb += F_WARPS * F_ITEMS) {
        FinIn r[F_ITEMS];
        bool live[F_ITEMS];
#pragma unroll
        for (int j = 0; j < F_ITEMS; j++) {
            const long long row = (wb + (long long)j * F_WARPS) * 32 + lane;
            live[j] = wb + (long long)j * F_WARPS < w1 && row < c1;
            if (live[j]) fin_load(A, row, r[j]);
        }
#pragma unroll
        for (int j = 0; j < F_ITEMS; j++)
            if (live[j]) fin_load_x(A, r[j]);
#pragma unroll
        for (int j = 0; j < F_ITEMS; j++) {
            bool p = false;
            if (live[j]) {
                long long v;
                bool vv;
                fin_eval(A, r[j], v, vv, p);
                if (staged) {
                    const long long lr = (wb + (long long)j * F_WARPS) * 32 + lane - c0;
                    s_v[lr] = v;
                    s_f[lr] = (uint8_t)((vv ? 1 : 0) | (p ? 2 : 0));
                }
            }
            const unsigned m = __ballot_sync(FULL, p);
            if (wb + (long long)j * F_WARPS < w1 && lane == 0) {
                bits[wb + (long long)j * F_WARPS] = m;
                mycount += __popc(m);
            }
        }
    }
    if (lane == 0) s_red[warp] = mycount;
    __syncthreads();
    if (tid == 0) {
        unsigned long long t = 0;
        for (int w = 0; w < F_WARPS; w++) t += s_red[w];
        st_relaxed_u64(counts + blockIdx.x, t);
        __threadfence();
        atomicAdd(barrier, 1u);
        while (ld_relaxed_u32(barrier) < gridDim.x) __nanosleep(64);
        __threadfence();
    }
    __syncthreads();
    unsigned long long pre = 0;
    for (int b = tid; b < (int)blockIdx.x; b += F_THREADS) pre += ld_relaxed_u64(counts + b);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) pre += __shfl_xor_sync(FULL, pre, o);
    if (lane == 0) s_red[warp] = pre;
    __syncthreads();
    if (tid == 0) {
        unsigned long long t = 0;
        for (int w = 0; w < F_WARPS; w++) t += s_red[w];
        s_base = t;
        if (blockIdx.x == gridDim.x - 1) *A.out_count = (long long)(t + ld_relaxed_u64(counts + blockIdx.x));
    }
    __syncthreads();
    // ---- phase 2: survivors, 32 at a time per warp (cf. filter_rp_kernel)
    unsigned long long run = s_base;
    for (long long g = w0; g < w1; g += 32 * F_WARPS) {
        const long long wi = g + warp * 32 + lane;
        const unsigned word = wi < w1 ? __ldcg(bits + wi) : 0u;
        const unsigned c = __popc(word);
        unsigned incl = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned t = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += t;
        }
        if (lane == 31) s_wtot[warp] = incl;
        __syncthreads();
        unsigned woff = 0, btot = 0;
#pragma unroll
        for (int w = 0; w < F_WARPS; w++) {
            const unsigned t = s_wtot[w];
            woff += w < warp ? t : 0;
            btot += t;
        }
        const unsigned excl = incl - c;
        const unsigned wtotal = __shfl_sync(FULL, incl, 31);
        for (unsigned b = 0; b < wtotal; b += 32) {
            const unsigned rk = b + lane;
            int w = 0;
#pragma unroll
            for (int step = 16; step > 0; step >>= 1) {
                const unsigned e = __shfl_sync(FULL, excl, w + step);
                if (e <= rk) w += step;
            }
            const unsigned ew = __shfl_sync(FULL, excl, w);
            const unsigned wv = __shfl_sync(FULL, word, w);
            if (rk < wtotal) {
                const long long row = (g + warp * 32 + w) * 32 + (int)__fns(wv, 0, (int)(rk - ew) + 1);
                const long long pos = (long long)run + woff + rk;
                if (staged) {
                    const uint8_t f = s_f[row - c0];
                    A.out_ids[pos] = A.row_id_base + A.ids[row];
                    A.out_vals[pos] = s_v[row - c0];
                    A.out_valid[pos] = f & 1;
                    A.out_passed[pos] = (f >> 1) & 1;
                } else {
                    FinIn r;
                    fin_load(A, row, r);
                    fin_load_x(A, r);
                    long long v;
                    bool vv, p;
                    fin_eval(A, r, v, vv, p);
                    fin_write(A, r, pos, v, vv, p);
                }
            }
        }
        run += btot;
        __syncthreads();
    }
}

size_t finalize_zero_bytes() { return 1024; }

cudaError_t launch_finalize(const FinalizeArgs &a, cudaStream_t st, long long *launches, bool prezeroed)
{
    cudaError_t e = prezeroed ? cudaSuccess : cudaMemsetAsync(a.out_count, 0, sizeof(long long), st);
    if (e != cudaSuccess || a.n_rp_max <= 0) return e;
    int sms = 0;
    e = per_device_setup((const void *)finalize_all_kernel, 0, &sms, [](int dev, int *v) {
        return cudaDeviceGetAttribute(v, cudaDevAttrMultiProcessorCount, dev);
    });
    if (e != cudaSuccess) return e;
    if (a.emit_all) {
        long long blocks = (a.n_rp_max + F_THREADS * F_ITEMS - 1) / (F_THREADS * F_ITEMS);
        if (blocks > (long long)sms * 8) blocks = (long long)sms * 8;
        finalize_all_kernel<<<(unsigned)blocks, F_THREADS, 0, st>>>(a);
        ++*launches;
        return cudaGetLastError();
    }
    if (!prezeroed) {
        e = cudaMemsetAsync(a.scratch, 0, finalize_zero_bytes(), st);
        if (e != cudaSuccess) return e;
    }
    const int smem = F_STAGE_ROWS * 9;
    int occ = 0;
    e = per_device_setup((const void *)finalize_compact_kernel, 0, &occ, [&](int, int *v) {
        cudaError_t e1 = cudaFuncSetAttribute(finalize_compact_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e1 != cudaSuccess) return e1;
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(v, finalize_compact_kernel, F_THREADS, smem);
    });
    if (e != cudaSuccess) return e;
    if (occ < 1) return cudaErrorInvalidConfiguration;
    // resident grid (the barrier), chunks of whole 32-row words; no more CTAs
    // than chunks of >= 1024 rows
    long long grid = (long long)sms * occ;
    if (grid > 2048) grid = 2048;
    const long long need = (a.n_rp_max + 1023) / 1024;
    if (grid > need) grid = need < 1 ? 1 : need;
    long long chunk = (a.n_rp_max + grid - 1) / grid;
    chunk = (chunk + 31) / 32 * 32;
    unsigned *barrier = (unsigned *)a.scratch;
    unsigned long long *counts = (unsigned long long *)((char *)a.scratch + 1024);
    unsigned *bits = (unsigned *)((char *)a.scratch + 1024 + 16384);
    FinalizeArgs aa = a;
    void *args[] = {(void *)&aa, (void *)&chunk, (void *)&bits, (void *)&counts, (void *)&barrier};
    e = cudaLaunchCooperativeKernel((const void *)finalize_compact_kernel, dim3((unsigned)grid), dim3(F_THREADS),
                                    args, (size_t)smem, st);
    ++*launches;
    return e;
}

// ------------------------------------------------------------------ partials
__global__ void init_partials_kernel(const long long *__restrict__ d_n, long long acc0, long long *__restrict__ acc,
                                     long long *__restrict__ cnt)
{
    const long long n = *d_n;   // the actual |R'| (the grid covers the host's upper bound)
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        acc[i] = acc0;
        cnt[i] = 0;
    }
}

cudaError_t launch_init_partials(long long n, const long long *d_n, int agg, long long *acc, long long *cnt,
                                 cudaStream_t st, long long *launches)
{
    if (n <= 0) return cudaSuccess;
    long long acc0 = agg == MIN ? LLONG_MAX : (agg == MAX ? LLONG_MIN : 0);
    long long blocks = (n + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    init_partials_kernel<<<(unsigned)blocks, 256, 0, st>>>(d_n, acc0, acc, cnt);
    ++*launches;
    return cudaGetLastError();
}

// ------------------------------------------------------------------ tiny queries
// The whole nested-method query in ONE launch for tiny inputs (|S| <= 4096,
// |R| <= 4096, |R| x |S| <= 2^21 pairs; the plan template's nested-loop
// strategy without caching).  Every stage of the regular sequence (fill, R'
// filter, S' filter, partial init, tiled nested loop, finalize + ordered
// compaction) costs a launch and a few microseconds of latency on inputs
// this small, so one kernel does them all.  CTA c of G owns a contiguous
// slice of R:
//   1. S' = rows of S whose inner predicates hold, key NOT NULL (and payload
//      NOT NULL for MIN/MAX/SUM/AVG), compacted into the CTA's shared memory
//      (any order: the aggregates are order-free; every CTA holds all of S');
//   2. warp w evaluates outer tuple r of the slice: outer predicates, then
//      the Fig. 2 loop over S' with the lanes striding S' (the correlated
//      predicate as one unsigned range test), a warp reduction (SUM / AVG
//      exact in int128, OVERFLOW when a sum leaves int64, as the oracle),
//      then fin_eval -- the finalize kernel's reading R1/R2/R6/R7 code;
//   3. a block scan of the slice's emit flags (row order inside the slice),
//      the slice's emit count published at once; the CTA's offset is the
//      sum of its predecessors' counts (no chain: each waits only for their
//      counts), then fin_write.
// Results are the regular path's, field for field (tests run the C1 plans
// and NULL / predicate / 64-bit / composite cases through both).
constexpr int TINY_T = 1024;   // one S row per thread for |S| <= 1024, one outer tuple per warp
constexpr int TINY_W = TINY_T / 32;

__device__ __forceinline__ bool tiny_pred_row(const DevPred &p, long long i)
{
    if (p.valid && !p.valid[i]) return false;
    const long long x = load_w(p.col, p.w, i);
    long long y = p.lit;
    if (p.rhs) {
        if (p.rhs_valid && !p.rhs_valid[i]) return false;
        y = load_w(p.rhs, p.rhs_w, i);
    }
    return cmp_rt<long long>(x, p.op, y);
}

__device__ __forceinline__ bool tiny_preds(const PredSet &ps, long long i)
{
    for (int k = 0; k < ps.n; k++)
        if (!tiny_pred_row(ps.p[k], i)) return false;
    return true;
}

// key of row i as a comparable int64 (single column: the signed value, the
// order of the encoded keys; composite: the packed pair, '=' only); false if NULL
__device__ __forceinline__ bool tiny_key(const KeySrc &k, long long i, long long &out)
{
    if (k.v0 && !k.v0[i]) return false;
    if (k.n_key == 2) {
        if (k.v1 && !k.v1[i]) return false;
        out = (long long)(((unsigned long long)(unsigned)__ldg((const int *)k.c0 + i) << 32) |
                          (unsigned)__ldg((const int *)k.c1 + i));
    } else {
        out = load_w(k.c0, k.w0, i);
    }
    return true;
}

// lanes fold S' entries j = lane, lane + 32, ... with s.key in [lo, hi]
// (unsigned offset test) XOR neg -- the correlated predicate r.key OP s.key
template <int AGG>
__device__ __forceinline__ void tiny_fold(const long long *s_key, const long long *s_val, int ns, int lane,
                                          long long lo, unsigned long long span, bool neg, long long &c,
                                          long long &m, __int128 &sm)
{
    for (int j = lane; j < ns; j += 32) {
        const bool q = ((unsigned long long)(s_key[j] - lo) <= span) != neg;
        if (q) {
            c++;
            if constexpr (AGG == MIN) m = min(m, s_val[j]);
            else if constexpr (AGG == MAX) m = max(m, s_val[j]);
            else if constexpr (AGG == SUM) sm += s_val[j];
        }
    }
}

__global__ void __launch_bounds__(TINY_T) tiny_exec_kernel(TinyArgs T)
{
    const FinalizeArgs &A = T.f;
    extern __shared__ __align__(16) unsigned char smem[];
    long long *s_key = (long long *)smem;                       // [TINY_S_MAX]
    long long *s_val = s_key + TINY_S_MAX;                      // [TINY_S_MAX]
    long long *r_val = s_val + TINY_S_MAX;                      // [chunk] Res value (0 when NULL)
    long long *r_sum = r_val + T.chunk;                         // [chunk] AVG: exact sum
    long long *r_cnt = r_sum + T.chunk;                         // [chunk] AVG: nn
    uint8_t *r_flag = (uint8_t *)(r_cnt + T.chunk);             // [chunk] bit0 valid, bit1 passed, bit2 in R'
    __shared__ int s_ns, s_ovf;
    __shared__ unsigned s_wsum[TINY_W];
    __shared__ unsigned long long s_pre;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const bool value_agg = A.agg == MIN || A.agg == MAX || A.agg == SUM || A.agg == AVG;
    const long long rb = (long long)blockIdx.x * T.chunk;
    const int m_rows = (int)max(0ll, min((long long)T.chunk, T.nR - rb));
    if (tid == 0) {
        s_ns = 0;
        s_ovf = 0;
    }
    __syncthreads();
    // 1. S' into shared memory
    for (long long i = tid; i < T.nS; i += TINY_T) {
        long long k;
        if (!tiny_key(T.sk, i, k) || !tiny_preds(T.sp, i)) continue;
        if (value_agg && T.v.v && !T.v.v[i]) continue;
        const int slot = atomicAdd(&s_ns, 1);
        s_key[slot] = k;
        if (value_agg) s_val[slot] = load_w(T.v.c, T.v.w, i);
    }
    __syncthreads();
    const int ns = s_ns;
    // 2. warp per outer tuple of the slice
    for (int q = warp; q < m_rows; q += TINY_W) {
        const long long r = rb + q;
        const bool in_rp = tiny_preds(T.rp, r);
        long long rk = 0;
        const bool kval = tiny_key(T.rk, r, rk);
        long long lo = rk, hi = rk;
        bool neg = false, empty = !(in_rp && kval);
        switch (T.corr_op) {   // r.key OP s.key  <=>  s.key in [lo, hi] (XOR neg)
        case NE: neg = true; break;
        case LT: if (rk == LLONG_MAX) empty = true; else { lo = rk + 1; hi = LLONG_MAX; } break;
        case LE: hi = LLONG_MAX; break;
        case GT: if (rk == LLONG_MIN) empty = true; else { lo = LLONG_MIN; hi = rk - 1; } break;
        case GE: lo = LLONG_MIN; break;
        default: break;
        }
        const unsigned long long span = (unsigned long long)hi - (unsigned long long)lo;
        long long c = 0, m = A.agg == MAX ? LLONG_MIN : LLONG_MAX;
        __int128 sm = 0;
        if (!empty) {
            switch (A.agg) {
            case MIN: tiny_fold<MIN>(s_key, s_val, ns, lane, lo, span, neg, c, m, sm); break;
            case MAX: tiny_fold<MAX>(s_key, s_val, ns, lane, lo, span, neg, c, m, sm); break;
            case SUM: case AVG: tiny_fold<SUM>(s_key, s_val, ns, lane, lo, span, neg, c, m, sm); break;
            default: tiny_fold<COUNT>(s_key, s_val, ns, lane, lo, span, neg, c, m, sm); break;
            }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            c += __shfl_xor_sync(FULL, c, o);
            const long long m2 = __shfl_xor_sync(FULL, m, o);
            m = A.agg == MAX ? max(m, m2) : min(m, m2);
            const long long lo2 = __shfl_xor_sync(FULL, (long long)(unsigned long long)sm, o);
            const long long hi2 = __shfl_xor_sync(FULL, (long long)(sm >> 64), o);
            sm += ((__int128)hi2 << 64) | (__int128)(unsigned long long)lo2;
        }
        if (lane == 0) {
            uint8_t f = 0;
            if (in_rp) {
                long long acc = m;
                if (A.agg == SUM || A.agg == AVG) {
                    acc = 0;
                    if (sm > (__int128)LLONG_MAX || sm < (__int128)LLONG_MIN) s_ovf = 1;
                    else acc = (long long)sm;
                }
                FinIn in;
                in.acc = acc;
                in.cnt = c;
                in.g = 0;
                in.row = (int)r;
                in.kval = kval;
                fin_load_x(A, in);
                long long value;
                bool valid, passed;
                fin_eval(A, in, value, valid, passed);
                r_val[q] = value;
                r_sum[q] = kval ? acc : 0;
                r_cnt[q] = kval ? c : 0;
                f = (valid ? 1 : 0) | (passed ? 2 : 0) | 4;
            }
            r_flag[q] = f;
        }
    }
    __syncthreads();
    // 3. positions in row order: consecutive rows per thread, a block scan
    const int per = (m_rows + TINY_T - 1) / TINY_T;
    const int q0 = tid * per;
    unsigned cnt_e = 0, cnt_rp = 0;
    for (int k = 0; k < per; k++) {
        const int q = q0 + k;
        if (q < m_rows) {
            const uint8_t f = r_flag[q];
            cnt_rp += (f >> 2) & 1;
            cnt_e += (f & 4) && (A.emit_all || (f & 2)) ? 1 : 0;
        }
    }
    unsigned inc = cnt_e;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned t = __shfl_up_sync(FULL, inc, o);
        if (lane >= o) inc += t;
    }
    if (lane == 31) s_wsum[warp] = inc;
    unsigned rp_w = cnt_rp;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) rp_w += __shfl_xor_sync(FULL, rp_w, o);
    if (lane == 0 && rp_w) atomicAdd((unsigned long long *)&T.counts[0], (unsigned long long)rp_w);
    __syncthreads();
    unsigned pos = inc - cnt_e, total = 0;
    for (int w = 0; w < TINY_W; w++) {
        const unsigned t = s_wsum[w];
        if (w < warp) pos += t;
        total += t;
    }
    // this CTA's count for its successors, then the sum of its predecessors'
    if (tid == 0) {
        st_relaxed_u64(T.status + blockIdx.x, (1ull << 63) | total);
        if (s_ovf) atomicOr((unsigned long long *)&T.counts[8], 1ull);
    }
    if (warp == 0) {
        unsigned long long pre = 0;
        for (int j = lane; j < (int)blockIdx.x; j += 32) {
            unsigned long long v;
            while (((v = ld_relaxed_u64(T.status + j)) >> 63) == 0) {
            }
            pre += v & ~(1ull << 63);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) pre += __shfl_xor_sync(FULL, pre, o);
        if (lane == 0) s_pre = pre;
    }
    __syncthreads();
    const unsigned long long base = s_pre;
    for (int k = 0; k < per; k++) {
        const int q = q0 + k;
        if (q >= m_rows) break;
        const uint8_t f = r_flag[q];
        if (!((f & 4) && (A.emit_all || (f & 2)))) continue;
        FinIn in;
        in.acc = r_sum[q];
        in.cnt = r_cnt[q];
        in.g = 0;
        in.row = (int)(rb + q);
        in.kval = true;   // r_sum / r_cnt already hold 0 for a NULL key
        fin_write(A, in, (long long)(base + pos), r_val[q], (f & 1) != 0, (f & 2) != 0);
        pos++;
    }
    if (tid == 0) {
        if (blockIdx.x == 0) T.counts[1] = ns;
        if (blockIdx.x == gridDim.x - 1) *A.out_count = (long long)(base + total);
    }
}

cudaError_t launch_tiny_exec(const TinyArgs &t0, int num_sms, cudaStream_t st, long long *launches)
{
    TinyArgs t = t0;
    // a slice of >= 32 outer tuples per CTA (one per warp), at most one CTA per SM
    long long g = (t.nR + 31) / 32;
    if (g > num_sms) g = num_sms;
    if (g > TINY_G_MAX) g = TINY_G_MAX;
    if (g < 1) g = 1;
    t.chunk = (int)((t.nR + g - 1) / g);
    if (t.chunk < 1) t.chunk = 1;
    g = t.nR > 0 ? (t.nR + t.chunk - 1) / t.chunk : 1;
    const size_t smem = (size_t)TINY_S_MAX * 16 + (size_t)t.chunk * 25;
    int dummy = 0;
    cudaError_t e = per_device_setup((const void *)tiny_exec_kernel, 0, &dummy, [](int, int *v) {
        *v = 1;
        return cudaFuncSetAttribute(tiny_exec_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)((size_t)TINY_S_MAX * 16 + (size_t)TINY_R_MAX * 25));
    });
    if (e != cudaSuccess) return e;
    e = cudaMemsetAsync(t.counts, 0, 128 + (size_t)TINY_G_MAX * 8, st);   // counts + the per-CTA emit counts
    if (e != cudaSuccess) return e;
    tiny_exec_kernel<<<(unsigned)g, TINY_T, smem, st>>>(t);
    ++*launches;
    return cudaGetLastError();
}

// ------------------------------------------------------------------ column min / max
// (for the SUM/AVG overflow pre-check, reading R5)
// (and out[2] != 0 iff some row is smaller than its predecessor: the
// column is not stored in key order -- the index build's sort-free path;
// out[3] / out[4] the AND / OR of the values: the key bits that vary, so an
// index build without predicates plans its radix passes with no sync)
__global__ void minmax_init_kernel(long long *out)
{
    out[0] = LLONG_MAX;
    out[1] = LLONG_MIN;
    out[2] = 0;
    out[3] = -1;   // AND of the (sign-extended) values
    out[4] = 0;    // OR
}

__global__ void minmax_kernel(const void *__restrict__ col, int w, const uint8_t *__restrict__ valid, long long n,
                              long long *__restrict__ out)
{
    long long mn = LLONG_MAX, mx = LLONG_MIN;
    unsigned long long ka = ~0ull, ko = 0ull;
    bool desc = false;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        if (valid && !valid[i]) continue;
        const long long v = load_w(col, w, i);
        mn = min(mn, v);
        mx = max(mx, v);
        ka &= (unsigned long long)v;
        ko |= (unsigned long long)v;
        if (i > 0 && !valid) desc |= load_w(col, w, i - 1) > v;
    }
    for (int o = 16; o > 0; o >>= 1) {
        mn = min(mn, __shfl_xor_sync(FULL, mn, o));
        mx = max(mx, __shfl_xor_sync(FULL, mx, o));
    }
    desc = __any_sync(FULL, desc);
    for (int o = 16; o > 0; o >>= 1) {
        ka &= __shfl_xor_sync(FULL, ka, o);
        ko |= __shfl_xor_sync(FULL, ko, o);
    }
    if ((threadIdx.x & 31) == 0) {
        atomicMin(&out[0], mn);
        atomicMax(&out[1], mx);
        if (desc) atomicOr((unsigned long long *)&out[2], 1ull);
        atomicAnd((unsigned long long *)&out[3], ka);
        atomicOr((unsigned long long *)&out[4], ko);
    }
}

cudaError_t launch_minmax(const void *col, int w, const uint8_t *valid, long long n, long long *out2, cudaStream_t st,
                          long long *launches)
{
    minmax_init_kernel<<<1, 1, 0, st>>>(out2);
    ++*launches;
    if (n > 0) {
        long long blocks = (n + 255) / 256;
        if (blocks > 148 * 8) blocks = 148 * 8;
        minmax_kernel<<<(unsigned)blocks, 256, 0, st>>>(col, w, valid, n, out2);
        ++*launches;
    }
    return cudaGetLastError();
}

}  // namespace ng

namespace ng {

// ------------------------------------------------------------------ gather
// out[i] = src[ids[i] - base]: materialises a column from a result's row ids
// (multi-level nesting, Fig. 6 -- a level's survivors feed the next).
template <typename T>
__global__ void gather_kernel(const T *__restrict__ src, const long long *__restrict__ ids, long long n,
                              long long base, T *__restrict__ out)
{
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        out[i] = src[ids[i] - base];
}

// ------------------------------------------------------------------ peer put
// Rank r's survivors -> rank 0's window (multi-GPU gather by peer stores):
// 16-byte vector loads / stores where both sides are 16-B aligned, the
// stores go over NVLink when the window is a peer device's memory.
__global__ void put_rows_kernel(const long long *__restrict__ ids, const long long *__restrict__ vals, long long n,
                                long long *__restrict__ wi, long long *__restrict__ wv)
{
    const long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    const long long nt = (long long)gridDim.x * blockDim.x;
    const bool vec = ((((unsigned long long)ids | (unsigned long long)vals | (unsigned long long)wi |
                        (unsigned long long)wv) & 15) == 0);
    if (vec) {
        const long long n2 = n / 2;
        for (long long i = t; i < n2; i += nt) {
            reinterpret_cast<longlong2 *>(wi)[i] = reinterpret_cast<const longlong2 *>(ids)[i];
            reinterpret_cast<longlong2 *>(wv)[i] = reinterpret_cast<const longlong2 *>(vals)[i];
        }
        if (t == 0 && (n & 1)) {
            wi[n - 1] = ids[n - 1];
            wv[n - 1] = vals[n - 1];
        }
    } else {
        for (long long i = t; i < n; i += nt) {
            wi[i] = ids[i];
            wv[i] = vals[i];
        }
    }
    __threadfence_system();
}

cudaError_t launch_put_rows(const long long *ids, const long long *vals, long long n, long long *win_ids,
                            long long *win_vals, cudaStream_t st, long long *launches)
{
    if (n <= 0) return cudaSuccess;
    long long blocks = (n / 2 + 255) / 256;
    if (blocks < 1) blocks = 1;
    if (blocks > 148 * 8) blocks = 148 * 8;
    put_rows_kernel<<<(unsigned)blocks, 256, 0, st>>>(ids, vals, n, win_ids, win_vals);
    ++*launches;
    return cudaGetLastError();
}

cudaError_t launch_gather(int w, const void *src, const long long *ids, long long n, long long base, void *out,
                          cudaStream_t st, long long *launches)
{
    if (n <= 0) return cudaSuccess;
    long long blocks = (n + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    if (w == 4) gather_kernel<int><<<(unsigned)blocks, 256, 0, st>>>((const int *)src, ids, n, base, (int *)out);
    else gather_kernel<long long><<<(unsigned)blocks, 256, 0, st>>>((const long long *)src, ids, n, base,
                                                                   (long long *)out);
    ++*launches;
    return cudaGetLastError();
}

}  // namespace ng

namespace ng {

// ------------------------------------------------------------------ synthetic fills
// Inputs for the cost model's calibration runs (cost.cpp): a counter-based
// hash (splitmix64 finaliser) and ascending runs.
__device__ __forceinline__ unsigned long long mix64(unsigned long long z)
{
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
    return z ^ (z >> 31);
}

template <typename T>
__global__ void fill_hash_kernel(T *__restrict__ out, long long n, unsigned seed, unsigned long long mod, long long lo)
{
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        out[i] = (T)(lo + (long long)(mix64(((unsigned long long)seed << 40) + (unsigned long long)i) % mod));
}

template <typename T>
__global__ void fill_runs_kernel(T *__restrict__ out, long long n, long long div, long long lo)
{
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        out[i] = (T)(lo + i / div);
}

cudaError_t launch_fill_hash(void *out, int w, long long n, unsigned seed, unsigned long long mod, long long lo,
                             cudaStream_t st, long long *launches)
{
    if (n <= 0) return cudaSuccess;
    long long blocks = (n + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    if (w == 4) fill_hash_kernel<int><<<(unsigned)blocks, 256, 0, st>>>((int *)out, n, seed, mod, lo);
    else fill_hash_kernel<long long><<<(unsigned)blocks, 256, 0, st>>>((long long *)out, n, seed, mod, lo);
    ++*launches;
    return cudaGetLastError();
}

cudaError_t launch_fill_runs(void *out, int w, long long n, long long div, long long lo, cudaStream_t st,
                             long long *launches)
{
    if (n <= 0) return cudaSuccess;
    long long blocks = (n + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    if (w == 4) fill_runs_kernel<int><<<(unsigned)blocks, 256, 0, st>>>((int *)out, n, div, lo);
    else fill_runs_kernel<long long><<<(unsigned)blocks, 256, 0, st>>>((long long *)out, n, div, lo);
    ++*launches;
    return cudaGetLastError();
}

}  // namespace ng
