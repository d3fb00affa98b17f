// k_filter.cu -- a2/a3 (outer / inner local predicates -> compacted R', S')
// and a8/a9 (aggregate finalize + outer comparison + ordered compaction).
//
// PAPER.md P:235 (§III-C): a Selection is "scan -> 0-1 vector -> prefix-sum ->
// materialize" over several primitive kernels with inter-kernel results in a
// pool.  On B200 this is ONE pass per relation: each CTA evaluates the
// predicates for a 4096-row tile with coalesced column loads, builds the 0-1
// vector in registers (warp __ballot_sync), ranks survivors with __popc, gets
// its global offset by decoupled look-back (no second pass over HBM), and
// writes the compacted (row id | encoded key | payload) directly.  The same
// tile machinery compacts the survivors of the outer comparison (the final
// "Selection(=, R.col1, Res)" + Materialize of P:183), fused with the
// aggregate finalisation.
#include <climits>
#include <type_traits>

#include "internal.h"

namespace ng {

constexpr int F_THREADS = 256;
constexpr int F_WARPS = F_THREADS / 32;
constexpr int F_ITEMS = 16;
constexpr int F_TILE = F_THREADS * F_ITEMS;

size_t filter_scratch_bytes(long long n)
{
    long long tiles = (n + F_TILE - 1) / F_TILE;
    return (size_t)(tiles + 1) * 8 + 256;
}

// Shared scan of the per-(item, warp) survivor counts in row order
// (item-major, then warp) + the tile's global offset.  Called by all threads.
// s_cnt holds counts on entry and exclusive offsets on exit.
__device__ __forceinline__ unsigned long long tile_offsets(unsigned (*s_cnt)[F_WARPS], unsigned long long *status,
                                                           long long tile, long long num_tiles,
                                                           long long *out_count,
                                                           unsigned long long *s_base)
{
    __syncthreads();
    if (threadIdx.x < 32) {
        unsigned *flat = &s_cnt[0][0];
        const unsigned lane = threadIdx.x;
        unsigned c[4], s = 0;
#pragma unroll
        for (int q = 0; q < 4; q++) { c[q] = flat[4 * lane + q]; s += c[q]; }
        unsigned incl = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            unsigned t = __shfl_up_sync(FULL, incl, o);
            if ((int)lane >= o) incl += t;
        }
        unsigned run = incl - s;
        const unsigned total = __shfl_sync(FULL, incl, 31);
#pragma unroll
        for (int q = 0; q < 4; q++) { unsigned t = c[q]; flat[4 * lane + q] = run; run += t; }
        unsigned long long base = lookback_warp(status, tile, total);
        if (lane == 0) {
            *s_base = base;
            if (tile == num_tiles - 1) *out_count = (long long)(base + total);
        }
    }
    __syncthreads();
    return *s_base;
}

template <int KB, int VB>
__global__ void __launch_bounds__(F_THREADS)
filter_kernel(long long n, PredSet preds, KeySrc ks, ValSrc vs, int drop_null_key, int drop_null_val,
              int *__restrict__ out_ids, void *__restrict__ out_keys, uint8_t *__restrict__ out_kvalid,
              void *__restrict__ out_vals, unsigned *__restrict__ hist, unsigned *__restrict__ extreme,
              unsigned long long *__restrict__ status, unsigned *__restrict__ counter,
              long long *__restrict__ out_count)
{
    using K = typename std::conditional<KB == 8, uint64_t, uint32_t>::type;
    using V = typename std::conditional<VB == 8, long long, int>::type;
    constexpr int HB = KB > 0 ? KB : 1;
    __shared__ unsigned s_tile;
    __shared__ unsigned s_cnt[F_ITEMS][F_WARPS];
    __shared__ unsigned long long s_base;
    __shared__ unsigned s_hist[HB * 256];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    if (tid == 0) s_tile = atomicAdd(counter, 1u);
    if (hist)
        for (int i = tid; i < HB * 256; i += F_THREADS) s_hist[i] = 0;
    __syncthreads();
    const long long tile = s_tile;
    const long long num_tiles = (n + F_TILE - 1) / F_TILE;
    const long long base = tile * F_TILE;
    const bool need_key = out_keys || out_kvalid || hist || drop_null_key;

    bool flag[F_ITEMS];
    unsigned rank[F_ITEMS];
    K key[F_ITEMS];
    V val[F_ITEMS];
    uint8_t kv[F_ITEMS];
    bool ext_max = false, ext_min = false;
#pragma unroll
    for (int j = 0; j < F_ITEMS; j++) {
        const long long row = base + (long long)j * F_THREADS + tid;
        bool f = row < n;
        key[j] = 0;
        val[j] = 0;
        kv[j] = 1;
        if (f) f = eval_preds(preds, row);
        if constexpr (KB > 0) {
            if (f && need_key) {
                bool ok;
                key[j] = encode_key<K>(ks, row, ok);
                kv[j] = ok;
                if (drop_null_key && !ok) f = false;
            }
        }
        if constexpr (VB > 0) {
            if (f) {
                if (vs.v && !__ldg(vs.v + row)) {
                    if (drop_null_val) f = false;
                } else {
                    val[j] = (V)load_w(vs.c, vs.w, row);
                    ext_max |= val[j] == (VB == 8 ? (V)LLONG_MAX : (V)INT_MAX);
                    ext_min |= val[j] == (VB == 8 ? (V)LLONG_MIN : (V)INT_MIN);
                }
            }
        }
        flag[j] = f;
        const unsigned m = __ballot_sync(FULL, f);
        if (lane == 0) s_cnt[j][warp] = __popc(m);
        rank[j] = __popc(m & lanemask_lt());
        if constexpr (KB > 0) {
            if (hist && f) {
#pragma unroll
                for (int d = 0; d < KB; d++) atomicAdd(&s_hist[d * 256 + (unsigned)((key[j] >> (8 * d)) & 255)], 1u);
            }
        }
    }
    const unsigned long long tb = tile_offsets(s_cnt, status, tile, num_tiles, out_count, &s_base);
#pragma unroll
    for (int j = 0; j < F_ITEMS; j++) {
        if (!flag[j]) continue;
        const long long pos = (long long)tb + s_cnt[j][warp] + rank[j];
        const long long row = base + (long long)j * F_THREADS + tid;
        if (out_ids) out_ids[pos] = (int)row;
        if constexpr (KB > 0) {
            if (out_keys) ((K *)out_keys)[pos] = key[j];
            if (out_kvalid) out_kvalid[pos] = kv[j];
        }
        if constexpr (VB > 0) {
            if (out_vals) ((V *)out_vals)[pos] = val[j];
        }
    }
    if (hist) {
        __syncthreads();
        for (int i = tid; i < HB * 256; i += F_THREADS)
            if (s_hist[i]) atomicAdd(&hist[i], s_hist[i]);
    }
    if constexpr (VB > 0) {
        if (extreme) {
            if (__any_sync(FULL, ext_max) && lane == 0) atomicOr(&extreme[0], 1u);
            if (__any_sync(FULL, ext_min) && lane == 0) atomicOr(&extreme[1], 1u);
        }
    }
}

cudaError_t launch_filter(long long n, const PredSet &preds, const KeySrc &key, int kb, const ValSrc &val,
                          int vb, int drop_null_key, int drop_null_val, int *out_ids, void *out_keys,
                          uint8_t *out_kvalid, void *out_vals, unsigned *hist, unsigned *extreme, void *scratch, long long *out_count, cudaStream_t st, long long *launches)
{
    cudaError_t e = cudaMemsetAsync(out_count, 0, sizeof(long long), st);
    if (e != cudaSuccess || n <= 0) return e;
    const long long tiles = (n + F_TILE - 1) / F_TILE;
    e = cudaMemsetAsync(scratch, 0, filter_scratch_bytes(n), st);
    if (e != cudaSuccess) return e;
    unsigned *counter = (unsigned *)scratch;
    unsigned long long *status = (unsigned long long *)((char *)scratch + 256);
    dim3 grid((unsigned)tiles), block(F_THREADS);
#define NG_FILTER(KB_, VB_)                                                                             \
    filter_kernel<KB_, VB_><<<grid, block, 0, st>>>(n, preds, key, val, drop_null_key, drop_null_val,   \
                                                    out_ids, out_keys, out_kvalid, out_vals, hist,      \
                                                    extreme, status, counter, out_count)
    const int k = kb == 8 ? 8 : (kb == 4 ? 4 : 0);
    const int v = val.c ? (vb == 8 ? 8 : 4) : 0;
    if (k == 0 && v == 0) NG_FILTER(0, 0);
    else if (k == 4 && v == 0) NG_FILTER(4, 0);
    else if (k == 4 && v == 4) NG_FILTER(4, 4);
    else if (k == 4 && v == 8) NG_FILTER(4, 8);
    else if (k == 8 && v == 0) NG_FILTER(8, 0);
    else if (k == 8 && v == 4) NG_FILTER(8, 4);
    else NG_FILTER(8, 8);
#undef NG_FILTER
    ++*launches;
    return cudaGetLastError();
}

// ------------------------------------------------------------------ a8 + a9
// round_half_away_from_zero(num / den), den > 0 (reading R6).
__device__ __forceinline__ long long div_round_half_away(__int128 num, long long den)
{
    __int128 mag = num < 0 ? -num : num;
    __int128 q = (2 * mag + den) / (2 * (__int128)den);
    return (long long)(num < 0 ? -q : q);
}

__global__ void __launch_bounds__(F_THREADS) finalize_kernel(FinalizeArgs A, unsigned long long *__restrict__ status,
                                                             unsigned *__restrict__ counter)
{
    __shared__ unsigned s_tile;
    __shared__ unsigned s_cnt[F_ITEMS][F_WARPS];
    __shared__ unsigned long long s_base;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const long long n = *A.d_nrp;
    const long long num_tiles = (n + F_TILE - 1) / F_TILE;
    if (tid == 0) s_tile = atomicAdd(counter, 1u);
    __syncthreads();
    const long long tile = s_tile;
    if (tile >= num_tiles) return;  // grid sized for the R' upper bound
    const long long base = tile * F_TILE;

    bool flag[F_ITEMS];
    unsigned rank[F_ITEMS];
    long long value[F_ITEMS];
    uint8_t valid[F_ITEMS], pass[F_ITEMS];
#pragma unroll
    for (int j = 0; j < F_ITEMS; j++) {
        const long long i = base + (long long)j * F_THREADS + tid;
        bool in = i < n;
        value[j] = 0;
        valid[j] = 0;
        pass[j] = 0;
        if (in) {
            const bool kval = A.kvalid ? A.kvalid[i] != 0 : true;
            const long long c = kval ? A.cnt[i] : 0;     // NULL key: empty subquery (R2)
            const long long acc = A.acc[i];
            bool vv = true;
            long long v = 0;
            switch (A.agg) {
            case MIN: case MAX: case SUM: vv = c > 0; v = acc; break;
            case COUNT: v = c; break;
            case AVG: vv = c > 0; if (vv) v = div_round_half_away((__int128)acc * 1000000, c); break;
            case EXISTS: v = c > 0; break;
            default: v = c == 0; break;
            }
            bool p;
            if (A.agg == EXISTS || A.agg == NOT_EXISTS) {
                p = v != 0;
            } else {
                const int row = A.ids[i];
                const bool xv = !(A.x_valid && !A.x_valid[row]);
                p = false;
                if (vv && xv) {
                    const __int128 x = load_w(A.x_col, A.x_w, row);
                    if (A.agg == AVG)
                        p = cmp_rt<__int128>((__int128)A.a * x * c, A.outer_op, (__int128)A.b * acc);
                    else
                        p = cmp_rt<__int128>((__int128)A.a * x, A.outer_op, (__int128)A.b * v);
                }
            }
            value[j] = vv ? v : 0;
            valid[j] = vv;
            pass[j] = p;
            in = A.emit_all ? true : p;
        }
        flag[j] = in;
        const unsigned m = __ballot_sync(FULL, in);
        if (lane == 0) s_cnt[j][warp] = __popc(m);
        rank[j] = __popc(m & lanemask_lt());
    }
    const unsigned long long tb = tile_offsets(s_cnt, status, tile, num_tiles, A.out_count, &s_base);
#pragma unroll
    for (int j = 0; j < F_ITEMS; j++) {
        if (!flag[j]) continue;
        const long long i = base + (long long)j * F_THREADS + tid;
        const long long pos = (long long)tb + s_cnt[j][warp] + rank[j];
        A.out_ids[pos] = A.row_id_base + A.ids[i];
        A.out_vals[pos] = value[j];
        A.out_valid[pos] = valid[j];
        A.out_passed[pos] = pass[j];
        if (A.out_sum) {
            const bool kval = A.kvalid ? A.kvalid[i] != 0 : true;
            A.out_sum[pos] = kval ? A.acc[i] : 0;
            A.out_cnt[pos] = kval ? A.cnt[i] : 0;
        }
    }
}

cudaError_t launch_finalize(const FinalizeArgs &a, cudaStream_t st, long long *launches)
{
    cudaError_t e = cudaMemsetAsync(a.out_count, 0, sizeof(long long), st);
    if (e != cudaSuccess || a.n_rp_max <= 0) return e;
    e = cudaMemsetAsync(a.scratch, 0, filter_scratch_bytes(a.n_rp_max), st);
    if (e != cudaSuccess) return e;
    const long long tiles = (a.n_rp_max + F_TILE - 1) / F_TILE;
    finalize_kernel<<<(unsigned)tiles, F_THREADS, 0, st>>>(a, (unsigned long long *)((char *)a.scratch + 256),
                                                         (unsigned *)a.scratch);
    ++*launches;
    return cudaGetLastError();
}

// ------------------------------------------------------------------ partials
__global__ void init_partials_kernel(long long n, long long acc0, long long *__restrict__ acc,
                                     long long *__restrict__ cnt)
{
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        acc[i] = acc0;
        cnt[i] = 0;
    }
}

cudaError_t launch_init_partials(long long n, int agg, long long *acc, long long *cnt, cudaStream_t st,
                                 long long *launches)
{
    if (n <= 0) return cudaSuccess;
    long long acc0 = agg == MIN ? LLONG_MAX : (agg == MAX ? LLONG_MIN : 0);
    long long blocks = (n + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    init_partials_kernel<<<(unsigned)blocks, 256, 0, st>>>(n, acc0, acc, cnt);
    ++*launches;
    return cudaGetLastError();
}

// ------------------------------------------------------------------ column min / max
// (for the SUM/AVG overflow pre-check, reading R5)
__global__ void minmax_init_kernel(long long *out)
{
    out[0] = LLONG_MAX;
    out[1] = LLONG_MIN;
}

__global__ void minmax_kernel(const void *__restrict__ col, int w, const uint8_t *__restrict__ valid, long long n,
                              long long *__restrict__ out)
{
    long long mn = LLONG_MAX, mx = LLONG_MIN;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        if (valid && !valid[i]) continue;
        const long long v = load_w(col, w, i);
        mn = min(mn, v);
        mx = max(mx, v);
    }
    for (int o = 16; o > 0; o >>= 1) {
        mn = min(mn, __shfl_xor_sync(FULL, mn, o));
        mx = max(mx, __shfl_xor_sync(FULL, mx, o));
    }
    if ((threadIdx.x & 31) == 0) {
        atomicMin(&out[0], mn);
        atomicMax(&out[1], mx);
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
