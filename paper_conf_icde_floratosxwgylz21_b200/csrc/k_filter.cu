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
// s_cnt holds counts on entry and exclusive offsets on exit.  The decoupled
// look-back is done by the whole CTA (the other warps would only wait at the
// barrier): thread t inspects predecessor tile-1-t, so one L2 round trip
// covers 256 predecessors; the nearest inclusive prefix ends the walk.
__device__ __forceinline__ unsigned long long tile_offsets(unsigned (*s_cnt)[F_WARPS], unsigned long long *status,
                                                           long long tile, long long num_tiles,
                                                           long long *out_count,
                                                           unsigned long long *s_base)
{
    __shared__ unsigned s_total;
    __shared__ int s_stop;
    __shared__ unsigned long long s_wsum[F_WARPS];
    __syncthreads();
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid < 32) {
        unsigned *flat = &s_cnt[0][0];
        unsigned c[4], s = 0;
#pragma unroll
        for (int q = 0; q < 4; q++) { c[q] = flat[4 * lane + q]; s += c[q]; }
        unsigned incl = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            unsigned t = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += t;
        }
        unsigned run = incl - s;
        const unsigned total = __shfl_sync(FULL, incl, 31);
#pragma unroll
        for (int q = 0; q < 4; q++) { unsigned t = c[q]; flat[4 * lane + q] = run; run += t; }
        if (lane == 0) {
            s_total = total;
            st_relaxed_u64(status + tile, (tile == 0 ? ST_INC : ST_AGG) | total);
            s_stop = 0x7fffffff;
        }
    }
    __syncthreads();
    const unsigned long long total = s_total;
    unsigned long long excl = 0;
    if (tile > 0) {
        for (long long round = 0;; round += F_THREADS) {
            const long long pred = tile - 1 - round - tid;
            unsigned long long sv = pred >= 0 ? ld_relaxed_u64(status + pred) : ST_INC;
            while ((sv >> 62) == 0) sv = ld_relaxed_u64(status + pred);
            if ((sv >> 62) == 2) atomicMin(&s_stop, tid);
            __syncthreads();
            const int stop = s_stop;                       // nearest inclusive predecessor
            unsigned long long v = tid <= stop ? (sv & ST_VAL) : 0;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
            if (lane == 0) s_wsum[warp] = v;
            __syncthreads();
#pragma unroll
            for (int w = 0; w < F_WARPS; w++) excl += s_wsum[w];
            if (stop != 0x7fffffff) break;
            __syncthreads();                               // s_wsum reuse
        }
        if (tid == 0) st_relaxed_u64(status + tile, ST_INC | (excl + total));
    }
    if (tid == 0 && tile == num_tiles - 1) *out_count = (long long)(excl + total);
    (void)s_base;
    __syncthreads();
    return excl;
}

// Load items j = 0..F_ITEMS-1 of one column for the rows still alive in
// `live` (bit j), all loads issued before any use (memory-level parallelism:
// 16 independent coalesced loads per thread).
template <int W>
__device__ __forceinline__ void load_items(const void *__restrict__ col, long long base, int tid, unsigned live,
                                           long long (&x)[F_ITEMS])
{
#pragma unroll
    for (int j = 0; j < F_ITEMS; j++) {
        const long long row = base + (long long)j * F_THREADS + tid;
        x[j] = 0;
        if (live >> j & 1u) {
            if constexpr (W == 4) x[j] = __ldg((const int *)col + row);
            else x[j] = __ldg((const long long *)col + row);
        }
    }
}

__device__ __forceinline__ unsigned valid_bits(const uint8_t *__restrict__ v, long long base, int tid, unsigned live)
{
    if (!v) return live;
    unsigned out = 0;
#pragma unroll
    for (int j = 0; j < F_ITEMS; j++) {
        const long long row = base + (long long)j * F_THREADS + tid;
        if ((live >> j & 1u) && __ldg(v + row)) out |= 1u << j;
    }
    return out;
}

template <int OP>
__device__ __forceinline__ unsigned cmp_bits(const long long (&x)[F_ITEMS], const long long (&y)[F_ITEMS])
{
    unsigned m = 0;
#pragma unroll
    for (int j = 0; j < F_ITEMS; j++)
        if (cmp_ct<OP>(x[j], y[j])) m |= 1u << j;
    return m;
}

// Conjunction of the local predicates for this thread's 16 rows, evaluated
// predicate by predicate (column-major) so each predicate's 16 loads are in
// flight together.  NULL operands make a predicate not TRUE (reading R2).
__device__ __forceinline__ unsigned eval_preds_tile(const PredSet &P, long long base, int tid, unsigned live)
{
    for (int k = 0; k < P.n && live; k++) {
        const DevPred &p = P.p[k];
        live = valid_bits(p.valid, base, tid, live);
        long long x[F_ITEMS], y[F_ITEMS];
        if (p.w == 4) load_items<4>(p.col, base, tid, live, x);
        else load_items<8>(p.col, base, tid, live, x);
        if (p.rhs) {
            live = valid_bits(p.rhs_valid, base, tid, live);
            if (p.rhs_w == 4) load_items<4>(p.rhs, base, tid, live, y);
            else load_items<8>(p.rhs, base, tid, live, y);
        } else {
#pragma unroll
            for (int j = 0; j < F_ITEMS; j++) y[j] = p.lit;
        }
        unsigned m;
        switch (p.op) {
        case EQ: m = cmp_bits<EQ>(x, y); break;
        case NE: m = cmp_bits<NE>(x, y); break;
        case LT: m = cmp_bits<LT>(x, y); break;
        case LE: m = cmp_bits<LE>(x, y); break;
        case GT: m = cmp_bits<GT>(x, y); break;
        default: m = cmp_bits<GE>(x, y); break;
        }
        live &= m;
    }
    return live;
}

template <int KB, int VB>
__global__ void __launch_bounds__(F_THREADS, 2)
filter_kernel(long long n, PredSet preds, KeySrc ks, ValSrc vs, int drop_null_key, int drop_null_val,
              int *__restrict__ out_ids, void *__restrict__ out_keys, uint8_t *__restrict__ out_kvalid,
              void *__restrict__ out_vals, unsigned long long *__restrict__ keymask,
              unsigned *__restrict__ extreme, unsigned long long *__restrict__ status,
              unsigned *__restrict__ counter, long long *__restrict__ out_count)
{
    using K = typename std::conditional<KB == 8, uint64_t, uint32_t>::type;
    using V = typename std::conditional<VB == 8, long long, int>::type;
    __shared__ unsigned s_tile;
    __shared__ unsigned s_cnt[F_ITEMS][F_WARPS];
    __shared__ unsigned long long s_base;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    if (tid == 0) s_tile = atomicAdd(counter, 1u);
    __syncthreads();
    const long long tile = s_tile;
    const long long num_tiles = (n + F_TILE - 1) / F_TILE;
    const long long base = tile * F_TILE;

    // rows of this thread: base + j*256 + tid (coalesced per warp)
    unsigned live = 0;
#pragma unroll
    for (int j = 0; j < F_ITEMS; j++)
        if (base + (long long)j * F_THREADS + tid < n) live |= 1u << j;
    live = eval_preds_tile(preds, base, tid, live);

    K key[F_ITEMS];
    unsigned kvalid = live;
    if constexpr (KB > 0) {
        // encoded correlated key (order-preserving unsigned)
        kvalid = valid_bits(ks.v0, base, tid, live);
        if (ks.n_key == 2) {
            kvalid = valid_bits(ks.v1, base, tid, kvalid);
            long long a[F_ITEMS], b[F_ITEMS];
            load_items<4>(ks.c0, base, tid, live, a);
            load_items<4>(ks.c1, base, tid, live, b);
#pragma unroll
            for (int j = 0; j < F_ITEMS; j++)
                key[j] = (K)(((uint64_t)enc32((int)a[j]) << 32) | (uint64_t)enc32((int)b[j]));
        } else {
            long long a[F_ITEMS];
            if (ks.w0 == 4) load_items<4>(ks.c0, base, tid, live, a);
            else load_items<8>(ks.c0, base, tid, live, a);
#pragma unroll
            for (int j = 0; j < F_ITEMS; j++) {
                if constexpr (KB == 4) key[j] = (K)enc32((int)a[j]);
                else key[j] = (K)enc64(a[j]);
            }
        }
        if (drop_null_key) live = kvalid;
    }
    V val[F_ITEMS];
    bool ext_max = false, ext_min = false;
    if constexpr (VB > 0) {
        const unsigned vv = valid_bits(vs.v, base, tid, live);
        if (drop_null_val) live = vv;
        long long a[F_ITEMS];
        if (vs.w == 4) load_items<4>(vs.c, base, tid, live, a);
        else load_items<8>(vs.c, base, tid, live, a);
#pragma unroll
        for (int j = 0; j < F_ITEMS; j++) {
            val[j] = (V)a[j];
            if (live >> j & 1u) {
                ext_max |= val[j] == (VB == 8 ? (V)LLONG_MAX : (V)INT_MAX);
                ext_min |= val[j] == (VB == 8 ? (V)LLONG_MIN : (V)INT_MIN);
            }
        }
    }
    unsigned rank[F_ITEMS];
    unsigned long long kand = ~0ull, kor = 0ull;
#pragma unroll
    for (int j = 0; j < F_ITEMS; j++) {
        const bool f = live >> j & 1u;
        const unsigned m = __ballot_sync(FULL, f);
        if (lane == 0) s_cnt[j][warp] = __popc(m);
        rank[j] = __popc(m & lanemask_lt());
        if constexpr (KB > 0) {
            if (f) {
                kand &= (unsigned long long)key[j];
                kor |= (unsigned long long)key[j];
            }
        }
    }
    const unsigned long long tb = tile_offsets(s_cnt, status, tile, num_tiles, out_count, &s_base);
#pragma unroll
    for (int j = 0; j < F_ITEMS; j++) {
        if (!(live >> j & 1u)) continue;
        const long long pos = (long long)tb + s_cnt[j][warp] + rank[j];
        const long long row = base + (long long)j * F_THREADS + tid;
        if (out_ids) out_ids[pos] = (int)row;
        if constexpr (KB > 0) {
            if (out_keys) ((K *)out_keys)[pos] = key[j];
            if (out_kvalid) out_kvalid[pos] = (kvalid >> j) & 1u;
        }
        if constexpr (VB > 0) {
            if (out_vals) ((V *)out_vals)[pos] = val[j];
        }
    }
    if constexpr (KB > 0) {
        if (keymask) {  // bits shared by every survivor key: which radix digits are constant
            const unsigned alo = __reduce_and_sync(FULL, (unsigned)kand), ahi = __reduce_and_sync(FULL, (unsigned)(kand >> 32));
            const unsigned olo = __reduce_or_sync(FULL, (unsigned)kor), ohi = __reduce_or_sync(FULL, (unsigned)(kor >> 32));
            if (lane == 0) {
                atomicAnd(&keymask[0], ((unsigned long long)ahi << 32) | alo);
                atomicOr(&keymask[1], ((unsigned long long)ohi << 32) | olo);
            }
        }
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
                          uint8_t *out_kvalid, void *out_vals, unsigned long long *keymask, unsigned *extreme,
                          void *scratch, long long *out_count, cudaStream_t st, long long *launches)
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
                                                    out_ids, out_keys, out_kvalid, out_vals, keymask,   \
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
