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
#define NG_F_ITEMS 4   // rows per thread per tile (rolled loop: also the serial memory-latency chain)
#endif
constexpr int F_ITEMS = NG_F_ITEMS;
constexpr int F_TILE = F_THREADS * F_ITEMS;

size_t finalize_scratch_bytes(long long n)
{
    long long tiles = (n + F_TILE - 1) / F_TILE;
    return (size_t)(tiles + 1) * 8 + 256;
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

// The per-row evaluation (int128 compares, the rare int128 division) is
// large; unrolled over the tile's 16 rows per thread it made a ~175 KB kernel
// whose instruction-cache misses dominated small R' (SF1 Q17: 69 us for 6.3k
// rows).  Rows are therefore evaluated in a rolled loop and staged in shared
// memory (value, valid|passed bits, one ballot per (row group, warp)).
__global__ void __launch_bounds__(F_THREADS) finalize_kernel(FinalizeArgs A, unsigned long long *__restrict__ status,
                                                             unsigned *__restrict__ counter)
{
    __shared__ unsigned s_tile;
    __shared__ unsigned s_cnt[F_ITEMS][F_WARPS];
    __shared__ unsigned s_bal[F_ITEMS][F_WARPS];
    __shared__ long long s_val[F_ITEMS][F_THREADS];
    __shared__ uint8_t s_vp[F_ITEMS][F_THREADS];   // bit 0 valid, bit 1 passed
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const unsigned lt = lanemask_lt();
    const long long n = *A.d_nrp;
    const long long num_tiles = (n + F_TILE - 1) / F_TILE;
    // persistent: the grid is sized for the host's upper bound of |R'| but
    // capped; CTAs take tiles of the ACTUAL |R'| until none are left
    for (;;) {
        if (tid == 0) s_tile = atomicAdd(counter, 1u);
        __syncthreads();
        const long long tile = s_tile;
        __syncthreads();
        if (tile >= num_tiles) return;
        const long long base = tile * F_TILE;

        // the rows' inputs are loaded for all F_ITEMS rows first (independent
        // loads in flight together; the rolled evaluation below would
        // otherwise wait one memory round trip per row)
        long long r_acc[F_ITEMS], r_cnt[F_ITEMS], r_x[F_ITEMS];
        int r_row[F_ITEMS];
        bool r_kval[F_ITEMS], r_xv[F_ITEMS];
#pragma unroll
        for (int j = 0; j < F_ITEMS; j++) {
            const long long i = base + (long long)j * F_THREADS + tid;
            r_acc[j] = r_cnt[j] = r_x[j] = 0;
            r_row[j] = 0;
            r_kval[j] = false;
            r_xv[j] = false;
            if (i < n) {
                r_kval[j] = A.kvalid ? A.kvalid[i] != 0 : true;
                const long long g = A.map ? (long long)A.map[i] : i;  // cached result slot
                r_cnt[j] = A.cnt[g];
                r_acc[j] = A.acc[g];
                r_row[j] = A.ids[i];
            }
        }
        if (A.agg != EXISTS && A.agg != NOT_EXISTS) {
#pragma unroll
            for (int j = 0; j < F_ITEMS; j++) {
                const long long i = base + (long long)j * F_THREADS + tid;
                if (i < n) {
                    r_xv[j] = !(A.x_valid && !A.x_valid[r_row[j]]);
                    r_x[j] = load_w(A.x_col, A.x_w, r_row[j]);
                }
            }
        }
#pragma unroll 1
        for (int j = 0; j < F_ITEMS; j++) {
            const long long i = base + (long long)j * F_THREADS + tid;
            bool in = i < n;
            long long value = 0;
            uint8_t vp = 0;
            if (in) {
                const bool kval = r_kval[j];
                const long long g = A.map ? (long long)A.map[i] : i;
                const long long c = kval ? r_cnt[j] : 0;     // NULL key: empty subquery (R2)
                long long acc = r_acc[j];
                bool vv = true;
                if (A.acc_hi && c > 0) {   // split SUM: hi * 2^32 + lo, exact (reading R5)
                    const __int128 t = (__int128)A.acc_hi[g] * 4294967296ll + (__int128)(unsigned long long)acc;
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
                    const bool xv = r_xv[j];
                    p = false;
                    if (vv && xv) {
                        const __int128 x = r_x[j];
                        if (A.agg == AVG)
                            p = cmp_rt<__int128>((__int128)A.a * x * c, A.outer_op, (__int128)A.b * acc);
                        else
                            p = cmp_rt<__int128>((__int128)A.a * x, A.outer_op, (__int128)A.b * v);
                    }
                }
                value = vv ? v : 0;
                vp = (uint8_t)((vv ? 1 : 0) | (p ? 2 : 0));
                in = A.emit_all ? true : p;
            }
            s_val[j][tid] = value;
            s_vp[j][tid] = vp;
            const unsigned m = __ballot_sync(FULL, in);
            if (lane == 0) {
                s_cnt[j][warp] = __popc(m);
                s_bal[j][warp] = m;
            }
        }
        const unsigned long long tb = tile_offsets<F_ITEMS, F_THREADS>(s_cnt, status, tile, num_tiles, A.out_count);
#pragma unroll 1
        for (int j = 0; j < F_ITEMS; j++) {
            const unsigned m = s_bal[j][warp];
            if (!((m >> lane) & 1u)) continue;
            const long long i = base + (long long)j * F_THREADS + tid;
            const long long pos = (long long)tb + s_cnt[j][warp] + __popc(m & lt);
            const uint8_t vp = s_vp[j][tid];
            A.out_ids[pos] = A.row_id_base + A.ids[i];
            A.out_vals[pos] = s_val[j][tid];
            A.out_valid[pos] = vp & 1;
            A.out_passed[pos] = (vp >> 1) & 1;
            if (A.out_sum) {
                const bool kval = A.kvalid ? A.kvalid[i] != 0 : true;
                const long long g = A.map ? (long long)A.map[i] : i;
                long long sum = kval ? A.acc[g] : 0;
                if (A.acc_hi && kval)
                    sum = (long long)((__int128)A.acc_hi[g] * 4294967296ll + (__int128)(unsigned long long)sum);
                A.out_sum[pos] = sum;
                A.out_cnt[pos] = kval ? A.cnt[g] : 0;
            }
        }
        __syncthreads();   // shared staging is rewritten by the next tile
    }
}

cudaError_t launch_finalize(const FinalizeArgs &a, cudaStream_t st, long long *launches, bool prezeroed)
{
    cudaError_t e = prezeroed ? cudaSuccess : cudaMemsetAsync(a.out_count, 0, sizeof(long long), st);
    if (e != cudaSuccess || a.n_rp_max <= 0) return e;
    if (!prezeroed) {
        e = cudaMemsetAsync(a.scratch, 0, finalize_scratch_bytes(a.n_rp_max), st);
        if (e != cudaSuccess) return e;
    }
    long long tiles = (a.n_rp_max + F_TILE - 1) / F_TILE;
    int cap = 0;
    e = per_device_setup((const void *)finalize_kernel, 0, &cap, [](int dev, int *v) {
        int sms = 0;
        cudaError_t e2 = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        *v = sms * 4;
        return e2;
    });
    if (e != cudaSuccess) return e;
    if (tiles > cap) tiles = cap;
    finalize_kernel<<<(unsigned)tiles, F_THREADS, 0, st>>>(a, (unsigned long long *)((char *)a.scratch + 256),
                                                         (unsigned *)a.scratch);
    ++*launches;
    return cudaGetLastError();
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
