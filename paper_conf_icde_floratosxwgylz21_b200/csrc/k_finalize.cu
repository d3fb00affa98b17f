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

// ------------------------------------------------------------------ column min / max
// (for the SUM/AVG overflow pre-check, reading R5)
// (and out[2] != 0 iff some row is smaller than its predecessor: the
// column is not stored in key order -- the index build's sort-free path)
__global__ void minmax_init_kernel(long long *out)
{
    out[0] = LLONG_MAX;
    out[1] = LLONG_MIN;
    out[2] = 0;
}

__global__ void minmax_kernel(const void *__restrict__ col, int w, const uint8_t *__restrict__ valid, long long n,
                              long long *__restrict__ out)
{
    long long mn = LLONG_MAX, mx = LLONG_MIN;
    bool desc = false;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        if (valid && !valid[i]) continue;
        const long long v = load_w(col, w, i);
        mn = min(mn, v);
        mx = max(mx, v);
        if (i > 0 && !valid) desc |= load_w(col, w, i - 1) > v;
    }
    for (int o = 16; o > 0; o >>= 1) {
        mn = min(mn, __shfl_xor_sync(FULL, mn, o));
        mx = max(mx, __shfl_xor_sync(FULL, mx, o));
    }
    desc = __any_sync(FULL, desc);
    if ((threadIdx.x & 31) == 0) {
        atomicMin(&out[0], mn);
        atomicMax(&out[1], mx);
        if (desc) atomicOr((unsigned long long *)&out[2], 1ull);
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
