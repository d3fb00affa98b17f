// k_collect.cu -- type-J subquery results as two-level arrays, and the IN
// selection that consumes them; plus the column materialisation of device
// int64 vectors (results, collections) used to chain levels and joins.
//
// PAPER.md P:231 (§III-B): "type-J correlated subqueries are different
// because their results have variable lengths ... we use a two-level arrays
// to store the results of subquery evaluations.  The first level is to store
// the lengths of variable results for each subquery evaluation and the second
// is to store the results."  With the sorted correlated-column index
// the result of r's subquery is one or two contiguous runs of the co-sorted
// payload, so the engine builds the arrays in three vectorised steps:
//   1. collect_bounds_kernel  -- per R' tuple: binary search -> the runs
//      [a0,b0) u [a1,b1) and their total length (level 1);
//   2. scan_*                 -- exclusive prefix sum of the lengths into
//      offsets[0..n] (int64; three-phase: tile sums, one-CTA scan of the
//      tile sums, tile-local scan + base);
//   3. collect_fill_kernel    -- element-parallel: each level-2 slot finds
//      its owner by binary search over the offsets (perfect load balance for
//      skewed lengths) and copies payload[run position] widened to int64.
// Runs follow the range table of k_range.cu (r.key OP s.key, S' ascending).
#include <climits>

#include "internal.h"

namespace ng {

constexpr int C_THREADS = 256;
constexpr int SCAN_ITEMS = 8;
constexpr int SCAN_TILE = C_THREADS * SCAN_ITEMS;

struct Runs {
    int a0, b0, a1, b1;
};

size_t collect_scratch_bytes(long long n_rp_max)
{
    const long long n = n_rp_max > 0 ? n_rp_max : 1;
    const long long tiles = (n + 1 + SCAN_TILE - 1) / SCAN_TILE;
    return 256 + (size_t)n * sizeof(Runs) + (size_t)(tiles + 1) * 8;
}

template <typename K>
__device__ __forceinline__ int lb_search(const K *__restrict__ a, int lo, int hi, K k)
{
    while (lo < hi) {
        const int mid = (int)(((unsigned)lo + (unsigned)hi) >> 1);
        if (__ldg(a + mid) < k) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}
template <typename K>
__device__ __forceinline__ int ub_search(const K *__restrict__ a, int lo, int hi, K k)
{
    while (lo < hi) {
        const int mid = (int)(((unsigned)lo + (unsigned)hi) >> 1);
        if (__ldg(a + mid) <= k) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

// Step 1: runs + length of every R' tuple; level-1 row ids (int64, + base).
template <typename K>
__global__ void __launch_bounds__(C_THREADS)
collect_bounds_kernel(const long long *__restrict__ d_nrp, const int *__restrict__ ids,
                      const K *__restrict__ rkeys, const uint8_t *__restrict__ rkvalid,
                      const K *__restrict__ skeys, int N, int op, long long base,
                      Runs *__restrict__ runs, long long *__restrict__ lens, long long *__restrict__ row_ids)
{
    const long long n = *d_nrp;
    for (long long i = blockIdx.x * (long long)C_THREADS + threadIdx.x; i < n;
         i += (long long)gridDim.x * C_THREADS) {
        Runs q{0, 0, 0, 0};
        if (!rkvalid || rkvalid[i]) {   // NULL r.key: empty subquery (reading R2)
            const K k = rkeys[i];
            const int lb = lb_search(skeys, 0, N, k);
            const int ub = ub_search(skeys, lb, N, k);
            switch (op) {
            case EQ: q = {lb, ub, 0, 0}; break;
            case LT: q = {ub, N, 0, 0}; break;   // s.key > r.key
            case LE: q = {lb, N, 0, 0}; break;   // s.key >= r.key
            case GT: q = {0, lb, 0, 0}; break;   // s.key < r.key
            case GE: q = {0, ub, 0, 0}; break;   // s.key <= r.key
            default: q = {0, lb, ub, N}; break;  // '!='
            }
        }
        runs[i] = q;
        lens[i] = (long long)(q.b0 - q.a0) + (q.b1 - q.a1);
        row_ids[i] = base + ids[i];
    }
}

// Step 2a: per-tile sums over n_v + add entries (v read as 0 past n_v).
__global__ void __launch_bounds__(C_THREADS)
scan_tile_sums_kernel(const long long *__restrict__ v, const long long *__restrict__ d_n, long long add,
                      long long *__restrict__ tile_sum)
{
    __shared__ long long s_w[C_THREADS / 32];
    const long long n_v = *d_n, n = n_v + add;
    const long long t0 = (long long)blockIdx.x * SCAN_TILE;
    if (t0 >= n) return;
    long long s = 0;
#pragma unroll
    for (int j = 0; j < SCAN_ITEMS; j++) {
        const long long i = t0 + (long long)j * C_THREADS + threadIdx.x;
        if (i < n_v) s += v[i];
    }
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(FULL, s, o);
    if ((threadIdx.x & 31) == 0) s_w[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        long long t = 0;
        for (int w = 0; w < C_THREADS / 32; w++) t += s_w[w];
        tile_sum[blockIdx.x] = t;
    }
}

// Step 2b: one CTA turns the tile sums into exclusive tile bases.
__global__ void __launch_bounds__(1024) scan_tile_bases_kernel(long long *__restrict__ tile_sum,
                                                               const long long *__restrict__ d_n, long long add)
{
    __shared__ long long s_w[32];
    __shared__ long long s_carry;
    const long long n = *d_n + add;
    const long long tiles = (n + SCAN_TILE - 1) / SCAN_TILE;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) s_carry = 0;
    __syncthreads();
    for (long long c0 = 0; c0 < tiles; c0 += 1024) {
        const long long i = c0 + tid;
        const long long x = i < tiles ? tile_sum[i] : 0;
        long long incl = x;
        for (int o = 1; o < 32; o <<= 1) {
            const long long y = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += y;
        }
        if (lane == 31) s_w[warp] = incl;
        __syncthreads();
        if (warp == 0) {
            long long w = s_w[lane], wi = w;
            for (int o = 1; o < 32; o <<= 1) {
                const long long y = __shfl_up_sync(FULL, wi, o);
                if (lane >= o) wi += y;
            }
            s_w[lane] = wi - w;   // exclusive warp base
        }
        __syncthreads();
        const long long carry = s_carry;
        if (i < tiles) tile_sum[i] = carry + s_w[warp] + incl - x;
        __syncthreads();
        if (tid == 1023) s_carry = carry + s_w[warp] + incl;
        __syncthreads();
    }
}

// Step 2c: exclusive scan within each tile plus its base: out[i] = sum(v[0..i)).
// Entries i in [n_v, n) read v as 0, so out[n_v] is the grand total (also
// written to *total).
__global__ void __launch_bounds__(C_THREADS)
scan_apply_kernel(const long long *__restrict__ v, const long long *__restrict__ d_n, long long add,
                  const long long *__restrict__ tile_base, long long *__restrict__ out, long long *__restrict__ total)
{
    __shared__ long long s_w[C_THREADS / 32];
    const long long n_v = *d_n, n = n_v + add;
    const long long t0 = (long long)blockIdx.x * SCAN_TILE;
    if (t0 >= n) return;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // thread-contiguous items: thread t owns [t0 + t*ITEMS, t0 + (t+1)*ITEMS)
    long long x[SCAN_ITEMS], s = 0;
#pragma unroll
    for (int j = 0; j < SCAN_ITEMS; j++) {
        const long long i = t0 + (long long)tid * SCAN_ITEMS + j;
        x[j] = i < n_v ? v[i] : 0;
        s += x[j];
    }
    long long incl = s;
    for (int o = 1; o < 32; o <<= 1) {
        const long long y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) s_w[warp] = incl;
    __syncthreads();
    long long wb = 0;
    for (int w = 0; w < warp; w++) wb += s_w[w];
    long long run = tile_base[blockIdx.x] + wb + incl - s;
#pragma unroll
    for (int j = 0; j < SCAN_ITEMS; j++) {
        const long long i = t0 + (long long)tid * SCAN_ITEMS + j;
        if (i < n) out[i] = run;
        if (i == n_v && total) *total = run;
        run += x[j];
    }
}

// Step 3: level-2 fill, one thread per output slot.
template <int VB>
__global__ void __launch_bounds__(C_THREADS)
collect_fill_kernel(const long long *__restrict__ d_nrp, const long long *__restrict__ offsets,
                    const Runs *__restrict__ runs, const long long *__restrict__ row_ids,
                    const void *__restrict__ payload, long long total, long long *__restrict__ values,
                    long long *__restrict__ owner)
{
    const long long n = *d_nrp;
    for (long long e = blockIdx.x * (long long)C_THREADS + threadIdx.x; e < total;
         e += (long long)gridDim.x * C_THREADS) {
        // owner r: the last r with offsets[r] <= e (offsets non-decreasing;
        // empty lists share an offset with their successor, so take the last)
        long long lo = 0, hi = n;   // search in [0, n)
        while (hi - lo > 1) {
            const long long mid = (lo + hi) >> 1;
            if (__ldg(offsets + mid) <= e) lo = mid;
            else hi = mid;
        }
        const long long r = lo;
        const Runs q = runs[r];
        const long long j = e - offsets[r];
        const long long l0 = q.b0 - q.a0;
        const long long p = j < l0 ? q.a0 + j : q.a1 + (j - l0);
        values[e] = VB == 4 ? (long long)__ldg((const int *)payload + p) : __ldg((const long long *)payload + p);
        owner[e] = row_ids[r];
    }
}

static unsigned grid_for(long long n, long long cap)
{
    long long b = (n + C_THREADS - 1) / C_THREADS;
    if (b < 1) b = 1;
    if (b > cap) b = cap;
    return (unsigned)b;
}

// Exclusive scan of v[0..n_v) into out[0..n_v] (n_v on the device, <= n_max).
static cudaError_t launch_scan_excl(const long long *v, const long long *d_n, long long n_max, long long *out,
                                    long long *total, long long *tile_sum, cudaStream_t st, long long *launches)
{
    const long long tiles = (n_max + 1 + SCAN_TILE - 1) / SCAN_TILE;
    scan_tile_sums_kernel<<<(unsigned)tiles, C_THREADS, 0, st>>>(v, d_n, 1, tile_sum);
    scan_tile_bases_kernel<<<1, 1024, 0, st>>>(tile_sum, d_n, 1);
    scan_apply_kernel<<<(unsigned)tiles, C_THREADS, 0, st>>>(v, d_n, 1, tile_sum, out, total);
    *launches += 3;
    return cudaGetLastError();
}

cudaError_t launch_collect_bounds(int kb, int op, long long n_rp_max, const long long *d_nrp, const int *ids,
                                  const void *rkeys, const uint8_t *rkvalid, const void *skeys, long long ns,
                                  long long base, void *scratch, long long *lens, long long *row_ids,
                                  long long *offsets, long long *total, cudaStream_t st, long long *launches)
{
    Runs *runs = (Runs *)((char *)scratch + 256);
    long long *tile_sum = (long long *)(runs + (n_rp_max > 0 ? n_rp_max : 1));
    const unsigned g = grid_for(n_rp_max, 148 * 16);
    if (kb == 4)
        collect_bounds_kernel<uint32_t><<<g, C_THREADS, 0, st>>>(d_nrp, ids, (const uint32_t *)rkeys, rkvalid,
                                                                 (const uint32_t *)skeys, (int)ns, op, base, runs,
                                                                 lens, row_ids);
    else
        collect_bounds_kernel<uint64_t><<<g, C_THREADS, 0, st>>>(d_nrp, ids, (const uint64_t *)rkeys, rkvalid,
                                                                 (const uint64_t *)skeys, (int)ns, op, base, runs,
                                                                 lens, row_ids);
    ++*launches;
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    return launch_scan_excl(lens, d_nrp, n_rp_max, offsets, total, tile_sum, st, launches);
}

cudaError_t launch_collect_fill(int vb, const long long *d_nrp, const long long *offsets, const void *scratch,
                                const long long *row_ids, const void *payload, long long total, long long *values,
                                long long *owner, cudaStream_t st, long long *launches)
{
    if (total <= 0) return cudaSuccess;
    const Runs *runs = (const Runs *)((const char *)scratch + 256);
    const unsigned g = grid_for(total, 148 * 32);
    if (vb == 4)
        collect_fill_kernel<4><<<g, C_THREADS, 0, st>>>(d_nrp, offsets, runs, row_ids, payload, total, values, owner);
    else
        collect_fill_kernel<8><<<g, C_THREADS, 0, st>>>(d_nrp, offsets, runs, row_ids, payload, total, values, owner);
    ++*launches;
    return cudaGetLastError();
}

// ------------------------------------------------------------------ IN
// Upper-level selection over a two-level array (R.x IN (...)): per
// level-1 entry, cnt = 1 iff x is not NULL and some element equals it.  The
// ordered compaction is finalize_kernel with agg = EXISTS.
__global__ void __launch_bounds__(C_THREADS)
in_list_kernel(long long n, const long long *__restrict__ row_ids, const long long *__restrict__ offsets,
               const long long *__restrict__ values, const void *__restrict__ x_col, int x_w,
               const uint8_t *__restrict__ x_valid, long long base, int *__restrict__ ids32,
               long long *__restrict__ cnt)
{
    for (long long i = blockIdx.x * (long long)C_THREADS + threadIdx.x; i < n; i += (long long)gridDim.x * C_THREADS) {
        const long long row = row_ids[i] - base;
        ids32[i] = (int)row;
        long long hit = 0;
        if (!x_valid || x_valid[row]) {
            const long long x = load_w(x_col, x_w, row);
            const long long e1 = offsets[i + 1];
            for (long long e = offsets[i]; e < e1; e++)
                if (__ldg(values + e) == x) { hit = 1; break; }
        }
        cnt[i] = hit;
    }
}

cudaError_t launch_in_list(long long n, const long long *row_ids, const long long *offsets, const long long *values,
                           const void *x_col, int x_w, const uint8_t *x_valid, long long base, int *ids32,
                           long long *cnt, cudaStream_t st, long long *launches)
{
    if (n <= 0) return cudaSuccess;
    in_list_kernel<<<grid_for(n, 148 * 16), C_THREADS, 0, st>>>(n, row_ids, offsets, values, x_col, x_w, x_valid,
                                                                base, ids32, cnt);
    ++*launches;
    return cudaGetLastError();
}

// ------------------------------------------------------------------ materialise
// out[i] = (T)src[i]; valid_out[i] = valid_in ? valid_in[i] : 1.  Narrowing to
// 4 bytes counts the valid values outside int32 into *bad.
template <typename T>
__global__ void __launch_bounds__(C_THREADS)
materialize_kernel(const long long *__restrict__ src, const uint8_t *__restrict__ valid_in, long long n,
                   T *__restrict__ out, uint8_t *__restrict__ valid_out, unsigned long long *__restrict__ bad)
{
    unsigned long long nb = 0;
    for (long long i = blockIdx.x * (long long)C_THREADS + threadIdx.x; i < n; i += (long long)gridDim.x * C_THREADS) {
        const long long v = src[i];
        const uint8_t ok = valid_in ? valid_in[i] : (uint8_t)1;
        if (valid_out) valid_out[i] = ok;
        if (sizeof(T) == 4 && ok && (v < INT_MIN || v > INT_MAX)) nb++;
        out[i] = ok ? (T)v : (T)0;
    }
    if (sizeof(T) == 4) {
        for (int o = 16; o > 0; o >>= 1) nb += __shfl_xor_sync(FULL, nb, o);
        if ((threadIdx.x & 31) == 0 && nb) atomicAdd(bad, nb);
    }
}

cudaError_t launch_materialize(int w, const long long *src, const uint8_t *valid_in, long long n, void *out,
                               uint8_t *valid_out, unsigned long long *bad, cudaStream_t st, long long *launches)
{
    if (n <= 0) return cudaSuccess;
    const unsigned g = grid_for(n, 148 * 16);
    if (w == 4)
        materialize_kernel<int><<<g, C_THREADS, 0, st>>>(src, valid_in, n, (int *)out, valid_out, bad);
    else
        materialize_kernel<long long><<<g, C_THREADS, 0, st>>>(src, valid_in, n, (long long *)out, valid_out, bad);
    ++*launches;
    return cudaGetLastError();
}

}  // namespace ng
