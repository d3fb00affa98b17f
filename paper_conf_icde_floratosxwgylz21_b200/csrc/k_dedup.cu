// k_dedup.cu -- caching of subquery results per distinct correlated value.
//
// PAPER.md P:331 (§III-D "Caching"): "If the passed-in parameter is not a
// primary key, subqueries would be re-evaluated with duplicate values. Thus,
// we build a cache for the results evaluated from the subquery, whose key is
// the combination of the passed-in parameters."  The cost model's (S - Ch)
// factor (Eq. 6) counts the evaluations it saves.
//
// B200 form: the R' keys are radix-sorted (k_sort.cu) together with their R'
// positions; this file turns the sorted run into the distinct-key list U (the
// subquery kernels evaluate U instead of R') and the map R' position ->
// distinct id that the finalize kernel gathers through.
#include "internal.h"
#include "scan.cuh"

namespace ng {

constexpr int G_THREADS = 256;
constexpr int G_ITEMS = 16;
constexpr int G_TILE = G_THREADS * G_ITEMS;

size_t group_scratch_bytes(long long n) { return (size_t)((n + G_TILE - 1) / G_TILE + 1) * 8 + 256; }

__global__ void iota_kernel(int *__restrict__ out, long long n)
{
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        out[i] = (int)i;
}

// sorted keys sk[0..n), their R' positions pos[0..n) ->
//   uk[u]        distinct keys in ascending order, *d_u = their number
//   map[pos[p]]  = id of sk[p]'s distinct key
template <typename K>
__global__ void __launch_bounds__(G_THREADS)
group_kernel(const K *__restrict__ sk, const int *__restrict__ pos, long long n, K *__restrict__ uk,
             int *__restrict__ map, long long *__restrict__ d_u, unsigned long long *__restrict__ status,
             unsigned *__restrict__ counter)
{
    __shared__ unsigned s_tile;
    __shared__ unsigned s_cnt[G_ITEMS][G_THREADS / 32];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    if (tid == 0) s_tile = atomicAdd(counter, 1u);
    __syncthreads();
    const long long tile = s_tile;
    const long long num_tiles = (n + G_TILE - 1) / G_TILE;
    const long long base = tile * G_TILE;
    unsigned first = 0;  // bit j: row j starts a new distinct key
    unsigned rank[G_ITEMS];
#pragma unroll
    for (int j = 0; j < G_ITEMS; j++) {
        const long long p = base + (long long)j * G_THREADS + tid;
        const bool f = p < n && (p == 0 || sk[p] != sk[p - 1]);
        if (f) first |= 1u << j;
        const unsigned m = __ballot_sync(FULL, f);
        if (lane == 0) s_cnt[j][warp] = __popc(m);
        rank[j] = __popc(m & lanemask_lt());
    }
    const unsigned long long tb = tile_offsets<G_ITEMS, G_THREADS>(s_cnt, status, tile, num_tiles, d_u);
#pragma unroll
    for (int j = 0; j < G_ITEMS; j++) {
        const long long p = base + (long long)j * G_THREADS + tid;
        if (p >= n) continue;
        const bool f = first >> j & 1u;
        const long long excl = (long long)tb + s_cnt[j][warp] + rank[j];  // distinct keys before row p
        const long long u = excl + (f ? 0 : -1);
        if (f) uk[excl] = sk[p];
        map[pos[p]] = (int)u;
    }
}

cudaError_t launch_iota(int *out, long long n, cudaStream_t st, long long *launches)
{
    if (n <= 0) return cudaSuccess;
    long long blocks = (n + 255) / 256;
    if (blocks > 148 * 8) blocks = 148 * 8;
    iota_kernel<<<(unsigned)blocks, 256, 0, st>>>(out, n);
    ++*launches;
    return cudaGetLastError();
}

cudaError_t launch_group(int kb, const void *sk, const int *pos, long long n, void *uk, int *map, long long *d_u,
                         void *scratch, cudaStream_t st, long long *launches)
{
    cudaError_t e = cudaMemsetAsync(d_u, 0, 8, st);
    if (e != cudaSuccess || n <= 0) return e;
    e = cudaMemsetAsync(scratch, 0, group_scratch_bytes(n), st);
    if (e != cudaSuccess) return e;
    const unsigned tiles = (unsigned)((n + G_TILE - 1) / G_TILE);
    unsigned *counter = (unsigned *)scratch;
    unsigned long long *status = (unsigned long long *)((char *)scratch + 256);
    if (kb == 4)
        group_kernel<uint32_t><<<tiles, G_THREADS, 0, st>>>((const uint32_t *)sk, pos, n, (uint32_t *)uk, map, d_u,
                                                           status, counter);
    else
        group_kernel<uint64_t><<<tiles, G_THREADS, 0, st>>>((const uint64_t *)sk, pos, n, (uint64_t *)uk, map, d_u,
                                                           status, counter);
    ++*launches;
    return cudaGetLastError();
}

}  // namespace ng
