// scan.cuh -- ordered tile compaction offsets with a CTA-wide decoupled
// look-back (the paper's "0-1 vector -> prefix-sum -> materialize", P:235,
// fused into one pass over the data).
#pragma once
#include "common.cuh"

namespace ng {

// s_cnt[ITEMS][WARPS] holds the survivor count of (item j, warp w) on entry --
// row order is item-major then warp (row = base + j*THREADS + tid) -- and the
// exclusive offset within the tile on exit.  Returns the tile's global offset.
// The look-back is done by the whole CTA (the other warps would only wait at
// the barrier): thread t inspects predecessor tile-1-t, so one L2 round trip
// covers THREADS predecessors; the nearest inclusive prefix ends the walk.
// `status` (one u64 per tile) must be zero before the launch; the last tile
// writes the grand total to *out_count.
template <int ITEMS, int THREADS>
__device__ __forceinline__ unsigned long long tile_offsets(unsigned (*s_cnt)[THREADS / 32],
                                                           unsigned long long *status, long long tile,
                                                           long long num_tiles, long long *out_count)
{
    constexpr int WARPS = THREADS / 32;
    constexpr int E = ITEMS * WARPS;            // entries to scan
    constexpr int PER = (E + 31) / 32;          // entries per lane of warp 0
    __shared__ unsigned s_total;
    __shared__ int s_stop;
    __shared__ unsigned long long s_wsum[WARPS];
    __syncthreads();
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid < 32) {
        unsigned *flat = &s_cnt[0][0];
        unsigned c[PER], s = 0;
#pragma unroll
        for (int q = 0; q < PER; q++) {
            const int e = PER * lane + q;
            c[q] = e < E ? flat[e] : 0u;
            s += c[q];
        }
        unsigned incl = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            unsigned t = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += t;
        }
        unsigned run = incl - s;
        const unsigned total = __shfl_sync(FULL, incl, 31);
#pragma unroll
        for (int q = 0; q < PER; q++) {
            const int e = PER * lane + q;
            if (e < E) flat[e] = run;
            run += c[q];
        }
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
        for (long long round = 0;; round += THREADS) {
            const long long pred = tile - 1 - round - tid;
            unsigned long long sv = pred >= 0 ? ld_relaxed_u64(status + pred) : ST_INC;
            while ((sv >> 62) == 0) sv = ld_relaxed_u64(status + pred);
            if ((sv >> 62) == 2) atomicMin(&s_stop, tid);
            __syncthreads();
            const int stop = s_stop;  // nearest inclusive predecessor
            unsigned long long v = tid <= stop ? (sv & ST_VAL) : 0;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
            if (lane == 0) s_wsum[warp] = v;
            __syncthreads();
#pragma unroll
            for (int w = 0; w < WARPS; w++) excl += s_wsum[w];
            if (stop != 0x7fffffff) break;
            __syncthreads();  // s_wsum reuse
        }
        if (tid == 0) st_relaxed_u64(status + tile, ST_INC | (excl + total));
    }
    if (tid == 0 && tile == num_tiles - 1) *out_count = (long long)(excl + total);
    __syncthreads();
    return excl;
}

// The same in two halves, so a kernel can publish its tile's aggregate as
// soon as the counts exist and do other work (e.g. issue loads) before it
// waits on its predecessors.  tile_publish: s_cnt counts -> exclusive
// in-tile offsets, publishes the tile's AGG status, returns the tile total
// (in *s_total too).  tile_lookback: the global offset (walks back to the
// nearest inclusive predecessor), publishes INC.  Both are CTA-wide.
template <int ITEMS, int THREADS>
__device__ __forceinline__ unsigned tile_publish(unsigned (*s_cnt)[THREADS / 32], unsigned long long *status,
                                                 long long tile, unsigned *s_total)
{
    constexpr int WARPS = THREADS / 32;
    constexpr int E = ITEMS * WARPS;
    constexpr int PER = (E + 31) / 32;
    __syncthreads();
    const int tid = threadIdx.x, lane = tid & 31;
    if (tid < 32) {
        unsigned *flat = &s_cnt[0][0];
        unsigned c[PER], s = 0;
#pragma unroll
        for (int q = 0; q < PER; q++) {
            const int e = PER * lane + q;
            c[q] = e < E ? flat[e] : 0u;
            s += c[q];
        }
        unsigned incl = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            unsigned t = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += t;
        }
        unsigned run = incl - s;
        const unsigned total = __shfl_sync(FULL, incl, 31);
#pragma unroll
        for (int q = 0; q < PER; q++) {
            const int e = PER * lane + q;
            if (e < E) flat[e] = run;
            run += c[q];
        }
        if (lane == 0) {
            *s_total = total;
            st_relaxed_u64(status + tile, (tile == 0 ? ST_INC : ST_AGG) | total);
        }
    }
    __syncthreads();
    return *s_total;
}

template <int THREADS>
__device__ __forceinline__ unsigned long long tile_lookback(unsigned long long *status, long long tile,
                                                            long long num_tiles, unsigned long long total,
                                                            long long *out_count)
{
    constexpr int WARPS = THREADS / 32;
    __shared__ int s_stop;
    __shared__ unsigned long long s_wsum[WARPS];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) s_stop = 0x7fffffff;
    __syncthreads();
    unsigned long long excl = 0;
    if (tile > 0) {
        for (long long round = 0;; round += THREADS) {
            const long long pred = tile - 1 - round - tid;
            unsigned long long sv = pred >= 0 ? ld_relaxed_u64(status + pred) : ST_INC;
            while ((sv >> 62) == 0) sv = ld_relaxed_u64(status + pred);
            if ((sv >> 62) == 2) atomicMin(&s_stop, tid);
            __syncthreads();
            const int stop = s_stop;
            unsigned long long v = tid <= stop ? (sv & ST_VAL) : 0;
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
            if (lane == 0) s_wsum[warp] = v;
            __syncthreads();
#pragma unroll
            for (int w = 0; w < WARPS; w++) excl += s_wsum[w];
            if (stop != 0x7fffffff) break;
            __syncthreads();
        }
        if (tid == 0) st_relaxed_u64(status + tile, ST_INC | (excl + total));
    }
    if (tid == 0 && tile == num_tiles - 1) *out_count = (long long)(excl + total);
    __syncthreads();
    return excl;
}

}  // namespace ng
