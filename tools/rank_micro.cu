// rank_micro.cu -- throughput of warp-level stable-ranking primitives on
// sm_100a (decides the radix pass's in-tile ranking).
// Each warp ranks ROWS rows of 32 digits; reported: ns per row per SM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o rank_micro tools/rank_micro.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr unsigned FULL = 0xffffffffu;

template <int RB>
__device__ __forceinline__ unsigned match_ballot(unsigned d)
{
    unsigned peers = FULL;
#pragma unroll
    for (int k = 0; k < RB; k++) {
        const bool p = (d >> k) & 1u;
        const unsigned b = __ballot_sync(FULL, p);
        peers &= p ? b : ~b;
    }
    return peers;
}

// mode 0: __match_any_sync, 1: 8 ballots, 2: 11 ballots, 3: match_any on 11-bit digits,
// 4: shared-memory counter increment per item (blocked, CUB-style), 5: empty loop
template <int MODE>
__global__ void k(unsigned *out, int rows, unsigned seed)
{
    __shared__ unsigned short cnt[16][1024];
    unsigned x = seed ^ (threadIdx.x * 0x9e3779b9u) ^ (blockIdx.x * 0x85ebca6bu);
    unsigned acc = 0;
    for (int i = threadIdx.x; i < 16 * 1024; i += blockDim.x) (&cnt[0][0])[i] = 0;
    __syncthreads();
    for (int r = 0; r < rows; r++) {
        x = x * 1664525u + 1013904223u;
        unsigned peers;
        if (MODE == 0) peers = __match_any_sync(FULL, x >> 24);
        else if (MODE == 1) peers = match_ballot<8>(x >> 24);
        else if (MODE == 2) peers = match_ballot<11>(x >> 21);
        else if (MODE == 3) peers = __match_any_sync(FULL, x >> 21);
        else if (MODE == 4) {
            const unsigned d = x >> 28;   // 4-bit digit: counter lane d/2, half d&1
            unsigned short *c = &cnt[d][threadIdx.x];
            const unsigned v = *c;
            *c = (unsigned short)(v + 1);
            peers = v;
        } else peers = x;
        const int top = 31 - __clz(peers | 1u);
        acc += top + __popc(peers & ((1u << (threadIdx.x & 31)) - 1));
    }
    if (acc == 0x12345678u) out[0] = acc;
}

template <int MODE>
float run(int blocks, int threads, int rows)
{
    unsigned *o;
    cudaMalloc(&o, 4);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    k<MODE><<<blocks, threads>>>(o, rows, 1);
    cudaEventRecord(a);
    k<MODE><<<blocks, threads>>>(o, rows, 2);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    cudaFree(o);
    return ms;
}

int main()
{
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const char *names[] = {"match_any 8-bit", "8 ballots", "11 ballots", "match_any 11-bit", "smem counter", "empty"};
    for (int occ : {4, 8}) {   // CTAs of 256 threads per SM
        const int blocks = sms * occ, threads = 256, rows = 1 << 14;
        const double wrows = (double)blocks * threads / 32 * rows;
        float t[6];
        t[0] = run<0>(blocks, threads, rows);
        t[1] = run<1>(blocks, threads, rows);
        t[2] = run<2>(blocks, threads, rows);
        t[3] = run<3>(blocks, threads, rows);
        t[4] = run<4>(blocks, threads, rows);
        t[5] = run<5>(blocks, threads, rows);
        for (int m = 0; m < 6; m++)
            printf("warps/SM %2d  %-18s %8.3f ms  %.3f SM-cycles per warp-row (at 1.965 GHz)\n", occ * 8, names[m],
                   t[m], t[m] * 1e-3 * 1.965e9 * sms / wrows);
    }
    return 0;
}
