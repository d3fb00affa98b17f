// k_sort.cu -- a4: index build = stable LSD radix sort of S' by the encoded
// correlated key, carrying the aggregate payload.
//
// PAPER.md P:315 (§III-D "Indexing"): sort the correlated column
// (O(N log N)) and keep "the sorted values and their original positions"
// (O(2N)), then binary-search a valid range per passed-in value.  Here the
// payload itself is carried through the sort instead of the positions, so the
// per-tuple range scan of a6 reads contiguous memory.
//
// One kernel per 8-bit digit ("onesweep"): each 4096-key tile ranks its keys
// with warp __match_any_sync (stable: warp-striped items, ranks in input
// order), publishes per-digit tile counts, resolves its global per-digit
// offset by decoupled look-back over preceding tiles (dynamic tile ids for
// forward progress), reorders the tile in shared memory and writes each
// digit run out coalesced, so a pass is one read and one write of (key,
// payload).  The S' filter kernel also reduces AND / OR over the keys: digits
// on which all keys agree are skipped; one histogram kernel covers the rest.
#include <type_traits>

#include "internal.h"

namespace ng {

#ifndef NG_S_ITEMS
#define NG_S_ITEMS 16
#endif
#ifndef NG_S_MINB
#define NG_S_MINB 4   // __launch_bounds__ min blocks per SM (register cap; 1 lets ptxas take 160+)
#endif
#ifndef NG_S_CARVEOUT
#define NG_S_CARVEOUT -1   // preferred shared-memory carveout (%); -1 = driver default
#endif
constexpr int S_THREADS = 256;
constexpr int S_WARPS = S_THREADS / 32;
constexpr int S_ITEMS = NG_S_ITEMS;
constexpr int S_TILE = S_THREADS * S_ITEMS;
constexpr unsigned D_AGG = 1u << 30, D_INC = 2u << 30, D_VAL = (1u << 30) - 1;

size_t sort_scratch_bytes(long long n)
{
    long long tiles = (n + S_TILE - 1) / S_TILE;
    return (size_t)tiles * 256 * 4 + 256;
}

// K: the key type read; KO: the key type written.  KO narrower than K drops
// the (constant) high word; KO wider than K re-attaches `hi` as the high word
// -- 64-bit keys whose high 32 bits agree are sorted as 32-bit keys.
template <typename K, int VB, typename KO = K>
__global__ void __launch_bounds__(S_THREADS, NG_S_MINB)
onesweep_kernel(const K *__restrict__ kin, KO *__restrict__ kout, const void *__restrict__ vin_,
                void *__restrict__ vout_, long long n, int shift, const unsigned *__restrict__ digit_base,
                unsigned *__restrict__ status, unsigned *__restrict__ counter, unsigned hi)
{
    using V = typename std::conditional<VB == 8, long long, int>::type;
    const V *vin = (const V *)vin_;
    V *vout = (V *)vout_;
    extern __shared__ __align__(16) unsigned char smem[];
    K *s_keys = (K *)smem;
    V *s_vals = (V *)(smem + S_TILE * sizeof(K));
    __shared__ unsigned s_whist[S_WARPS][256];
    __shared__ unsigned s_tdig[256];
    __shared__ unsigned s_gdig[256];
    __shared__ unsigned s_wsum[S_WARPS];
    __shared__ unsigned s_tile;

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    if (tid == 0) s_tile = atomicAdd(counter, 1u);
    for (int i = tid; i < S_WARPS * 256; i += S_THREADS) (&s_whist[0][0])[i] = 0;
    __syncthreads();
    const long long tile = s_tile;
    const long long base = tile * S_TILE;
    const long long wbase = base + (long long)warp * 32 * S_ITEMS;

    K key[S_ITEMS];
    V val[S_ITEMS];
    int dig[S_ITEMS];
    unsigned rank[S_ITEMS];
#pragma unroll
    for (int j = 0; j < S_ITEMS; j++) {
        const long long idx = wbase + j * 32 + lane;
        const bool ok = idx < n;
        key[j] = ok ? kin[idx] : (K)0;
        if constexpr (VB > 0) val[j] = ok ? vin[idx] : (V)0;
        dig[j] = ok ? (int)((key[j] >> shift) & 255) : 256;
    }
    const unsigned lt = lanemask_lt();
#pragma unroll
    for (int j = 0; j < S_ITEMS; j++) {
        const unsigned peers = __match_any_sync(FULL, dig[j]);
        const int leader = __ffs(peers) - 1;
        unsigned b = 0;
        if (lane == leader && dig[j] < 256) {
            b = s_whist[warp][dig[j]];
            s_whist[warp][dig[j]] = b + __popc(peers);
        }
        b = __shfl_sync(FULL, b, leader);
        rank[j] = b + __popc(peers & lt);
        __syncwarp();
    }
    __syncthreads();
    // per digit (thread == digit): exclusive offsets across warps, tile count
    const int d = tid;
    unsigned cnt = 0;
#pragma unroll
    for (int w = 0; w < S_WARPS; w++) {
        unsigned t = s_whist[w][d];
        s_whist[w][d] = cnt;
        cnt += t;
    }
    unsigned *my_status = status + tile * 256 + d;
    if (tile == 0) st_relaxed_u32(my_status, D_INC | cnt);
    else st_relaxed_u32(my_status, D_AGG | cnt);
    // tile-local exclusive scan over digits
    unsigned incl = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        unsigned t = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += t;
    }
    if (lane == 31) s_wsum[warp] = incl;
    // decoupled look-back for digit d
    unsigned excl = 0;
    if (tile > 0) {
        // walk back 4 predecessors per round trip (loads issued together)
        long long p = tile - 1;
        bool done = false;
        while (!done) {
            unsigned sv[4];
#pragma unroll
            for (int q = 0; q < 4; q++) sv[q] = p - q >= 0 ? ld_relaxed_u32(status + (p - q) * 256 + d) : D_INC;
#pragma unroll
            for (int q = 0; q < 4; q++) {
                if (done) break;
                unsigned s = sv[q];
                while ((s >> 30) == 0) s = ld_relaxed_u32(status + (p - q) * 256 + d);
                excl += s & D_VAL;
                done = (s >> 30) == 2;
            }
            p -= 4;
        }
        st_relaxed_u32(my_status, D_INC | (excl + cnt));
    }
    __syncthreads();
    unsigned wpre = 0;
    for (int w = 0; w < warp; w++) wpre += s_wsum[w];
    s_tdig[d] = wpre + incl - cnt;
    s_gdig[d] = digit_base[d] + excl;
    __syncthreads();
#pragma unroll
    for (int j = 0; j < S_ITEMS; j++) {
        if (dig[j] < 256) {
            const unsigned pos = s_tdig[dig[j]] + s_whist[warp][dig[j]] + rank[j];
            s_keys[pos] = key[j];
            if constexpr (VB > 0) s_vals[pos] = val[j];
        }
    }
    __syncthreads();
    const long long rem = n - base;
    const int tile_n = rem < S_TILE ? (int)rem : S_TILE;
    for (int p = tid; p < tile_n; p += S_THREADS) {
        const K k = s_keys[p];
        const int dd = (int)((k >> shift) & 255);
        const long long dst = (long long)s_gdig[dd] + (p - (int)s_tdig[dd]);
        if constexpr (sizeof(KO) > sizeof(K)) kout[dst] = ((KO)hi << 32) | (KO)k;
        else kout[dst] = (KO)k;
        if constexpr (VB > 0) vout[dst] = s_vals[p];
    }
}

// Histograms of the 8-bit digits that vary (the others were dropped using
// the AND / OR masks the S' filter computed): one pass over the keys, per-CTA
// shared-memory bins, one global atomic per bin per CTA.
struct DigitList {
    int n;
    int shift[8];
};

template <typename K>
__global__ void __launch_bounds__(256) digit_hist_kernel(const K *__restrict__ keys, long long n, DigitList dl,
                                                         unsigned *__restrict__ hist)
{
    __shared__ unsigned s_hist[8 * 256];
    for (int i = threadIdx.x; i < dl.n * 256; i += 256) s_hist[i] = 0;
    __syncthreads();
    const long long stride = (long long)gridDim.x * 256;
    for (long long i = blockIdx.x * 256LL + threadIdx.x; i < n; i += stride) {
        const K k = keys[i];
#pragma unroll
        for (int p = 0; p < 8; p++)
            if (p < dl.n) atomicAdd(&s_hist[p * 256 + (unsigned)((k >> dl.shift[p]) & 255)], 1u);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < dl.n * 256; i += 256)
        if (s_hist[i]) atomicAdd(&hist[i], s_hist[i]);
}

// Exclusive scan of each pass's 256 bins -> global digit base offsets.
__global__ void __launch_bounds__(256) digit_scan_kernel(const unsigned *__restrict__ hist, unsigned *__restrict__ base)
{
    __shared__ unsigned s_w[8];
    const unsigned *h = hist + blockIdx.x * 256;
    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
    const unsigned c = h[t];
    unsigned incl = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        unsigned v = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += v;
    }
    if (lane == 31) s_w[warp] = incl;
    __syncthreads();
    unsigned pre = 0;
    for (int w = 0; w < warp; w++) pre += s_w[w];
    base[blockIdx.x * 256 + t] = pre + incl - c;
}

cudaError_t launch_digit_hist(int kb, const void *keys, long long n, const int *shifts, int np, unsigned *hist,
                              unsigned *digit_base, int num_sms, cudaStream_t st, long long *launches)
{
    if (np <= 0) return cudaSuccess;
    cudaError_t e = cudaMemsetAsync(hist, 0, (size_t)np * 256 * 4, st);
    if (e != cudaSuccess) return e;
    DigitList dl{};
    dl.n = np;
    for (int p = 0; p < np; p++) dl.shift[p] = shifts[p];
    long long blocks = (n + 255) / 256;
    if (blocks > (long long)num_sms * 8) blocks = (long long)num_sms * 8;
    if (blocks < 1) blocks = 1;
    if (kb == 4) digit_hist_kernel<uint32_t><<<(unsigned)blocks, 256, 0, st>>>((const uint32_t *)keys, n, dl, hist);
    else digit_hist_kernel<uint64_t><<<(unsigned)blocks, 256, 0, st>>>((const uint64_t *)keys, n, dl, hist);
    digit_scan_kernel<<<np, 256, 0, st>>>(hist, digit_base);
    *launches += 2;
    return cudaGetLastError();
}

template <typename K, int VB, typename KO>
static cudaError_t run_pass(const void *kin, void *kout, const void *vin, void *vout, long long n, int shift,
                            const unsigned *digit_base, void *scratch, unsigned hi, cudaStream_t st)
{
    using V = typename std::conditional<VB == 8, long long, int>::type;
    const long long tiles = (n + S_TILE - 1) / S_TILE;
    const size_t smem = S_TILE * (sizeof(K) + (VB > 0 ? sizeof(V) : 0));
    static bool attr_set = false;
    if (!attr_set) {
        cudaError_t e = cudaFuncSetAttribute(onesweep_kernel<K, VB, KO>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)smem);
        if (e != cudaSuccess) return e;
        if (NG_S_CARVEOUT >= 0) {
            e = cudaFuncSetAttribute(onesweep_kernel<K, VB, KO>, cudaFuncAttributePreferredSharedMemoryCarveout,
                                     NG_S_CARVEOUT);
            if (e != cudaSuccess) return e;
        }
        attr_set = true;
    }
    cudaError_t e = cudaMemsetAsync(scratch, 0, sort_scratch_bytes(n), st);
    if (e != cudaSuccess) return e;
    onesweep_kernel<K, VB, KO><<<(unsigned)tiles, S_THREADS, smem, st>>>(
        (const K *)kin, (KO *)kout, vin, vout, n, shift, digit_base, (unsigned *)((char *)scratch + 256),
        (unsigned *)scratch, hi);
    return cudaGetLastError();
}

template <typename K, typename KO>
static cudaError_t run_pass_v(int vb, const void *kin, void *kout, const void *vin, void *vout, long long n, int shift,
                              const unsigned *digit_base, void *scratch, unsigned hi, cudaStream_t st)
{
    if (vb == 0) return run_pass<K, 0, KO>(kin, kout, vin, vout, n, shift, digit_base, scratch, hi, st);
    if (vb == 4) return run_pass<K, 4, KO>(kin, kout, vin, vout, n, shift, digit_base, scratch, hi, st);
    return run_pass<K, 8, KO>(kin, kout, vin, vout, n, shift, digit_base, scratch, hi, st);
}

cudaError_t launch_radix_pass_x(int kb_in, int kb_out, int vb, const void *kin, void *kout, const void *vin,
                                void *vout, long long n, int shift, const unsigned *digit_base, void *scratch,
                                unsigned hi, cudaStream_t st, long long *launches)
{
    if (n <= 0) return cudaSuccess;
    if (n >= (1ll << 30)) return cudaErrorInvalidValue;
    cudaError_t e;
    if (kb_in == 4 && kb_out == 4)
        e = run_pass_v<uint32_t, uint32_t>(vb, kin, kout, vin, vout, n, shift, digit_base, scratch, hi, st);
    else if (kb_in == 8 && kb_out == 8)
        e = run_pass_v<uint64_t, uint64_t>(vb, kin, kout, vin, vout, n, shift, digit_base, scratch, hi, st);
    else if (kb_in == 8)
        e = run_pass_v<uint64_t, uint32_t>(vb, kin, kout, vin, vout, n, shift, digit_base, scratch, hi, st);
    else
        e = run_pass_v<uint32_t, uint64_t>(vb, kin, kout, vin, vout, n, shift, digit_base, scratch, hi, st);
    ++*launches;
    return e;
}

cudaError_t launch_radix_pass(int kb, int vb, const void *kin, void *kout, const void *vin, void *vout,
                              long long n, int shift, const unsigned *digit_base, void *scratch, cudaStream_t st,
                              long long *launches)
{
    return launch_radix_pass_x(kb, kb, vb, kin, kout, vin, vout, n, shift, digit_base, scratch, 0u, st, launches);
}

}  // namespace ng
