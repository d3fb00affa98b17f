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
#ifndef NG_S_NBUF
#define NG_S_NBUF 1   // persistent pass: tile buffers per CTA (2 = next tile prefetched)
#endif
#ifndef NG_S_LATE_PREFETCH
#define NG_S_LATE_PREFETCH 0   // 1: two buffers, the next tile taken once this tile's offsets are known
#endif
#if NG_S_LATE_PREFETCH && NG_S_NBUF != 2
#error "NG_S_LATE_PREFETCH needs NG_S_NBUF 2"
#endif
#ifndef NG_S_LB_EARLY
#define NG_S_LB_EARLY 0   // look-back before ranking (1) or after (0)
#endif
#ifndef NG_S_LB_BATCH
#define NG_S_LB_BATCH 4  // look-back: predecessor tiles examined per round trip
#endif
#ifndef NG_S_PITEMS
#define NG_S_PITEMS 24   // persistent pass: items per thread for <= 8-byte (key, payload) items
#endif
#ifndef NG_S_PMINB
#define NG_S_PMINB 3  // persistent pass: CTAs per SM the register budget must allow
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
    // status words for the smallest tile any pass uses (16-byte items)
    long long tiles = (n + S_THREADS * (NG_S_PITEMS / 2) - 1) / (S_THREADS * (NG_S_PITEMS / 2));
    return (size_t)tiles * 256 * 4 + 256;
}

// K: the key type read; KO: the key type written.  KO narrower than K drops
// the (constant) high word; KO wider than K re-attaches `hi` as the high word
// -- 64-bit keys whose high 32 bits agree are sorted as 32-bit keys.
#ifdef NG_SORT_LEGACY
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
#endif  // NG_SORT_LEGACY


// ---------------------------------------------------------------------------
// Persistent onesweep pass (default).  grid = #SMs x occupancy; each CTA
// pulls tile ids from an atomic counter (so every tile's predecessors are
// held by running CTAs: the look-back cannot deadlock) and keeps TWO tiles in
// flight: while it ranks and scatters tile t out of one shared-memory buffer,
// the bulk-copy engine (cp.async.bulk, mbarrier completion) fills the other
// with its next tile.  Per tile:
//   1. each thread copies its 16 (8 for 16-byte items) warp-striped items
//      from the buffer into registers and counts their digits into its warp's
//      256 shared counters (early counts, order-free atomics);
//   2. thread d (one per digit) publishes the tile's count of digit d for the
//      decoupled look-back BEFORE ranking, scans counts over warps and digits,
//      and walks back over predecessor tiles for the global offset;
//   3. ranking: per row of 32 items, __match_any_sync groups equal digits,
//      the group's highest lane advances the warp's running counter (seeded
//      with the tile-local start of (warp, digit)), so each item gets its
//      stable tile position directly;
//   4. items are scattered into the SAME buffer (sorted by digit) and every
//      digit run is written out coalesced.
// Lanes of the warp whose 8-bit digit equals this lane's: one ballot per
// digit bit (vote + select + and), where __match_any_sync is a long-latency,
// low-throughput instruction on this part (it dominated the pass's stalls).
__device__ __forceinline__ unsigned match_digit8(unsigned d)
{
    unsigned peers;
    asm("{\n\t.reg .pred p;\n\t.reg .b32 b, m;\n\t"
        "mov.b32 %0, -1;\n\t"
#define NG_MBIT(K)                                                                                    \
        "and.b32 m, %1, " #K ";\n\t"                                                                  \
        "setp.ne.u32 p, m, 0;\n\t"                                                                    \
        "vote.sync.ballot.b32 b, p, -1;\n\t"                                                          \
        "selp.b32 m, 0, -1, p;\n\t"                                                                   \
        "xor.b32 b, b, m;\n\t"                                                                        \
        "and.b32 %0, %0, b;\n\t"
        NG_MBIT(1) NG_MBIT(2) NG_MBIT(4) NG_MBIT(8) NG_MBIT(16) NG_MBIT(32) NG_MBIT(64) NG_MBIT(128)
#undef NG_MBIT
        "}"
        : "=&r"(peers) : "r"(d));
    return peers;
}

template <typename K, int VB>
struct PassCfg {
    using V = typename std::conditional<VB == 8, long long, int>::type;
    static constexpr int ITEMS = (sizeof(K) + VB) > 8 ? NG_S_PITEMS / 2 : NG_S_PITEMS;
    static constexpr int TILE = S_THREADS * ITEMS;
    static constexpr int KBYTES = TILE * (int)sizeof(K);
    static constexpr int BUF = KBYTES + (VB ? TILE * VB : 0);
    static constexpr size_t SMEM = NG_S_NBUF * (size_t)BUF;
};

template <typename K, int VB, typename KO = K>
__global__ void __launch_bounds__(S_THREADS, NG_S_PMINB)
onesweep_p_kernel(const K *__restrict__ kin, KO *__restrict__ kout, const void *__restrict__ vin_,
                  void *__restrict__ vout_, long long n, int shift, const unsigned *__restrict__ digit_base,
                  unsigned *__restrict__ status, unsigned *__restrict__ counter, unsigned hi)
{
    using C = PassCfg<K, VB>;
    using V = typename C::V;
    constexpr int ITEMS = C::ITEMS, TILE = C::TILE;
    const V *vin = (const V *)vin_;
    V *vout = (V *)vout_;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ unsigned s_cnt[S_WARPS][256];   // early counts, then running counters
    __shared__ unsigned s_off[256];            // global destination - tile start of the digit
    __shared__ unsigned s_wsum[S_WARPS];
    __shared__ unsigned s_tile[NG_S_NBUF];
    __shared__ __align__(8) unsigned long long bar[NG_S_NBUF];

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const long long tiles = (n + TILE - 1) / TILE;

    auto issue = [&](long long t, int b) {
        const long long base = t * TILE;
        const long long rem = n - base;
        const unsigned cnt = rem < TILE ? (unsigned)rem : (unsigned)TILE;
        const unsigned kb = (cnt * (unsigned)sizeof(K) + 15u) & ~15u;
        const unsigned vb = VB ? ((cnt * (unsigned)VB + 15u) & ~15u) : 0u;
        unsigned char *buf = smem + b * C::BUF;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_expect_tx(&bar[b], kb + vb);
        bulk_g2s(buf, kin + base, kb, &bar[b]);
        if (VB) bulk_g2s(buf + C::KBYTES, vin + base, vb, &bar[b]);
    };

    for (int i = tid; i < S_WARPS * 256; i += S_THREADS) (&s_cnt[0][0])[i] = 0;
    if (tid == 0) {
        for (int b = 0; b < NG_S_NBUF; b++) mbar_init(&bar[b], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int b = 0; b < (NG_S_LATE_PREFETCH ? 1 : NG_S_NBUF); b++) {
            const unsigned t = atomicAdd(counter, 1u);
            s_tile[b] = t;
            if (t < tiles) issue(t, b);
        }
    }
    __syncthreads();
    const unsigned lt = lanemask_lt();
    const int d = tid;   // the digit this thread owns in the per-digit steps

    for (int it = 0;; it++) {
        const int b = it % NG_S_NBUF;
        const long long tile = s_tile[b];
        if (tile >= tiles) break;
        mbar_wait(&bar[b], (unsigned)(it / NG_S_NBUF) & 1u);
        K *s_k = (K *)(smem + b * C::BUF);
        V *s_v = (V *)(smem + b * C::BUF + C::KBYTES);
        const long long base = tile * TILE;
        const long long rem = n - base;
        const int tile_n = rem < TILE ? (int)rem : TILE;

        // 1. items -> registers (warp-striped: row j of warp w = 32 consecutive
        // keys), early counts.  Items past the end of the last tile rank as
        // digit 255 without being counted: they sort after every real item
        // of their warp, land at positions >= tile_n and are never written.
        K key[ITEMS];
        V val[ITEMS];
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const int p = warp * 32 * ITEMS + j * 32 + lane;
            const bool ok = p < tile_n;
            key[j] = ok ? s_k[p] : (K)0;
            if constexpr (VB > 0) val[j] = ok ? s_v[p] : (V)0;
            if (ok) atomicAdd(&s_cnt[warp][(unsigned)(key[j] >> shift) & 255u], 1u);
        }
        __syncthreads();

        // 2. per digit: counts over warps, publish the tile's count for the
        // look-back at once, tile-local scan; the first look-back loads are
        // issued here and consumed after ranking
        unsigned wex[S_WARPS];
        unsigned cnt = 0;
#pragma unroll
        for (int w = 0; w < S_WARPS; w++) {
            wex[w] = cnt;
            cnt += s_cnt[w][d];
        }
        unsigned *my_status = status + tile * 256 + d;
        st_relaxed_u32(my_status, (tile == 0 ? D_INC : D_AGG) | cnt);
        // decoupled look-back for digit d over the preceding tiles (their
        // counts were published right after their early counts)
        // first batch of predecessor statuses: loads in flight from here on
        unsigned sv[NG_S_LB_BATCH];
#pragma unroll
        for (int q = 0; q < NG_S_LB_BATCH; q++)
            sv[q] = tile - 1 - q >= 0 ? ld_relaxed_u32(status + (tile - 1 - q) * 256 + d) : D_INC;
        auto lookback = [&]() -> unsigned {
            unsigned ex = 0;
            for (long long p = tile - 1; p >= 0; p -= NG_S_LB_BATCH) {
                if (p != tile - 1) {
#pragma unroll
                    for (int q = 0; q < NG_S_LB_BATCH; q++)
                        sv[q] = p - q >= 0 ? ld_relaxed_u32(status + (p - q) * 256 + d) : D_INC;
                }
                bool done = false;
#pragma unroll
                for (int q = 0; q < NG_S_LB_BATCH; q++) {
                    if (!done) {
                        unsigned sq = sv[q];
                        while ((sq >> 30) == 0) sq = ld_relaxed_u32(status + (p - q) * 256 + d);
                        ex += sq & D_VAL;
                        done = (sq >> 30) == 2;
                    }
                }
                if (done) break;
            }
            if (tile > 0) st_relaxed_u32(my_status, D_INC | (ex + cnt));
            return ex;
        };
#if NG_S_LB_EARLY
        const unsigned excl = lookback();   // INC published before ranking: successors find it at once
#endif
        unsigned incl = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned t = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += t;
        }
        if (lane == 31) s_wsum[warp] = incl;
        __syncthreads();
        unsigned wpre = 0;
        for (int w = 0; w < warp; w++) wpre += s_wsum[w];
        const unsigned tex = wpre + incl - cnt;   // tile-local start of digit d
#pragma unroll
        for (int w = 0; w < S_WARPS; w++) s_cnt[w][d] = tex + wex[w];
        __syncthreads();

        // 3. stable ranks.  Equal digits of a row are found with 8 ballots
        // (one per digit bit: cheap ALU/vote work, where __match_any_sync is
        // a long-latency, low-throughput instruction); the group's highest
        // lane advances the (warp, digit) counter, seeded with the tile-local
        // start, so each item gets its tile position directly.
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const unsigned dj = (tile_n == TILE || warp * 32 * ITEMS + j * 32 + lane < tile_n)
                                    ? ((unsigned)(key[j] >> shift) & 255u) : 255u;
            const unsigned peers = match_digit8(dj);
            const int top = 31 - __clz(peers);
            unsigned start = 0;
            if (lane == top) {
                start = s_cnt[warp][dj];
                s_cnt[warp][dj] = start + __popc(peers);
            }
            start = __shfl_sync(FULL, start, top);
            const unsigned pos = start + __popc(peers & lt);
            // 4. reorder in place (every item of the tile is already in registers)
            s_k[pos] = key[j];
            if constexpr (VB > 0) s_v[pos] = val[j];
            __syncwarp();
        }
#if !NG_S_LB_EARLY
        const unsigned excl = lookback();
#endif
        s_off[d] = digit_base[d] + excl - tex;
        __syncthreads();
#if NG_S_LATE_PREFETCH
        // this tile's counts are published and its offsets resolved: take the
        // next tile now (its predecessors wait for it only one write-out
        // long) and let its bulk copy overlap the write-out
        if (tid == 0) {
            const unsigned t = atomicAdd(counter, 1u);
            s_tile[b ^ 1] = t;
            if (t < tiles) issue(t, b ^ 1);
        }
#endif
        for (int i = tid; i < S_WARPS * 256; i += S_THREADS) (&s_cnt[0][0])[i] = 0;
#pragma unroll 4
        for (int p = tid; p < tile_n; p += S_THREADS) {
            const K k = s_k[p];
            const long long dst = (long long)s_off[(unsigned)(k >> shift) & 255u] + p;
            if constexpr (sizeof(KO) > sizeof(K)) kout[dst] = ((KO)hi << 32) | (KO)k;
            else kout[dst] = (KO)k;
            if constexpr (VB > 0) vout[dst] = s_v[p];
        }
        __syncthreads();
#if !NG_S_LATE_PREFETCH
        if (tid == 0) {
            const unsigned t = atomicAdd(counter, 1u);
            s_tile[b] = t;
            if (t < tiles) issue(t, b);
        }
        __syncthreads();
#endif
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
#ifdef NG_SORT_LEGACY
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
#else
    using Cfg = PassCfg<K, VB>;
    const long long tiles = (n + Cfg::TILE - 1) / Cfg::TILE;
    static int grid_max = 0;   // resident CTAs (persistent grid), per instantiation
    if (!grid_max) {
        cudaError_t e = cudaFuncSetAttribute(onesweep_p_kernel<K, VB, KO>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Cfg::SMEM);
        if (e != cudaSuccess) return e;
        int dev = 0, sms = 0, occ = 0;
        if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
        if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
        if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, onesweep_p_kernel<K, VB, KO>, S_THREADS,
                                                               Cfg::SMEM)) != cudaSuccess)
            return e;
        if (occ < 1) return cudaErrorInvalidConfiguration;
        grid_max = sms * occ;
    }
    cudaError_t e = cudaMemsetAsync(scratch, 0, (size_t)tiles * 256 * 4 + 256, st);
    if (e != cudaSuccess) return e;
    const unsigned grid = (unsigned)(tiles < grid_max ? tiles : grid_max);
    onesweep_p_kernel<K, VB, KO><<<grid, S_THREADS, Cfg::SMEM, st>>>(
        (const K *)kin, (KO *)kout, vin, vout, n, shift, digit_base, (unsigned *)((char *)scratch + 256),
        (unsigned *)scratch, hi);
    return cudaGetLastError();
#endif
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
