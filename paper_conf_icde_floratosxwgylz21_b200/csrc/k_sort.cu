// k_sort.cu -- a4: index build = stable LSD radix sort of S' by the encoded
// correlated key, carrying the aggregate payload.
//
// PAPER.md P:315 (§III-D "Indexing"): sort the correlated column
// (O(N log N)) and keep "the sorted values and their original positions"
// (O(2N)), then binary-search a valid range per passed-in value.  Here the
// payload itself is carried through the sort instead of the positions, so the
// per-tuple range scan of a6 reads contiguous memory.
//
// One persistent kernel per 8- or 9-bit digit ("onesweep"): each tile of
// 3-12k items is staged in shared memory by a bulk copy, counted per warp,
// its per-digit counts published for a decoupled look-back over preceding
// tiles (dynamic tile ids for forward progress), ranked stably with warp
// ballots, reordered in place and written out one coalesced digit run per
// digit, so a pass is one read and one write of (key, payload).  The S'
// filter kernel also reduces AND / OR over the keys: only the bits that vary
// are sorted (api.cpp plans the digit windows; 9-bit digits when they save a
// pass); one histogram kernel covers every pass.
#include <type_traits>

#include "internal.h"

namespace ng {

#ifndef NG_S_NBUF
#define NG_S_NBUF 1   // persistent pass: tile buffers per CTA (2 = next tile prefetched)
#endif
#ifndef NG_S_LATE_PREFETCH
#define NG_S_LATE_PREFETCH 0   // 1: two buffers, the next tile taken once this tile's offsets are known
#endif
#if NG_S_LATE_PREFETCH && NG_S_NBUF != 2
#error "NG_S_LATE_PREFETCH needs NG_S_NBUF 2"
#endif
#ifndef NG_S_LB_BATCH
#define NG_S_LB_BATCH 4  // look-back: predecessor tiles examined per round trip
#endif
#ifndef NG_S_PITEMS
#define NG_S_PITEMS 24   // persistent pass: items per thread for <= 8-byte (key, payload) items
#endif
#ifndef NG_S_PITEMS4
#define NG_S_PITEMS4 48   // ... for 4-byte items (32-bit keys, no payload)
#endif
#ifndef NG_S_PREAGG
#define NG_S_PREAGG 0   // 1: a tile-histogram kernel publishes every tile's digit counts before the pass
#endif
#ifndef NG_H_KEYS
#define NG_H_KEYS 4096   // digit histogram: keys per CTA (fewer CTAs = fewer same-bin global atomics)
#endif
#ifndef NG_S_PMINB
#define NG_S_PMINB 3  // persistent pass: CTAs per SM the register budget must allow
#endif
constexpr int S_THREADS = 256;
constexpr int S_WARPS = S_THREADS / 32;
constexpr unsigned D_AGG = 1u << 30, D_INC = 2u << 30, D_VAL = (1u << 30) - 1;

size_t sort_scratch_bytes(long long n)
{
    // status words for the smallest tile any pass uses (16-byte items)
    long long tiles = (n + S_THREADS * (NG_S_PITEMS / 2) - 1) / (S_THREADS * (NG_S_PITEMS / 2));
    return (size_t)tiles * 512 * 4 + 256;   // 9-bit digits: 512 status words per tile
}

// K: the key type read; KO: the key type written.  KO narrower than K drops
// the (constant) high word; KO wider than K re-attaches `hi` as the high word
// -- 64-bit keys whose high 32 bits agree are sorted as 32-bit keys.


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
template <int RB>
__device__ __forceinline__ unsigned match_digit(unsigned d)
{
    unsigned peers;
#define NG_MBIT(K)                                                                                    \
        "and.b32 m, %1, " #K ";\n\t"                                                                  \
        "setp.ne.u32 p, m, 0;\n\t"                                                                    \
        "vote.sync.ballot.b32 b, p, -1;\n\t"                                                          \
        "selp.b32 m, 0, -1, p;\n\t"                                                                   \
        "xor.b32 b, b, m;\n\t"                                                                        \
        "and.b32 %0, %0, b;\n\t"
    if constexpr (RB == 8)
        asm("{\n\t.reg .pred p;\n\t.reg .b32 b, m;\n\t"
            "mov.b32 %0, -1;\n\t"
            NG_MBIT(1) NG_MBIT(2) NG_MBIT(4) NG_MBIT(8) NG_MBIT(16) NG_MBIT(32) NG_MBIT(64) NG_MBIT(128)
            "}"
            : "=&r"(peers) : "r"(d));
    else
        asm("{\n\t.reg .pred p;\n\t.reg .b32 b, m;\n\t"
            "mov.b32 %0, -1;\n\t"
            NG_MBIT(1) NG_MBIT(2) NG_MBIT(4) NG_MBIT(8) NG_MBIT(16) NG_MBIT(32) NG_MBIT(64) NG_MBIT(128)
            NG_MBIT(256)
            "}"
            : "=&r"(peers) : "r"(d));
#undef NG_MBIT
    return peers;
}

template <typename K, int VB, int RB = 8>
struct PassCfg {
    using V = typename std::conditional<VB == 8, long long, int>::type;
    // items per thread by item size; fewer with 9-bit digits (2 digits per
    // thread in the per-digit steps) so everything stays in 80 registers
    static constexpr int ITEMS = (sizeof(K) + VB) > 8 ? NG_S_PITEMS / 2
                                 : ((sizeof(K) + VB) == 4 ? (RB == 8 ? NG_S_PITEMS4 : 32)
                                                          : (RB == 8 ? NG_S_PITEMS : 20));
    static constexpr int TILE = S_THREADS * ITEMS;
    static constexpr int KBYTES = TILE * (int)sizeof(K);
    static constexpr int BUF = KBYTES + (VB ? TILE * VB : 0);
    static constexpr size_t SMEM = NG_S_NBUF * (size_t)BUF;
};

template <typename K, int VB, int RB>
static size_t pass_zero_t(long long n)
{
    using Cfg = PassCfg<K, VB, RB>;
    const long long tiles = (n + Cfg::TILE - 1) / Cfg::TILE;
    return (size_t)tiles * (1 << RB) * 4 + 256;
}

// kb: the key width the pass READS (the tile size follows the items read)
size_t sort_pass_zero_bytes(long long n, int kb, int vb, int rb)
{
#define NG_PZ(K_, RB_) (vb == 0 ? pass_zero_t<K_, 0, RB_>(n) : (vb == 4 ? pass_zero_t<K_, 4, RB_>(n) : pass_zero_t<K_, 8, RB_>(n)))
    if (kb == 4) return rb == 8 ? NG_PZ(uint32_t, 8) : NG_PZ(uint32_t, 9);
    return rb == 8 ? NG_PZ(uint64_t, 8) : NG_PZ(uint64_t, 9);
#undef NG_PZ
}

template <typename K, int VB, typename KO, int RB>
__global__ void __launch_bounds__(S_THREADS, NG_S_PMINB)
onesweep_p_kernel(const K *__restrict__ kin, KO *__restrict__ kout, const void *__restrict__ vin_,
                  void *__restrict__ vout_, long long n, int shift, const unsigned *__restrict__ digit_base,
                  unsigned *__restrict__ status, unsigned *__restrict__ counter, unsigned hi, K encx)
{
    // encx: XOR applied to every key read (the sign-bit flip that encodes a
    // raw signed key column; 0 when the input is already encoded)
    using C = PassCfg<K, VB, RB>;
    using V = typename C::V;
    constexpr int ITEMS = C::ITEMS, TILE = C::TILE;
    constexpr int NB = 1 << RB;            // digit values (256 or 512)
    constexpr unsigned DM = NB - 1;
    constexpr int DPT = NB / S_THREADS;    // digits per thread in the per-digit steps
    const V *vin = (const V *)vin_;
    V *vout = (V *)vout_;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ unsigned s_cnt[S_WARPS][NB];    // early counts, then running counters
    __shared__ unsigned s_off[NB];             // global destination - tile start of the digit
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

    for (int i = tid; i < S_WARPS * NB; i += S_THREADS) (&s_cnt[0][0])[i] = 0;
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
            key[j] = ok ? (K)(s_k[p] ^ encx) : (K)0;
            if constexpr (VB > 0) val[j] = ok ? s_v[p] : (V)0;
            if (ok) atomicAdd(&s_cnt[warp][(unsigned)(key[j] >> shift) & DM], 1u);
        }
        __syncthreads();

        // 2. per digit (thread t owns digits t*DPT .. t*DPT+DPT-1): counts
        // over warps, publish the tile's counts for the look-back at once,
        // tile-local scan; the first look-back loads are issued here and
        // consumed after ranking
        // (9-bit digits, two per thread: the per-warp prefixes are re-read
        // from shared memory instead of held in registers, and the first
        // look-back batch is half as deep -- the register budget is 80)
        constexpr int LBB = DPT == 1 ? NG_S_LB_BATCH : (NG_S_LB_BATCH + 1) / 2;
        unsigned wex[DPT == 1 ? S_WARPS : 1], cnt[DPT], loc = 0;
#pragma unroll
        for (int q = 0; q < DPT; q++) {
            const int d = tid * DPT + q;
            unsigned c = 0;
#pragma unroll
            for (int w = 0; w < S_WARPS; w++) {
                if constexpr (DPT == 1) wex[w] = c;
                c += s_cnt[w][d];
            }
            cnt[q] = c;
            loc += c;
            if (!NG_S_PREAGG) st_relaxed_u32(status + tile * NB + d, (tile == 0 ? D_INC : D_AGG) | c);
        }
        unsigned sv[DPT][LBB];
#pragma unroll
        for (int q = 0; q < DPT; q++)
#pragma unroll
            for (int b2 = 0; b2 < LBB; b2++)
                sv[q][b2] = tile - 1 - b2 >= 0 ? ld_relaxed_u32(status + (tile - 1 - b2) * NB + tid * DPT + q) : D_INC;
        // decoupled look-back for digit tid*DPT+q over the preceding tiles
        auto lookback = [&](int q) -> unsigned {
            const int d = tid * DPT + q;
            unsigned ex = 0;
            for (long long p = tile - 1; p >= 0; p -= LBB) {
                if (p != tile - 1) {
#pragma unroll
                    for (int b2 = 0; b2 < LBB; b2++)
                        sv[q][b2] = p - b2 >= 0 ? ld_relaxed_u32(status + (p - b2) * NB + d) : D_INC;
                }
                bool done = false;
#pragma unroll
                for (int b2 = 0; b2 < LBB; b2++) {
                    if (!done) {
                        unsigned sq = sv[q][b2];
                        while ((sq >> 30) == 0) sq = ld_relaxed_u32(status + (p - b2) * NB + d);
                        ex += sq & D_VAL;
                        done = (sq >> 30) == 2;
                    }
                }
                if (done) break;
            }
            if (tile > 0) st_relaxed_u32(status + tile * NB + d, D_INC | (ex + cnt[q]));
            return ex;
        };
        unsigned incl = loc;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned t = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += t;
        }
        if (lane == 31) s_wsum[warp] = incl;
        __syncthreads();
        unsigned wpre = 0;
        for (int w = 0; w < warp; w++) wpre += s_wsum[w];
        unsigned tex[DPT];   // tile-local start of each owned digit
        {
            unsigned run = wpre + incl - loc;
#pragma unroll
            for (int q = 0; q < DPT; q++) {
                tex[q] = run;
                run += cnt[q];
                unsigned c = tex[q];
#pragma unroll
                for (int w = 0; w < S_WARPS; w++) {
                    if constexpr (DPT == 1) {
                        s_cnt[w][tid] = tex[q] + wex[w];
                    } else {
                        const unsigned t = s_cnt[w][tid * DPT + q];
                        s_cnt[w][tid * DPT + q] = c;
                        c += t;
                    }
                }
            }
        }
        __syncthreads();

        // 3. stable ranks.  Equal digits of a row are found with 8 ballots
        // (one per digit bit: cheap ALU/vote work, where __match_any_sync is
        // a long-latency, low-throughput instruction); the group's highest
        // lane advances the (warp, digit) counter, seeded with the tile-local
        // start, so each item gets its tile position directly.
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const unsigned dj = (tile_n == TILE || warp * 32 * ITEMS + j * 32 + lane < tile_n)
                                    ? ((unsigned)(key[j] >> shift) & DM) : DM;
            const unsigned peers = match_digit<RB>(dj);
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
#pragma unroll
        for (int q = 0; q < DPT; q++) {
            const unsigned excl = lookback(q);
            s_off[tid * DPT + q] = digit_base[tid * DPT + q] + excl - tex[q];
        }
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
        for (int i = tid; i < S_WARPS * NB; i += S_THREADS) (&s_cnt[0][0])[i] = 0;
#pragma unroll 4
        for (int p = tid; p < tile_n; p += S_THREADS) {
            const K k = s_k[p];
            const long long dst = (long long)s_off[(unsigned)(k >> shift) & DM] + p;
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

// Histograms of the digits that vary (the others were dropped using the
// AND / OR masks the S' filter computed): one pass over the keys, per-CTA
// shared-memory bins, one global atomic per bin per CTA.  NB = 256 or 512
// bins per pass (8- or 9-bit digits).
struct DigitList {
    int n;
    int shift[8];
};

template <typename K, int NB>
__global__ void __launch_bounds__(256) digit_hist_kernel(const K *__restrict__ keys, long long n, DigitList dl,
                                                         unsigned *__restrict__ hist,
                                                         unsigned *__restrict__ done,
                                                         unsigned *__restrict__ digit_base, K encx)
{
    __shared__ unsigned s_hist[8 * NB];
    __shared__ bool s_last;
    __shared__ unsigned s_w[8];
    for (int i = threadIdx.x; i < dl.n * NB; i += 256) s_hist[i] = 0;
    __syncthreads();
    // HB keys per thread per round are loaded before any is counted: the
    // shared-memory atomics would otherwise serialise one DRAM round trip per
    // key (a small S' has only a few CTAs, each with a long chain)
    constexpr int HB = 8;
    const long long stride = (long long)gridDim.x * 256;
    for (long long i0 = blockIdx.x * 256LL + threadIdx.x; i0 < n; i0 += stride * HB) {
        K k[HB];
#pragma unroll
        for (int u = 0; u < HB; u++) k[u] = i0 + u * stride < n ? (K)(__ldg(keys + i0 + u * stride) ^ encx) : (K)0;
#pragma unroll
        for (int u = 0; u < HB; u++) {
            if (i0 + u * stride >= n) break;
#pragma unroll
            for (int p = 0; p < 8; p++)
                if (p < dl.n) atomicAdd(&s_hist[p * NB + (unsigned)((k[u] >> dl.shift[p]) & (NB - 1))], 1u);
        }
    }
    __syncthreads();
    for (int i = threadIdx.x; i < dl.n * NB; i += 256)
        if (s_hist[i]) atomicAdd(&hist[i], s_hist[i]);
    // the last CTA to finish scans every pass's bins into the digit bases
    // (replaces a separate scan launch)
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_last = atomicAdd(done, 1u) == gridDim.x - 1;
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    constexpr int PER = NB / 256;   // bins per thread (consecutive)
    for (int p = 0; p < dl.n; p++) {
        unsigned c[PER], s = 0;
#pragma unroll
        for (int q = 0; q < PER; q++) {
            c[q] = __ldcg(hist + p * NB + threadIdx.x * PER + q);
            s += c[q];
        }
        unsigned incl = s;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned v = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += v;
        }
        if (lane == 31) s_w[warp] = incl;
        __syncthreads();
        unsigned run = incl - s;
        for (int w = 0; w < warp; w++) run += s_w[w];
#pragma unroll
        for (int q = 0; q < PER; q++) {
            digit_base[p * NB + threadIdx.x * PER + q] = run;
            run += c[q];
        }
        __syncthreads();
    }
}

size_t hist_bytes() { return 8 * 512 * 4 + 256; }

cudaError_t launch_digit_hist(int kb, const void *keys, long long n, const int *shifts, int np, unsigned *hist,
                              unsigned *digit_base, int num_sms, cudaStream_t st, long long *launches, int rb,
                              bool prezeroed, unsigned long long encx)
{
    if (np <= 0) return cudaSuccess;
    const int nb = 1 << rb;
    // hist holds 8 * 512 bins + the CTA-done counter at hist[8 * 512]
    unsigned *done = hist + 8 * 512;
    cudaError_t e = prezeroed ? cudaSuccess : cudaMemsetAsync(hist, 0, hist_bytes(), st);
    if (e != cudaSuccess) return e;
    DigitList dl{};
    dl.n = np;
    for (int p = 0; p < np; p++) dl.shift[p] = shifts[p];
    // >= 4096 keys per CTA: the shared bins' init / merge and the last CTA's
    // scan stay small next to the counting
    long long blocks = (n + NG_H_KEYS - 1) / NG_H_KEYS;
    if (blocks > (long long)num_sms * 8) blocks = (long long)num_sms * 8;
    if (blocks < 1) blocks = 1;
    if (rb == 8) {
        if (kb == 4) digit_hist_kernel<uint32_t, 256><<<(unsigned)blocks, 256, 0, st>>>((const uint32_t *)keys, n, dl, hist, done, digit_base, (uint32_t)encx);
        else digit_hist_kernel<uint64_t, 256><<<(unsigned)blocks, 256, 0, st>>>((const uint64_t *)keys, n, dl, hist, done, digit_base, (uint64_t)encx);
    } else {
        if (kb == 4) digit_hist_kernel<uint32_t, 512><<<(unsigned)blocks, 256, 0, st>>>((const uint32_t *)keys, n, dl, hist, done, digit_base, (uint32_t)encx);
        else digit_hist_kernel<uint64_t, 512><<<(unsigned)blocks, 256, 0, st>>>((const uint64_t *)keys, n, dl, hist, done, digit_base, (uint64_t)encx);
    }
    *launches += 1;
    return cudaGetLastError();
}

// NG_S_PREAGG: every tile's per-digit counts published (as look-back AGG
// statuses, tile 0 as INC) by one extra pass over the keys before the
// radix pass, so the pass's look-back never waits for a predecessor to load
// and count its tile -- it only sums published counts back to the nearest
// inclusive prefix.  Also zeroes the tile counter.
template <typename K, int NB, int TILE>
__global__ void __launch_bounds__(256) tile_agg_kernel(const K *__restrict__ keys, long long n, int shift,
                                                       unsigned *__restrict__ status, unsigned *__restrict__ counter,
                                                       K encx)
{
    __shared__ unsigned h[NB];
    for (int d = threadIdx.x; d < NB; d += 256) h[d] = 0;
    __syncthreads();
    const long long t = blockIdx.x;
    const long long b0 = t * TILE;
    const long long b1 = min(n, b0 + TILE);
    for (long long i = b0 + threadIdx.x; i < b1; i += 256)
        atomicAdd(&h[(unsigned)((__ldg(keys + i) ^ encx) >> shift) & (NB - 1)], 1u);
    __syncthreads();
    for (int d = threadIdx.x; d < NB; d += 256) status[t * NB + d] = (t == 0 ? D_INC : D_AGG) | h[d];
    if (t == 0 && threadIdx.x == 0) *counter = 0;
}

template <typename K, int VB, typename KO, int RB>
static cudaError_t run_pass(const void *kin, void *kout, const void *vin, void *vout, long long n, int shift,
                            const unsigned *digit_base, void *scratch, unsigned hi, cudaStream_t st, bool prezeroed,
                            unsigned long long encx)
{
    using Cfg = PassCfg<K, VB, RB>;
    const long long tiles = (n + Cfg::TILE - 1) / Cfg::TILE;
    int grid_max = 0;   // resident CTAs (persistent grid), per instantiation and device
    cudaError_t e = per_device_setup((const void *)onesweep_p_kernel<K, VB, KO, RB>, 0, &grid_max,
                                     [](int dev, int *v) {
        cudaError_t e1 = cudaFuncSetAttribute(onesweep_p_kernel<K, VB, KO, RB>,
                                              cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Cfg::SMEM);
        if (e1 != cudaSuccess) return e1;
        int sms = 0, occ = 0;
        if ((e1 = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e1;
        if ((e1 = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, onesweep_p_kernel<K, VB, KO, RB>, S_THREADS,
                                                                Cfg::SMEM)) != cudaSuccess)
            return e1;
        if (occ < 1) return cudaErrorInvalidConfiguration;
        *v = sms * occ;
        return cudaSuccess;
    });
    if (e != cudaSuccess) return e;
    if (NG_S_PREAGG) {
        tile_agg_kernel<K, (1 << RB), Cfg::TILE><<<(unsigned)tiles, 256, 0, st>>>(
            (const K *)kin, n, shift, (unsigned *)((char *)scratch + 256), (unsigned *)scratch, (K)encx);
    } else if (!prezeroed) {
        e = cudaMemsetAsync(scratch, 0, (size_t)tiles * (1 << RB) * 4 + 256, st);
        if (e != cudaSuccess) return e;
    }
    const unsigned grid = (unsigned)(tiles < grid_max ? tiles : grid_max);
    onesweep_p_kernel<K, VB, KO, RB><<<grid, S_THREADS, Cfg::SMEM, st>>>(
        (const K *)kin, (KO *)kout, vin, vout, n, shift, digit_base, (unsigned *)((char *)scratch + 256),
        (unsigned *)scratch, hi, (K)encx);
    return cudaGetLastError();
}

template <typename K, typename KO, int RB>
static cudaError_t run_pass_v(int vb, const void *kin, void *kout, const void *vin, void *vout, long long n, int shift,
                              const unsigned *digit_base, void *scratch, unsigned hi, cudaStream_t st, bool pz,
                              unsigned long long encx)
{
    if (vb == 0) return run_pass<K, 0, KO, RB>(kin, kout, vin, vout, n, shift, digit_base, scratch, hi, st, pz, encx);
    if (vb == 4) return run_pass<K, 4, KO, RB>(kin, kout, vin, vout, n, shift, digit_base, scratch, hi, st, pz, encx);
    return run_pass<K, 8, KO, RB>(kin, kout, vin, vout, n, shift, digit_base, scratch, hi, st, pz, encx);
}

template <int RB>
static cudaError_t run_pass_kk(int kb_in, int kb_out, int vb, const void *kin, void *kout, const void *vin,
                               void *vout, long long n, int shift, const unsigned *digit_base, void *scratch,
                               unsigned hi, cudaStream_t st, bool pz, unsigned long long encx)
{
#define NG_RPV(KI, KO_) run_pass_v<KI, KO_, RB>(vb, kin, kout, vin, vout, n, shift, digit_base, scratch, hi, st, pz, encx)
    if (kb_in == 4 && kb_out == 4) return NG_RPV(uint32_t, uint32_t);
    if (kb_in == 8 && kb_out == 8) return NG_RPV(uint64_t, uint64_t);
    if (kb_in == 8) return NG_RPV(uint64_t, uint32_t);
    return NG_RPV(uint32_t, uint64_t);
#undef NG_RPV
}

cudaError_t launch_radix_pass_x(int kb_in, int kb_out, int vb, const void *kin, void *kout, const void *vin,
                                void *vout, long long n, int shift, const unsigned *digit_base, void *scratch,
                                unsigned hi, cudaStream_t st, long long *launches, int rb, bool prezeroed,
                                unsigned long long encx)
{
    if (n <= 0) return cudaSuccess;
    if (n >= (1ll << 30)) return cudaErrorInvalidValue;
    if (rb != 8 && rb != 9) return cudaErrorInvalidValue;
    const cudaError_t e = rb == 8 ? run_pass_kk<8>(kb_in, kb_out, vb, kin, kout, vin, vout, n, shift, digit_base,
                                                   scratch, hi, st, prezeroed, encx)
                                  : run_pass_kk<9>(kb_in, kb_out, vb, kin, kout, vin, vout, n, shift, digit_base,
                                                   scratch, hi, st, prezeroed, encx);
    ++*launches;
    return e;
}

cudaError_t launch_radix_pass(int kb, int vb, const void *kin, void *kout, const void *vin, void *vout,
                              long long n, int shift, const unsigned *digit_base, void *scratch, cudaStream_t st,
                              long long *launches, int rb)
{
    return launch_radix_pass_x(kb, kb, vb, kin, kout, vin, vout, n, shift, digit_base, scratch, 0u, st, launches, rb);
}

}  // namespace ng
