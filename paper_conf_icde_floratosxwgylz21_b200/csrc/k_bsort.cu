// k_bsort.cu -- a4: index build as a two-round-trip MSD bucket sort.
//
// PAPER.md P:315 (§III-D "Indexing"): sort the correlated column and
// binary-search a qualifying range per outer tuple.  The LSD onesweep
// (k_sort.cu) reads and writes every (key, payload) once per 8/9-bit digit:
// 3-4 HBM round trips for 26-32-bit keys, each bound by its in-tile ranking
// (8 warp ballots per row of 32 items) and its look-back chain.  This sort
// makes two round trips over the data:
//
//   1. group histograms of the top D varying key bits (2^D buckets):
//      H[group][d] (u16); a two-kernel column scan rewrites H in place as each
//      group's start inside every bucket (u16: a bucket never exceeds the
//      finish capacity, checked) and produces the bucket bases (u32) and the
//      largest bucket -- the host falls back to the LSD sort when a bucket
//      would not fit shared memory (skewed keys);
//   2. partition: a CTA takes one group (a few tiles); each tile is sorted
//      stably by its D-bit digit in shared memory and written out run by run
//      at  base[d] + H[group][d] + (items of d in earlier tiles of the group)
//      + (position - run start)  -- no look-back chain, the offsets were
//      scanned beforehand;
//   3. finish: one CTA per bucket loads it into shared memory, sorts the
//      remaining varying bits stably (<= 6 bits per pass) and writes the
//      bucket back coalesced (re-attaching a constant high key word).
//
// In-block ranking is counter based (no ballots, no match.any -- 27 and 60
// SM cycles per 32-item row on this part, tools/rank_micro.cu): each thread
// owns I consecutive items (blocked arrangement) and one packed pair of
// 16-bit counters per digit pair in a [lane][thread] word array; it counts
// its own items sequentially (stable by construction, priors kept as bytes),
// a raking exclusive scan over the words in memory order turns the counters
// into rank bases, and each item adds its prior.  Blocked shared-memory reads
// use 16-byte vectors under an XOR chunk swizzle so that 8 consecutive
// threads hit 8 different bank quads.  Every step is stable, so equal keys
// keep their S' order: the index equals the LSD sort's, byte for byte.
#include <type_traits>

#include "internal.h"

namespace ng {

constexpr int BS_T = 256;   // threads per CTA (partition and finish)

constexpr int ilog2c(int x) { return x <= 1 ? 0 : 1 + ilog2c(x / 2); }

// XOR-swizzled blocked layout: element p of a T x I block belongs to thread
// p / I; its 16-byte chunk is permuted within the thread's chunks.
template <int ES, int I>
struct Swz {
    static constexpr int E = 16 / ES;   // elements per 16-byte chunk
    static constexpr int C = I / E;     // chunks per thread
    static_assert(C >= 1 && (C & (C - 1)) == 0, "chunks per thread must be a power of two");
    static constexpr int LI = ilog2c(I), LE = ilog2c(E);
    __device__ static __forceinline__ int f(int t)
    {
        if constexpr (C >= 8) return t & 7;
        else return (t / (8 / C)) & (C - 1);
    }
    __device__ static __forceinline__ int phys(int p)
    {
        const int t = p >> LI, i = p & (I - 1);
        return ((t * C + ((i >> LE) ^ f(t))) << LE) + (i & (E - 1));
    }
};

template <typename T>
union Vec16 {
    uint4 v;
    T e[16 / sizeof(T)];
};

template <typename T, int I>
__device__ __forceinline__ void smem_read_blocked(const T *s, T (&x)[I])
{
    using S = Swz<sizeof(T), I>;
    const int t = threadIdx.x;
    const uint4 *s4 = reinterpret_cast<const uint4 *>(s);
#pragma unroll
    for (int c = 0; c < S::C; c++) {
        Vec16<T> u;
        u.v = s4[t * S::C + (c ^ S::f(t))];
#pragma unroll
        for (int e = 0; e < S::E; e++) x[c * S::E + e] = u.e[e];
    }
}

// thread t's items [base + t*I, base + t*I + I) of src[0, n); pad past n
template <typename T, int I>
__device__ __forceinline__ void gmem_read_blocked(const T *__restrict__ src, long long base, long long n, T (&x)[I],
                                                  T pad)
{
    const long long b = base + (long long)threadIdx.x * I;
    if (b + I <= n) {
        const uint4 *s4 = reinterpret_cast<const uint4 *>(src + b);
        constexpr int E = 16 / sizeof(T);
#pragma unroll
        for (int c = 0; c < I / E; c++) {
            Vec16<T> u;
            u.v = __ldg(s4 + c);
#pragma unroll
            for (int e = 0; e < E; e++) x[c * E + e] = u.e[e];
        }
    } else {
#pragma unroll
        for (int i = 0; i < I; i++) x[i] = b + i < n ? src[b + i] : pad;
    }
}

template <typename K>
__device__ __forceinline__ unsigned digit_of(K k, int shift, unsigned mask)
{
    return (unsigned)(k >> shift) & mask;
}

template <typename K, typename KO>
__device__ __forceinline__ KO key_out(K k, unsigned hi)
{
    if constexpr (sizeof(KO) > sizeof(K)) return ((KO)hi << 32) | (KO)k;
    else return (KO)k;
}

// An opaque copy: the compiler must recompute what it derives from x
// instead of keeping it live across a barrier (digit addresses of I items
// would double the registers of the ranking pass).
template <typename K>
__device__ __forceinline__ K opaque(K x)
{
    if constexpr (sizeof(K) == 8) {
        unsigned long long y = x;
        asm volatile("" : "+l"(y));
        return (K)y;
    } else {
        unsigned y = x;
        asm volatile("" : "+r"(y));
        return (K)y;
    }
}

struct BsPasses {
    int n;
    int shift[12];
    int bits[12];
};

// One stable counter-ranking pass over the block's T*I blocked items by the
// digit (key >> shift) & (2^bits - 1), bits <= MAXB, then the items are
// scattered to their ranks in s_k / s_v (swizzled).  cnt: (2^(MAXB-1) + 1)
// * T words; wsum: T/32 words.  The caller has passed a barrier since the
// previous pass (every thread holds its items; cnt and the buffers are free);
// the scatter is followed by a barrier.
template <typename K, typename V, int VB, int T, int I>
__device__ __forceinline__ void rank_scatter(const K (&key)[I], const V (&val)[I], int shift, int bits, K *s_k,
                                             V *s_v, unsigned *cnt, unsigned *wsum)
{
    using SK = Swz<sizeof(K), I>;
    using SV = Swz<sizeof(V), I>;
    const int t = threadIdx.x;
    const int hb = bits - 1;
    const unsigned nl = 1u << hb, dm = (1u << bits) - 1;
    for (unsigned l = 0; l <= nl; l++) cnt[l * T + t] = 0;
    unsigned pr[(I + 3) / 4];   // sequential priors (< I <= 64), one byte each
#pragma unroll
    for (int q = 0; q < (I + 3) / 4; q++) pr[q] = 0;
#pragma unroll
    for (int i = 0; i < I; i++) {
        const unsigned d = digit_of(key[i], shift, dm);
        const unsigned a = (d & (nl - 1)) * T + t;
        const unsigned sh = (d >> hb) << 4;
        const unsigned w = cnt[a];
        pr[i / 4] |= ((w >> sh) & 0xffu) << (8 * (i % 4));
        cnt[a] = w + (1u << sh);
    }
    __syncthreads();
    // raking exclusive scan of the (nl + 1) x T words in memory order; the
    // odd segment length keeps the 32 lanes of a warp on 32 banks
    const unsigned seg = nl + 1;
    unsigned *sp = cnt + t * seg;
    unsigned s = 0;
    for (unsigned k = 0; k < seg; k++) s += sp[k];
    const int lane = t & 31, warp = t >> 5;
    unsigned inc = s;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned v = __shfl_up_sync(FULL, inc, o);
        if (lane >= o) inc += v;
    }
    if (lane == 31) wsum[warp] = inc;
    __syncthreads();
    unsigned run = inc - s, tot = 0;
#pragma unroll
    for (int w = 0; w < T / 32; w++) {
        const unsigned x = wsum[w];
        if (w < warp) run += x;
        tot += x;
    }
    for (unsigned k = 0; k < seg; k++) {
        const unsigned v = sp[k];
        sp[k] = run;
        run += v;
    }
    __syncthreads();
    // low halves hold digits [0, nl), high halves [nl, 2 nl): the high
    // digits come after every low one.  Every thread read its items before
    // the first barrier above, so the scatter may overwrite the buffers.
    const unsigned lowtot = tot & 0xffffu;
#pragma unroll
    for (int i = 0; i < I; i++) {
        const unsigned d = digit_of(opaque(key[i]), shift, dm);
        const unsigned a = (d & (nl - 1)) * T + t;
        const unsigned sh = (d >> hb) << 4;
        const unsigned r = ((cnt[a] >> sh) & 0xffffu) + (sh ? lowtot : 0u) + ((pr[i / 4] >> (8 * (i % 4))) & 0xffu);
        s_k[SK::phys(r)] = key[i];
        if constexpr (VB > 0) s_v[SV::phys(r)] = val[i];
    }
    __syncthreads();
}

// Sort the block's blocked register items stably by the listed digits
// (least significant first).  On return the T*I items sit sorted in s_k /
// s_v (swizzled), after a barrier.
template <typename K, typename V, int VB, int T, int I>
__device__ __forceinline__ void sort_block(K (&key)[I], V (&val)[I], const BsPasses &ps, K *s_k, V *s_v,
                                           unsigned *cnt, unsigned *wsum)
{
    for (int p = 0; p < ps.n; p++) {
        if (p > 0) {
            smem_read_blocked<K, I>(s_k, key);
            if constexpr (VB > 0) smem_read_blocked<V, I>(s_v, val);
        }
        rank_scatter<K, V, VB, T, I>(key, val, ps.shift[p], ps.bits[p], s_k, s_v, cnt, wsum);
    }
}

// ---------------------------------------------------------------------------
// Step 1a: per-group histograms of the D-bit bucket digit (u16 per group and
// bucket; groups of `group` items, a multiple of 16 bytes of keys).
template <typename K>
__global__ void __launch_bounds__(256) bs_grouphist_kernel(const K *__restrict__ keys, long long n, int group, int s1,
                                                           int nb, uint16_t *__restrict__ H)
{
    __shared__ unsigned h[4096];
    for (int d = threadIdx.x; d < nb; d += 256) h[d] = 0;
    __syncthreads();
    const long long b0 = (long long)blockIdx.x * group;
    const long long b1 = min(n, b0 + group);
    const unsigned dm = (unsigned)nb - 1;
    constexpr int E = 16 / sizeof(K);
    const long long nv = (b1 - b0) / E;   // whole 16-byte vectors
    const uint4 *s4 = reinterpret_cast<const uint4 *>(keys + b0);
#pragma unroll 4
    for (long long c = threadIdx.x; c < nv; c += 256) {
        Vec16<K> u;
        u.v = __ldg(s4 + c);
#pragma unroll
        for (int e = 0; e < E; e++) atomicAdd(&h[digit_of(u.e[e], s1, dm)], 1u);
    }
    for (long long i = b0 + nv * E + threadIdx.x; i < b1; i += 256) atomicAdd(&h[digit_of(keys[i], s1, dm)], 1u);
    __syncthreads();
    uint16_t *row = H + (size_t)blockIdx.x * nb;
    for (int d = threadIdx.x; d < nb; d += 256) row[d] = (uint16_t)h[d];
}

// Step 1b: column sums.  grid (nb / 64, slabs); warp w of CTA (c, y) sums
// band y*8 + w (rpb consecutive rows) of buckets [64c, 64c + 64) (two per
// lane) into part[band][d], and adds them to tot[d] (zeroed).  The last CTA
// scans tot into base[0..nb] and writes the largest bucket to *maxb.
__global__ void __launch_bounds__(256) bs_colsum_kernel(const uint16_t *__restrict__ H, int nrows, int nb, int rpb,
                                                        unsigned *__restrict__ part, unsigned *__restrict__ tot,
                                                        unsigned *__restrict__ base, unsigned *__restrict__ maxb,
                                                        unsigned *__restrict__ done)
{
    __shared__ bool s_last;
    __shared__ unsigned s_w[8], s_m[8];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int d0 = blockIdx.x * 64 + 2 * lane;
    const int band = blockIdx.y * 8 + warp;
    const int r0 = band * rpb, r1 = min(nrows, r0 + rpb);
    unsigned a = 0, b = 0;
    if (d0 < nb) {
#pragma unroll 8
        for (int r = r0; r < r1; r++) {
            const unsigned w = __ldg(reinterpret_cast<const unsigned *>(H + (size_t)r * nb + d0));
            a += w & 0xffffu;
            b += w >> 16;
        }
        part[(size_t)band * nb + d0] = a;
        part[(size_t)band * nb + d0 + 1] = b;
        if (a) atomicAdd(tot + d0, a);
        if (b) atomicAdd(tot + d0 + 1, b);
    }
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_last = atomicAdd(done, 1u) == gridDim.x * gridDim.y - 1;
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    // last CTA: exclusive scan of the nb (<= 4096) totals, 16 per thread
    const int per = (nb + 255) / 256;
    const int q0 = threadIdx.x * per;
    unsigned s = 0, m = 0;
    for (int q = q0; q < min(nb, q0 + per); q++) {
        const unsigned x = __ldcg(tot + q);
        s += x;
        m = max(m, x);
    }
    unsigned inc = s;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned v = __shfl_up_sync(FULL, inc, o);
        if (lane >= o) inc += v;
    }
    unsigned wm = m;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) wm = max(wm, __shfl_xor_sync(FULL, wm, o));
    if (lane == 31) s_w[warp] = inc;
    if (lane == 0) s_m[warp] = wm;
    __syncthreads();
    unsigned run = inc - s, total = 0, allm = 0;
    for (int w = 0; w < 8; w++) {
        if (w < warp) run += s_w[w];
        total += s_w[w];
        allm = max(allm, s_m[w]);
    }
    for (int q = q0; q < min(nb, q0 + per); q++) {
        base[q] = run;
        run += __ldcg(tot + q);
    }
    if (threadIdx.x == 0) {
        base[nb] = total;
        *maxb = allm;
    }
}

// Step 1c: H[r][d] <- sum of H[r'][d] over rows r' < r (in place, u16 pairs).
__global__ void __launch_bounds__(256) bs_colapply_kernel(uint16_t *__restrict__ H, int nrows, int nb, int rpb,
                                                          const unsigned *__restrict__ part)
{
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int d0 = blockIdx.x * 64 + 2 * lane;
    const int band = blockIdx.y * 8 + warp;
    const int r0 = band * rpb, r1 = min(nrows, r0 + rpb);
    if (d0 >= nb || r0 >= r1) return;
    unsigned a = 0, b = 0;
#pragma unroll 8
    for (int q = 0; q < band; q++) {
        a += __ldg(part + (size_t)q * nb + d0);
        b += __ldg(part + (size_t)q * nb + d0 + 1);
    }
    for (int r = r0; r < r1; r++) {
        unsigned *p = reinterpret_cast<unsigned *>(H + (size_t)r * nb + d0);
        const unsigned w = *p;
        *p = (a & 0xffffu) | (b << 16);   // buckets past 16 bits are rejected by *maxb
        a += w & 0xffffu;
        b += w >> 16;
    }
}

// ---------------------------------------------------------------------------
// Step 2: partition.  CTA = one group of GT tiles of T*I items.  Each tile is
// sorted by the D-bit digit in shared memory, run starts / ends are found by
// comparing neighbours, and item p of digit d goes to
//   goff[d] + (p - start[d]),   goff[d] = base[d] + H[group][d] + (earlier tiles' d items).
constexpr int BS_PART_MAXB = 5;   // sub-pass digit bits (counter area 17 x T words)
constexpr int BS_PART_CNT = ((1 << (BS_PART_MAXB - 1)) + 1) * BS_T;
constexpr int BS_FIN_MAXB = 6;
constexpr int BS_FIN_CNT = ((1 << (BS_FIN_MAXB - 1)) + 1) * BS_T;
constexpr int BS_GROUP = 32768;   // items per partition group

template <typename K, int VB>
struct BsShape {
    static constexpr int I = (sizeof(K) == 4 && VB == 0) ? 64 : ((int)sizeof(K) + VB <= 8 ? 32 : 16);
    static constexpr int TILE = BS_T * I;
    static constexpr int GT = BS_GROUP / TILE;
};

template <typename K, int VB, typename KO>
__global__ void __launch_bounds__(BS_T, 2) bs_part_kernel(const K *__restrict__ kin, const void *__restrict__ vin_,
                                                          KO *__restrict__ kout, void *__restrict__ vout_, long long n,
                                                          BsPasses ps, int s1, int nb,
                                                          const uint16_t *__restrict__ H,
                                                          const unsigned *__restrict__ base, unsigned hi)
{
    using V = typename std::conditional<VB == 8, unsigned long long, unsigned>::type;
    constexpr int T = BS_T, I = BsShape<K, VB>::I, TILE = BsShape<K, VB>::TILE, GT = BsShape<K, VB>::GT;
    using SK = Swz<sizeof(K), I>;
    using SV = Swz<sizeof(V), I>;
    const V *vin = (const V *)vin_;
    V *vout = (V *)vout_;
    extern __shared__ __align__(16) unsigned char smem[];
    K *s_k = (K *)smem;
    V *s_v = (V *)(smem + (size_t)TILE * sizeof(K));
    unsigned *cnt = (unsigned *)(smem + (size_t)TILE * (sizeof(K) + VB));
    unsigned *s_goff = cnt + BS_PART_CNT;                 // [nb]
    uint16_t *s_start = (uint16_t *)cnt, *s_end = s_start + nb;   // overlay the counters
    __shared__ unsigned wsum[T / 32];
    const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
    const unsigned dm = (unsigned)nb - 1;
    {
        const uint16_t *row = H + (size_t)blockIdx.x * nb;
        for (int d = t; d < nb; d += T) s_goff[d] = __ldg(base + d) + (unsigned)__ldg(row + d);
    }
    for (int g = 0; g < GT; g++) {
        const long long tb = (long long)blockIdx.x * BS_GROUP + (long long)g * TILE;
        if (tb >= n) break;
        const int m = (int)min((long long)TILE, n - tb);
        K key[I];
        V val[I];
        gmem_read_blocked<K, I>(kin, tb, n, key, (K)~(K)0);
        if constexpr (VB > 0) gmem_read_blocked<V, I>(vin, tb, n, val, (V)0);
        sort_block<K, V, VB, T, I>(key, val, ps, s_k, s_v, cnt, wsum);
        for (int d = t; d < nb; d += T) s_end[d] = 0;
        __syncthreads();
        // run boundaries: neighbours by shuffle, lanes 0 / 31 from shared memory
        for (int p0 = warp * 32; p0 < m; p0 += T) {
            const int p = p0 + lane;
            const unsigned d = p < m ? digit_of(s_k[SK::phys(p)], s1, dm) : 0xffffffffu;
            unsigned dp = __shfl_up_sync(FULL, d, 1), dn = __shfl_down_sync(FULL, d, 1);
            if (lane == 0) dp = p > 0 ? digit_of(s_k[SK::phys(p - 1)], s1, dm) : 0xffffffffu;
            if (lane == 31) dn = p + 1 < m ? digit_of(s_k[SK::phys(p + 1)], s1, dm) : 0xffffffffu;
            if (p < m) {
                if (dp != d) s_start[d] = (uint16_t)p;
                if (dn != d) s_end[d] = (uint16_t)(p + 1);
            }
        }
        __syncthreads();
#pragma unroll 4
        for (int p = t; p < m; p += T) {
            const K k = s_k[SK::phys(p)];
            const unsigned d = digit_of(k, s1, dm);
            const unsigned dst = s_goff[d] + (unsigned)p - (unsigned)s_start[d];
            kout[dst] = key_out<K, KO>(k, hi);
            if constexpr (VB > 0) vout[dst] = s_v[SV::phys(p)];
        }
        __syncthreads();
        for (int d = t; d < nb; d += T) {
            const unsigned e = s_end[d];
            if (e) s_goff[d] += e - (unsigned)s_start[d];
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------------------
// Step 3: finish one bucket [s, s + m) of m <= T*I items.
template <typename K, int VB, typename KO, int I>
__device__ __forceinline__ void bucket_body(const K *__restrict__ kin, const void *__restrict__ vin_,
                                            KO *__restrict__ kout, void *__restrict__ vout_, unsigned s, int m,
                                            const BsPasses &ps, unsigned hi, unsigned char *smem, unsigned *wsum,
                                            int tile_cap)
{
    using V = typename std::conditional<VB == 8, unsigned long long, unsigned>::type;
    constexpr int T = BS_T, TILE = T * I;
    using SK = Swz<sizeof(K), I>;
    using SV = Swz<sizeof(V), I>;
    const V *vin = (const V *)vin_;
    V *vout = (V *)vout_;
    K *s_k = (K *)smem;
    V *s_v = (V *)(smem + (size_t)tile_cap * sizeof(K));
    unsigned *cnt = (unsigned *)(smem + (size_t)tile_cap * (sizeof(K) + VB));
    const int t = threadIdx.x;
    // coalesced load into the swizzled blocked layout, padded with all-ones
    // keys (they rank after every real item of the last digit)
#pragma unroll 4
    for (int p = t; p < TILE; p += T) {
        s_k[SK::phys(p)] = p < m ? kin[s + p] : (K)~(K)0;
        if constexpr (VB > 0) s_v[SV::phys(p)] = p < m ? vin[s + p] : (V)0;
    }
    __syncthreads();
    K key[I];
    V val[I];
    smem_read_blocked<K, I>(s_k, key);
    if constexpr (VB > 0) smem_read_blocked<V, I>(s_v, val);
    sort_block<K, V, VB, T, I>(key, val, ps, s_k, s_v, cnt, wsum);
#pragma unroll 4
    for (int p = t; p < m; p += T) {
        kout[s + p] = key_out<K, KO>(s_k[SK::phys(p)], hi);
        if constexpr (VB > 0) vout[s + p] = s_v[SV::phys(p)];
    }
}

template <typename K, int VB, typename KO>
__global__ void __launch_bounds__(BS_T, 2) bs_bucket_kernel(const K *__restrict__ kin, const void *__restrict__ vin,
                                                            KO *__restrict__ kout, void *__restrict__ vout,
                                                            const unsigned *__restrict__ base, BsPasses ps, unsigned hi)
{
    using V = typename std::conditional<VB == 8, unsigned long long, unsigned>::type;
    constexpr int IMAX = BsShape<K, VB>::I, CAP = BS_T * IMAX;
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ unsigned wsum[BS_T / 32];
    const unsigned s = __ldg(base + blockIdx.x);
    const int m = (int)(__ldg(base + blockIdx.x + 1) - s);
    if (m <= 0) return;
    if (m == 1) {
        if (threadIdx.x == 0) {
            kout[s] = key_out<K, KO>(kin[s], hi);
            if constexpr (VB > 0) ((V *)vout)[s] = ((const V *)vin)[s];
        }
        return;
    }
    // the smallest register tile that holds the bucket
    if (m <= BS_T * 8) bucket_body<K, VB, KO, 8>(kin, vin, kout, vout, s, m, ps, hi, smem, wsum, CAP);
    else if (m <= BS_T * 16 || IMAX == 16) bucket_body<K, VB, KO, 16>(kin, vin, kout, vout, s, m, ps, hi, smem, wsum, CAP);
    else if constexpr (IMAX >= 32) {
        if (m <= BS_T * 32 || IMAX == 32) bucket_body<K, VB, KO, 32>(kin, vin, kout, vout, s, m, ps, hi, smem, wsum, CAP);
        else if constexpr (IMAX >= 64) bucket_body<K, VB, KO, 64>(kin, vin, kout, vout, s, m, ps, hi, smem, wsum, CAP);
    }
}

// ---------------------------------------------------------------------------
// Host side.
template <typename K, int VB>
static int cap_t() { return BS_T * BsShape<K, VB>::I; }

int bsort_capacity(int kb_mid, int vb)
{
    if (kb_mid == 4) return vb == 0 ? cap_t<uint32_t, 0>() : (vb == 4 ? cap_t<uint32_t, 4>() : cap_t<uint32_t, 8>());
    return vb == 0 ? cap_t<uint64_t, 0>() : (vb == 4 ? cap_t<uint64_t, 4>() : cap_t<uint64_t, 8>());
}

int bsort_group() { return BS_GROUP; }

static void col_grid(long long nrows, int nb, int *slabs, int *rpb)
{
    // ~4 CTAs per column group and >= 2 rows per band
    int y = 4;
    while (y > 1 && (long long)y * 8 * 2 > nrows) y /= 2;
    *slabs = y;
    *rpb = (int)((nrows + (long long)y * 8 - 1) / ((long long)y * 8));
}

size_t bsort_hist_bytes(long long n, int nb)
{
    const long long rows = (n + BS_GROUP - 1) / BS_GROUP;
    int slabs, rpb;
    col_grid(rows, nb, &slabs, &rpb);
    const size_t hb = ((size_t)rows * nb * 2 + 255) / 256 * 256;
    const size_t pb = (size_t)slabs * 8 * nb * 4;
    return hb + pb;
}

size_t bsort_zero_bytes(int nb) { return ((size_t)nb * 4 + 4 + 255) / 256 * 256; }   // tot[nb] + done

cudaError_t launch_bsort_hist(int kb_in, const void *keys, long long n, int s1, int nb, void *hscratch,
                              unsigned *zscratch, unsigned *base, unsigned *maxb, cudaStream_t st, long long *launches)
{
    const long long rows = (n + BS_GROUP - 1) / BS_GROUP;
    if (nb > 4096 || nb < 2 || rows <= 0) return cudaErrorInvalidValue;
    int slabs, rpb;
    col_grid(rows, nb, &slabs, &rpb);
    uint16_t *H = (uint16_t *)hscratch;
    unsigned *part = (unsigned *)((char *)hscratch + ((size_t)rows * nb * 2 + 255) / 256 * 256);
    unsigned *tot = zscratch, *done = zscratch + nb;
    if (kb_in == 4) bs_grouphist_kernel<uint32_t><<<(unsigned)rows, 256, 0, st>>>((const uint32_t *)keys, n, BS_GROUP, s1, nb, H);
    else bs_grouphist_kernel<uint64_t><<<(unsigned)rows, 256, 0, st>>>((const uint64_t *)keys, n, BS_GROUP, s1, nb, H);
    const dim3 g((unsigned)((nb + 63) / 64), (unsigned)slabs);
    bs_colsum_kernel<<<g, 256, 0, st>>>(H, (int)rows, nb, rpb, part, tot, base, maxb, done);
    bs_colapply_kernel<<<g, 256, 0, st>>>(H, (int)rows, nb, rpb, part);
    *launches += 3;
    return cudaGetLastError();
}

template <typename K, int VB, typename KO>
static cudaError_t part_t(const void *kin, const void *vin, void *kout, void *vout, long long n, const BsPasses &ps,
                          int s1, int nb, const uint16_t *H, const unsigned *base, unsigned hi, cudaStream_t st)
{
    const size_t sm = (size_t)BsShape<K, VB>::TILE * (sizeof(K) + VB) + (size_t)BS_PART_CNT * 4 + (size_t)nb * 4;
    int dummy = 0;
    cudaError_t e = per_device_setup((const void *)bs_part_kernel<K, VB, KO>, 0, &dummy, [](int, int *v) {
        *v = 1;
        const size_t mx = (size_t)BsShape<K, VB>::TILE * (sizeof(K) + VB) + (size_t)BS_PART_CNT * 4 + 4096 * 4;
        return cudaFuncSetAttribute(bs_part_kernel<K, VB, KO>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)mx);
    });
    if (e != cudaSuccess) return e;
    const long long groups = (n + BS_GROUP - 1) / BS_GROUP;
    bs_part_kernel<K, VB, KO><<<(unsigned)groups, BS_T, sm, st>>>((const K *)kin, vin, (KO *)kout, vout, n, ps, s1, nb,
                                                                  H, base, hi);
    return cudaGetLastError();
}

template <typename K, int VB, typename KO>
static cudaError_t bucket_t(const void *kin, const void *vin, void *kout, void *vout, int nb, const BsPasses &ps,
                            const unsigned *base, unsigned hi, cudaStream_t st)
{
    const size_t sm = (size_t)BsShape<K, VB>::TILE * (sizeof(K) + VB) + (size_t)BS_FIN_CNT * 4;
    int dummy = 0;
    cudaError_t e = per_device_setup((const void *)bs_bucket_kernel<K, VB, KO>, 0, &dummy, [sm](int, int *v) {
        *v = 1;
        return cudaFuncSetAttribute(bs_bucket_kernel<K, VB, KO>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    });
    if (e != cudaSuccess) return e;
    bs_bucket_kernel<K, VB, KO><<<(unsigned)nb, BS_T, sm, st>>>((const K *)kin, vin, (KO *)kout, vout, base, ps, hi);
    return cudaGetLastError();
}

#define NG_BS_VB(FN, K, KO, ...)                                                                         \
    (vb == 0 ? FN<K, 0, KO>(__VA_ARGS__) : (vb == 4 ? FN<K, 4, KO>(__VA_ARGS__) : FN<K, 8, KO>(__VA_ARGS__)))

cudaError_t launch_bsort_sort(int kb_in, int kb_mid, int kb_out, int vb, const void *kin, const void *vin,
                              void *kmid, void *vmid, void *kout, void *vout, long long n, int s1, int D,
                              const int *pshift, const int *pbits, int np2, const void *hscratch,
                              const unsigned *base, unsigned hi, cudaStream_t st, long long *launches)
{
    if (n <= 0) return cudaSuccess;
    if (D < 1 || D > 12 || np2 < 1 || np2 > 12) return cudaErrorInvalidValue;
    const int nb = 1 << D;
    const uint16_t *H = (const uint16_t *)hscratch;
    BsPasses p1{};
    {   // D bits in sub-passes of <= BS_PART_MAXB bits, least significant first
        const int k = (D + BS_PART_MAXB - 1) / BS_PART_MAXB;
        int sh = s1;
        for (int i = 0; i < k; i++) {
            const int b = D / k + (i < D % k ? 1 : 0);
            p1.shift[i] = sh;
            p1.bits[i] = b;
            sh += b;
        }
        p1.n = k;
    }
    BsPasses p2{};
    p2.n = np2;
    for (int i = 0; i < np2; i++) {
        if (pbits[i] < 1 || pbits[i] > BS_FIN_MAXB) return cudaErrorInvalidValue;
        p2.shift[i] = pshift[i];
        p2.bits[i] = pbits[i];
    }
    cudaError_t e;
    if (kb_in == 4 && kb_mid == 4) e = NG_BS_VB(part_t, uint32_t, uint32_t, kin, vin, kmid, vmid, n, p1, s1, nb, H, base, 0u, st);
    else if (kb_in == 8 && kb_mid == 8) e = NG_BS_VB(part_t, uint64_t, uint64_t, kin, vin, kmid, vmid, n, p1, s1, nb, H, base, 0u, st);
    else if (kb_in == 8 && kb_mid == 4) e = NG_BS_VB(part_t, uint64_t, uint32_t, kin, vin, kmid, vmid, n, p1, s1, nb, H, base, 0u, st);
    else return cudaErrorInvalidValue;
    if (e != cudaSuccess) return e;
    if (kb_mid == 4 && kb_out == 4) e = NG_BS_VB(bucket_t, uint32_t, uint32_t, kmid, vmid, kout, vout, nb, p2, base, hi, st);
    else if (kb_mid == 8 && kb_out == 8) e = NG_BS_VB(bucket_t, uint64_t, uint64_t, kmid, vmid, kout, vout, nb, p2, base, hi, st);
    else if (kb_mid == 4 && kb_out == 8) e = NG_BS_VB(bucket_t, uint32_t, uint64_t, kmid, vmid, kout, vout, nb, p2, base, hi, st);
    else return cudaErrorInvalidValue;
    *launches += 2;
    return e;
}
#undef NG_BS_VB

}  // namespace ng
