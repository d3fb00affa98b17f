// k_bnl.cuh -- a7: tiled block-nested-loop subquery kernel (non-equality
// correlations and index-less plans).
//
// PAPER.md P:55 (§I): the nested method "iterat[es] all tuples of the
// correlated columns from the outer query block and execut[es] the subquery
// as many times as the number of the outer-loop tuples" -- O(|R'| x |S'|).
// P:317 ("Vectorization"): evaluate many passed-in values in one kernel;
// abstract P:31: "exploiting cache locality for loops".  The B200 design:
//
//  * persistent CTAs (grid = #SMs x occupancy) pull work units
//    (R block of 2048 tuples) x (S' chunk) from an atomic counter;
//  * each thread keeps RPT = 8 outer tuples' encoded keys and accumulators
//    in registers, so every S' element read from shared memory is reused
//    2048 times per CTA (the cache-locality loop);
//  * S' (key, payload) tiles of 16 KB stream global -> shared through a
//    B_STAGES-deep ring (NG_B_STAGES, 3 by default) of cp.async.bulk copies (TMA bulk engine, UBLKCP) completed
//    on mbarriers by one elected thread; consumers read them with 128-bit
//    broadcast LDS;
//  * per (r, s) pair the work is one compare (ISETP) and one predicated
//    combine (IMNMX / IADD3) on the integer ALU pipe -- the roofline of this
//    kernel;
//  * EXISTS stops streaming a unit once every tuple of the block has found a
//    match (semi-join early exit);
//  * partial aggregates of a unit are merged into per-tuple int64 partials
//    with 64-bit atomics (MIN/MAX/ADD are associative and commutative on
//    integers, so the merge order cannot change the result).
#pragma once
#include <type_traits>

#include "internal.h"

namespace ng {

#ifndef NG_B_RPT
#define NG_B_RPT 8
#endif
#ifndef NG_B_STAGES
#define NG_B_STAGES 3
#endif
#ifndef NG_B_UNITS
#define NG_B_UNITS 64      // work units per persistent CTA (tail granularity vs per-unit fill + merge)
#endif
#ifndef NG_B_UNROLL
#define NG_B_UNROLL 2      // element groups per inner iteration (DESIGN.md §8 tuning log)
#endif
#ifndef NG_B_UNROLL_V0
#define NG_B_UNROLL_V0 4   // ... for COUNT / EXISTS / SUM with 32-bit keys
#endif
constexpr int B_THREADS = 256;
constexpr int B_RPT = NG_B_RPT;        // outer tuples per thread (register blocking)
constexpr int B_RBLOCK = B_THREADS * B_RPT;
constexpr int B_STAGES = NG_B_STAGES;  // shared-memory ring depth
constexpr int B_STAGE_BYTES = 16384;

struct BnlArgs {
    const long long *d_nrp;
    const long long *d_nsp;
    const void *rkeys;
    const void *skeys;
    const void *svals;
    const unsigned *extreme;   // [0] payload == max, [1] == min, (u64)[2..3] max |payload|
    unsigned one;              // runtime 1 (keeps the IMAD multiplier opaque to ptxas)
    long long *acc;
    long long *cnt;
    long long *acc_hi;         // SUM/AVG of 64-bit payloads, exact split accumulation (nullable)
    unsigned *unit_counter;
    unsigned *rb_done;         // EXISTS: per R block, set once every tuple of the block found a match
    long long target_units;    // work units to aim for (grid x 16)
    int shape;                 // R-block shape: 0 automatic, 1 full, 2 warp-split (test knob)
    bool prezeroed;            // scratch already zeroed by the caller's fill list (host side only)
};

template <typename K, int VB>
struct BnlTile {
    static constexpr int VSZ = VB;
    // elements per stage, a multiple of 16 so every array stays 16-B aligned
    static constexpr int TILE = (B_STAGE_BYTES / (int)(sizeof(K) + VSZ)) & ~15;
    static constexpr int KBYTES = TILE * (int)sizeof(K);
};

template <int AGG>
struct AccKind {
    static constexpr bool minmax = AGG == MIN || AGG == MAX;
    static constexpr bool sum = AGG == SUM || AGG == AVG;
    static constexpr bool count = AGG == COUNT;
    static constexpr bool exists = AGG == EXISTS || AGG == NOT_EXISTS;
};

// PTX spelling of the correlated operator (r.key OP s.key, reading R8).
template <int OP>
struct OpName;
template <> struct OpName<EQ> { static constexpr const char *s = "eq"; };
template <> struct OpName<NE> { static constexpr const char *s = "ne"; };
template <> struct OpName<LT> { static constexpr const char *s = "lt"; };
template <> struct OpName<LE> { static constexpr const char *s = "le"; };
template <> struct OpName<GT> { static constexpr const char *s = "gt"; };
template <> struct OpName<GE> { static constexpr const char *s = "ge"; };

#define NG_SETP_U32(OPS) "setp." OPS ".u32 p, %1, %2;"
#define NG_SETP_U64(OPS) "setp." OPS ".u64 p, %1, %2;"
#define NG_SETP2_U32(OPS) "setp." OPS ".u32 p, %2, %3;"
#define NG_SETP2_U64(OPS) "setp." OPS ".u64 p, %2, %3;"

// The multiplier of every predicated accumulate below: a 1 in the constant
// bank, so ptxas can neither fold the IMAD into an ALU add nor needs a GPR
// for it (IMAD slot B takes the constant-bank / uniform operand).
static __constant__ unsigned ng_cnt_one = 1u;

// c += (r OP s): one ISETP on the ALU pipe + one predicated IMAD on the FMA
// pipe -- the two pipes split the pair's work evenly.  The IMAD is
// c = c * cb_one + one: the addend `one` (a runtime 1 in a GPR) sits in slot
// C, whose reuse cache the interleaved ISETPs (slots A, B) leave intact, so
// each IMAD reads a single GPR -- the accumulator.  With `one` in slots B and
// C, the accumulator and `one` (same register bank) conflicted on every IMAD:
// ncu "dispatch stall" 1.1 per issue, COUNT at 0.79 of the two-pipe bound;
// now 0.95 (C2 '>' COUNT 68.0 -> 56.3 ms).
template <int OP, typename K>
__device__ __forceinline__ void count_if(const K rk, const K sk, unsigned &c, const unsigned one)
{
#define NG_CNT(OPS)                                                                                  \
    if constexpr (sizeof(K) == 4)                                                                     \
        asm("{.reg .pred p;\n\t" NG_SETP_U32(OPS) "\n\t@p mad.lo.u32 %0, %0, %4, %3;}"                \
            : "+r"(c) : "r"((uint32_t)rk), "r"((uint32_t)sk), "r"(one), "r"(ng_cnt_one));             \
    else                                                                                              \
        asm("{.reg .pred p;\n\t" NG_SETP_U64(OPS) "\n\t@p mad.lo.u32 %0, %0, %4, %3;}"                \
            : "+r"(c) : "l"((uint64_t)rk), "l"((uint64_t)sk), "r"(one), "r"(ng_cnt_one));
    if constexpr (OP == EQ) { NG_CNT("eq") } else if constexpr (OP == NE) { NG_CNT("ne") }
    else if constexpr (OP == LT) { NG_CNT("lt") } else if constexpr (OP == LE) { NG_CNT("le") }
    else if constexpr (OP == GT) { NG_CNT("gt") } else { NG_CNT("ge") }
#undef NG_CNT
}

// c += (r OP s); sum += (r OP s) ? v : 0 -- ISETP + predicated IMAD (count)
// + predicated IMAD.WIDE (sum = v*one + sum, 32-bit payload) on the FMA pipe;
// 64-bit payloads add on the ALU pipe.
#define NG_SUM_BODY(SETP, KCON, VADD, VCON)                                                           \
    asm("{.reg .pred p;\n\t" SETP "\n\t@p mad.lo.u32 %0, %0, %6, %4;\n\t" VADD "}"                    \
        : "+r"(c), "+l"(sm) : KCON((rk)), KCON((sk)), "r"(one), VCON(v), "r"(ng_cnt_one));
#define NG_ADD32 "@p mad.wide.s32 %1, %5, %6, %1;"
#define NG_K32(x) "r"((uint32_t)x)
#define NG_K64(x) "l"((uint64_t)x)
#define NG_V32(x) "r"((int)x)
#define NG_V64(x) "l"((long long)x)
#define NG_ADD64 "@p add.s64 %1, %1, %5;"
#define NG_SUM_OP(OPS)                                                                                \
    if constexpr (sizeof(K) == 4 && sizeof(V) == 4) { NG_SUM_BODY(NG_SETP2_U32(OPS), NG_K32, NG_ADD32, NG_V32) } \
    else if constexpr (sizeof(K) == 4) { NG_SUM_BODY(NG_SETP2_U32(OPS), NG_K32, NG_ADD64, NG_V64) }  \
    else if constexpr (sizeof(V) == 4) { NG_SUM_BODY(NG_SETP2_U64(OPS), NG_K64, NG_ADD32, NG_V32) }  \
    else { NG_SUM_BODY(NG_SETP2_U64(OPS), NG_K64, NG_ADD64, NG_V64) }
template <int OP, typename K, typename V>
__device__ __forceinline__ void sum_if(const K rk, const K sk, const V v, long long &sm, unsigned &c,
                                       const unsigned one)
{
    if constexpr (OP == EQ) { NG_SUM_OP("eq") } else if constexpr (OP == NE) { NG_SUM_OP("ne") }
    else if constexpr (OP == LT) { NG_SUM_OP("lt") } else if constexpr (OP == LE) { NG_SUM_OP("le") }
    else if constexpr (OP == GT) { NG_SUM_OP("gt") } else { NG_SUM_OP("ge") }
}
#undef NG_SUM_OP
#undef NG_ADD64
#undef NG_ADD32
#undef NG_V64
#undef NG_V32
#undef NG_K64
#undef NG_K32
#undef NG_SUM_BODY

// c += (r OP s); s32 += (r OP s) ? v : 0 -- ISETP + two predicated IMADs
// (FMA pipe); s32 is a per-tile partial sum that cannot overflow (checked).
#define NG_S32_BODY(SETP, KCON)                                                                       \
    asm("{.reg .pred p;\n\t" SETP "\n\t@p mad.lo.u32 %0, %0, %6, %4;\n\t"                            \
        "@p mad.lo.s32 %1, %5, %6, %1;}"                                                              \
        : "+r"(c), "+r"(s32) : KCON((rk)), KCON((sk)), "r"(one), "r"((int)v), "r"(ng_cnt_one));
#define NG_K32(x) "r"((uint32_t)x)
#define NG_K64(x) "l"((uint64_t)x)
#define NG_S32_OP(OPS)                                                                                \
    if constexpr (sizeof(K) == 4) { NG_S32_BODY(NG_SETP2_U32(OPS), NG_K32) }                          \
    else { NG_S32_BODY(NG_SETP2_U64(OPS), NG_K64) }
template <int OP, typename K, typename V>
__device__ __forceinline__ void sum32_if(const K rk, const K sk, const V v, V &s32, unsigned &c, const unsigned one)
{
    if constexpr (OP == EQ) { NG_S32_OP("eq") } else if constexpr (OP == NE) { NG_S32_OP("ne") }
    else if constexpr (OP == LT) { NG_S32_OP("lt") } else if constexpr (OP == LE) { NG_S32_OP("le") }
    else if constexpr (OP == GT) { NG_S32_OP("gt") } else { NG_S32_OP("ge") }
}
#undef NG_S32_OP
#undef NG_K64
#undef NG_K32
#undef NG_S32_BODY

// One (r, s) pair: the whole nested-method inner step.
//   MIN/MAX: ISETP + predicated IMNMX (both ALU pipe); with TRACK also
//            "found" (only when some payload equals the MIN/MAX identity).
//   COUNT:   ISETP (ALU) + predicated IMAD (FMA).
//   SUM/AVG: ISETP (ALU) + predicated IMAD + IMAD.WIDE (FMA).  With TRACK
//            and 64-bit payloads ("wide": |S'| * max|payload| may reach
//            2^63): the payload's low 32-bit half (unsigned) goes to sm and
//            its high half (signed) to mm; neither sum can overflow int64
//            (|S'| < 2^31), finalize recombines them exactly (reading R5).
//   EXISTS:  predicate OR.
template <int OP, int AGG, bool TRACK, typename K, typename V>
__device__ __forceinline__ void pair_step(const K rk, const K sk, const V sv, V &mm, long long &sm, unsigned &c,
                                          bool &found, const unsigned one)
{
    if constexpr (AccKind<AGG>::minmax) {
        const bool p = cmp_ct<OP>(rk, sk);
        if (p) mm = (AGG == MIN) ? min(mm, sv) : max(mm, sv);
        if constexpr (TRACK) found |= p;
    } else if constexpr (AccKind<AGG>::sum) {
        if constexpr (TRACK && sizeof(V) == 4) {
            sum32_if<OP>(rk, sk, sv, mm, c, one);
        } else if constexpr (TRACK) {
            if (cmp_ct<OP>(rk, sk)) {
                c += 1u;
                sm += (long long)(unsigned long long)(unsigned)sv;
                mm += sv >> 32;
            }
        } else {
            sum_if<OP>(rk, sk, sv, sm, c, one);
        }
    } else if constexpr (AccKind<AGG>::count) {
        count_if<OP>(rk, sk, c, one);
    } else {
        found |= cmp_ct<OP>(rk, sk);
    }
}

// SPLIT: the CTA's 8 warps hold the SAME outer tuples and each warp scans
// every 8th group of the tile (small-R' mode); otherwise every warp scans the
// whole tile for its own tuples.
template <int RPT, bool SPLIT, int OP, int AGG, bool TRACK, typename K, typename V, int VB>
__device__ __forceinline__ void tile_full(const K *__restrict__ tk, const V *__restrict__ tv, const K (&rk)[RPT],
                                          V (&mm)[RPT], long long (&sm)[RPT], unsigned (&c)[RPT],
                                          bool (&found)[RPT], const unsigned mul)
{
    constexpr int TILE = BnlTile<K, VB>::TILE;
    constexpr int KV = 16 / (int)sizeof(K);  // keys per 128-bit load
    constexpr int STEP = SPLIT ? KV * (B_THREADS / 32) : KV;
    // U groups of KV elements per iteration, all loaded up front (no
    // cross-iteration software pipelining: ptxas would add register moves)
    // (MIN/MAX or 64-bit keys: 2 groups -- MIN stays at 3 CTAs/SM; COUNT /
    // EXISTS / SUM with 32-bit keys: 4, measured fastest)
    constexpr int U = (AccKind<AGG>::minmax || sizeof(K) == 8) ? NG_B_UNROLL : NG_B_UNROLL_V0;
    const int e0 = SPLIT ? (int)(threadIdx.x >> 5) * KV : 0;
#pragma unroll 1
    for (int e = e0; e < TILE; e += STEP * U) {
        K kk[U][KV];
        V vv[U][KV];
#pragma unroll
        for (int u = 0; u < U; u++) {
            // clamped when whole iterations do not tile TILE: the ragged tail is skipped below
            const int eu = (TILE % (STEP * U)) == 0 ? e + u * STEP : min(e + u * STEP, TILE - KV);
            if constexpr (sizeof(K) == 4) {
                const uint4 q = *reinterpret_cast<const uint4 *>(tk + eu);
                kk[u][0] = q.x; kk[u][1] = q.y; kk[u][2] = q.z; kk[u][3] = q.w;
            } else {
                const ulonglong2 q = *reinterpret_cast<const ulonglong2 *>(tk + eu);
                kk[u][0] = q.x; kk[u][1] = q.y;
            }
            if constexpr (VB == 4) {
                if constexpr (KV == 4) {
                    const int4 q = *reinterpret_cast<const int4 *>(tv + eu);
                    vv[u][0] = q.x; vv[u][1] = q.y; vv[u][2] = q.z; vv[u][3] = q.w;
                } else {
                    const int2 q = *reinterpret_cast<const int2 *>(tv + eu);
                    vv[u][0] = q.x; vv[u][1] = q.y;
                }
            } else if constexpr (VB == 8) {
#pragma unroll
                for (int q = 0; q < KV; q += 2) {
                    const longlong2 w = *reinterpret_cast<const longlong2 *>(tv + eu + q);
                    vv[u][q] = w.x; vv[u][q + 1] = w.y;
                }
            } else {
#pragma unroll
                for (int q = 0; q < KV; q++) vv[u][q] = 0;
            }
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            // whole iterations cover the tile unless TILE / KV is not a
            // multiple of the per-iteration stride (uniform per warp)
            if ((TILE % (STEP * U)) != 0 && e + u * STEP >= TILE) break;
#pragma unroll
            for (int q = 0; q < KV; q++) {
#pragma unroll
                for (int i = 0; i < RPT; i++)
                    pair_step<OP, AGG, TRACK>(rk[i], kk[u][q], vv[u][q], mm[i], sm[i], c[i], found[i], mul);
            }
        }
    }
}

template <int RPT, bool SPLIT, int OP, int AGG, bool TRACK, typename K, typename V, int VB>
__device__ __forceinline__ void tile_part(const K *__restrict__ tk, const V *__restrict__ tv, int count,
                                          const K (&rk)[RPT], V (&mm)[RPT], long long (&sm)[RPT],
                                          unsigned (&c)[RPT], bool (&found)[RPT], const unsigned mul)
{
    for (int e = SPLIT ? (int)(threadIdx.x >> 5) : 0; e < count; e += SPLIT ? B_THREADS / 32 : 1) {
        const K k = tk[e];
        const V v = VB ? tv[e] : (V)0;
#pragma unroll
        for (int i = 0; i < RPT; i++) pair_step<OP, AGG, TRACK>(rk[i], k, v, mm[i], sm[i], c[i], found[i], mul);
    }
}

// The whole loop: RPT outer tuples per thread; R blocks of B_THREADS * RPT
// tuples (every warp its own tuples), or with SPLIT of 32 * RPT tuples held
// by all 8 warps, each scanning 1/8 of every S' tile -- 8x more R blocks for
// an |R'| so small that full blocks would leave CTAs idle (Q2 / Q5 / cached
// Q17 have a few hundred R' tuples).  Same ILP and registers either way.
template <int RPT, bool SPLIT, typename K, int VB, int OP, int AGG>
__device__ __forceinline__ void bnl_body(const BnlArgs &A, unsigned char *smem, unsigned long long *full_bar,
                                         long long &s_unit, const long long nrp, const long long nsp)
{
    using V = typename std::conditional<VB == 8, long long, int>::type;
    constexpr int TILE = BnlTile<K, VB>::TILE;
    constexpr int KBYTES = BnlTile<K, VB>::KBYTES;
    constexpr V VMAX = VB == 8 ? (V)LLONG_MAX : (V)INT_MAX;
    constexpr V VMIN = VB == 8 ? (V)LLONG_MIN : (V)INT_MIN;
    constexpr V MM0 = AGG == MIN ? VMAX : (AGG == MAX ? VMIN : (V)0);
    constexpr long long RSTRIDE = SPLIT ? 32 : B_THREADS;   // tuple stride within a block
    constexpr long long RBLOCK = RSTRIDE * RPT;
    static_assert(!SPLIT || RBLOCK * 28 <= (long long)B_STAGES * B_STAGE_BYTES, "split merge area");
    const int tid = threadIdx.x;
    const int rlane = SPLIT ? (tid & 31) : tid;

    // Work decomposition from the ACTUAL |R'| and |S'| (device counts; the
    // host only knows upper bounds): (R block) x (S' chunk of whole tiles)
    // units, about target_units of them, chunks down to a single tile so a
    // small R' (few R blocks) still spreads over every CTA.
    const long long n_rb = (nrp + RBLOCK - 1) / RBLOCK;
    const long long n_ts = (nsp + TILE - 1) / TILE;
    long long n_sc = n_rb > 0 ? (A.target_units + n_rb - 1) / n_rb : 1;
    // chunks of at least one tile; in the warp-split shape at least 4 tiles, so
    // the TMA fill latency and the per-unit merge amortise over a unit
    const long long max_sc = SPLIT ? (n_ts + 3) / 4 : n_ts;
    n_sc = n_sc < 1 ? 1 : (n_sc > max_sc ? max_sc : n_sc);
    const long long chunk_tiles = n_sc > 0 ? (n_ts + n_sc - 1) / n_sc : 1;
    const long long chunk = chunk_tiles * TILE;
    n_sc = chunk_tiles > 0 ? (n_ts + chunk_tiles - 1) / chunk_tiles : 0;
    const long long n_units = n_rb * n_sc;
    // MIN/MAX: if some S' payload equals the identity, track "found"
    // explicitly (uniform per launch, flag from the S' filter kernel).
    // SUM/AVG with 32-bit payloads: when max|payload| * TILE < 2^31 a tile's
    // partial sum fits int32 -> "ALT" path accumulates it with a predicated
    // 32-bit IMAD (FMA pipe) and widens once per tile.
    bool track = false;
    if constexpr (AccKind<AGG>::minmax) track = A.extreme[AGG == MIN ? 0 : 1] != 0;
    if constexpr (AccKind<AGG>::sum && VB == 4)
        track = *(const unsigned long long *)(A.extreme + 2) < (0x80000000ull / (unsigned long long)TILE);
    if constexpr (AccKind<AGG>::sum && VB == 8) track = A.acc_hi != nullptr;   // exact split sums
    const unsigned mul = A.one;
    const K *rkeys = (const K *)A.rkeys;
    const K *skeys = (const K *)A.skeys;
    const V *svals = (const V *)A.svals;
    unsigned g = 0;  // tiles consumed by this CTA so far (ring position / phase)

    auto issue = [&](long long tile_start, long long s1, unsigned stage) {
        const int cnt = (int)min((long long)TILE, s1 - tile_start);
        const unsigned kb = ((unsigned)cnt * (unsigned)sizeof(K) + 15u) & ~15u;
        const unsigned vb = VB ? (((unsigned)cnt * (unsigned)VB + 15u) & ~15u) : 0u;
        unsigned char *base = smem + stage * B_STAGE_BYTES;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_expect_tx(&full_bar[stage], kb + vb);
        bulk_g2s(base, skeys + tile_start, kb, &full_bar[stage]);
        if (VB) bulk_g2s(base + KBYTES, (const char *)svals + tile_start * VB, vb, &full_bar[stage]);
    };

    while (true) {
        if (tid == 0) s_unit = (long long)atomicAdd(A.unit_counter, 1u);
        __syncthreads();
        const long long u = s_unit;
        __syncthreads();
        if (u >= n_units) break;
        const long long sc = u / n_rb, rb = u - sc * n_rb;
        const long long s0 = sc * chunk;
        const long long s1 = min(nsp, s0 + chunk);
        const int ntiles = s1 > s0 ? (int)((s1 - s0 + TILE - 1) / TILE) : 0;
        if (ntiles == 0) continue;
        if constexpr (AccKind<AGG>::exists) {
            // semi-join early exit across units: another S' chunk already
            // satisfied every tuple of this R block (flag read by one thread,
            // decision made uniform through the barrier)
            if (__syncthreads_or(tid == 0 && ld_relaxed_u32(A.rb_done + rb) != 0)) continue;
        }

        K rk[RPT];
        V mm[RPT];
        long long sm[RPT];
        unsigned c[RPT];
        bool found[RPT];
        const long long r0 = rb * RBLOCK + rlane;
#pragma unroll
        for (int i = 0; i < RPT; i++) {
            const long long r = r0 + (long long)i * RSTRIDE;
            rk[i] = r < nrp ? rkeys[r] : (K)0;
            mm[i] = MM0;
            sm[i] = 0;
            c[i] = 0;
            found[i] = false;
        }
        int issued = min(ntiles, B_STAGES);
        if (tid == 0)
            for (int t = 0; t < issued; t++) issue(s0 + (long long)t * TILE, s1, (g + t) % B_STAGES);
        bool stop = false;
        for (int t = 0; t < issued; t++) {
            const unsigned stage = g % B_STAGES;
            mbar_wait(&full_bar[stage], (g / B_STAGES) & 1u);
            if (!stop) {
                const unsigned char *base = smem + stage * B_STAGE_BYTES;
                const K *tk = (const K *)base;
                const V *tv = (const V *)(base + KBYTES);
                const long long ts = s0 + (long long)t * TILE;
                const int cnt = (int)min((long long)TILE, s1 - ts);
                if (cnt == TILE) {
                    if (track) tile_full<RPT, SPLIT, OP, AGG, true, K, V, VB>(tk, tv, rk, mm, sm, c, found, mul);
                    else tile_full<RPT, SPLIT, OP, AGG, false, K, V, VB>(tk, tv, rk, mm, sm, c, found, mul);
                } else {
                    if (track) tile_part<RPT, SPLIT, OP, AGG, true, K, V, VB>(tk, tv, cnt, rk, mm, sm, c, found, mul);
                    else tile_part<RPT, SPLIT, OP, AGG, false, K, V, VB>(tk, tv, cnt, rk, mm, sm, c, found, mul);
                }
            }
            ++g;
            if constexpr (AccKind<AGG>::sum && VB == 4) {
                if (track) {  // widen the per-tile 32-bit partial sums
#pragma unroll
                    for (int i = 0; i < RPT; i++) {
                        sm[i] += (long long)mm[i];
                        mm[i] = 0;
                    }
                }
            }
            if constexpr (AccKind<AGG>::exists) {
                bool all = true;
#pragma unroll
                // (SPLIT: a warp only saw 1/8 of the tile, so this stops only
                // once every warp found a match for every tuple -- later than
                // necessary, never too early)
                for (int i = 0; i < RPT; i++) all = all && (found[i] || r0 + (long long)i * RSTRIDE >= nrp);
                stop = __syncthreads_and(all) != 0;
                if (stop && tid == 0) st_relaxed_u32(A.rb_done + rb, 1u);
            } else {
                __syncthreads();
            }
            if (!stop && t + B_STAGES < ntiles) {
                if (tid == 0) issue(s0 + (long long)(t + B_STAGES) * TILE, s1, stage);
                issued = t + B_STAGES + 1;
            }
        }
        // merge this unit's partial aggregates
        if constexpr (SPLIT) {
            // the 8 warps hold partials of the SAME 256 tuples: combine them
            // in shared memory (the ring is idle: every issued tile has been
            // consumed), then one global atomic per tuple instead of eight
            long long *s_acc = (long long *)smem;
            unsigned long long *s_cnt = (unsigned long long *)(smem + RBLOCK * 8);
            int *s_found = (int *)(smem + RBLOCK * 16);
            long long *s_hi = (long long *)(smem + RBLOCK * 20);   // split SUM high halves
            for (int t = tid; t < RBLOCK; t += B_THREADS) {
                s_acc[t] = AccKind<AGG>::minmax ? (long long)MM0 : 0;
                s_cnt[t] = 0;
                s_found[t] = 0;
                s_hi[t] = 0;
            }
            __syncthreads();
#pragma unroll
            for (int i = 0; i < RPT; i++) {
                const int t = rlane + i * (int)RSTRIDE;
                if (r0 + (long long)i * RSTRIDE >= nrp) continue;
                if constexpr (AccKind<AGG>::minmax) {
                    if (track ? found[i] : (mm[i] != MM0)) {
                        if (AGG == MIN) atomicMin(&s_acc[t], (long long)mm[i]);
                        else atomicMax(&s_acc[t], (long long)mm[i]);
                        s_found[t] = 1;
                    }
                } else if constexpr (AccKind<AGG>::sum) {
                    if (c[i]) {
                        atomicAdd((unsigned long long *)&s_acc[t], (unsigned long long)sm[i]);
                        atomicAdd(&s_cnt[t], (unsigned long long)c[i]);
                        if (VB == 8 && track) atomicAdd((unsigned long long *)&s_hi[t], (unsigned long long)mm[i]);
                    }
                } else if constexpr (AccKind<AGG>::count) {
                    if (c[i]) atomicAdd(&s_cnt[t], (unsigned long long)c[i]);
                } else {
                    if (found[i]) s_found[t] = 1;
                }
            }
            __syncthreads();
            for (int t = tid; t < RBLOCK; t += B_THREADS) {
                const long long r = rb * RBLOCK + t;
                if (r >= nrp) continue;
                if constexpr (AccKind<AGG>::minmax) {
                    if (s_found[t]) {
                        if (AGG == MIN) atomicMin(&A.acc[r], s_acc[t]);
                        else atomicMax(&A.acc[r], s_acc[t]);
                        A.cnt[r] = 1;
                    }
                } else if constexpr (AccKind<AGG>::sum) {
                    if (s_cnt[t]) {
                        atomicAdd((unsigned long long *)&A.acc[r], (unsigned long long)s_acc[t]);
                        atomicAdd((unsigned long long *)&A.cnt[r], s_cnt[t]);
                        if (VB == 8 && track) atomicAdd((unsigned long long *)&A.acc_hi[r], (unsigned long long)s_hi[t]);
                    }
                } else if constexpr (AccKind<AGG>::count) {
                    if (s_cnt[t]) atomicAdd((unsigned long long *)&A.cnt[r], s_cnt[t]);
                } else {
                    if (s_found[t]) A.cnt[r] = 1;
                }
            }
            __syncthreads();   // the ring is refilled by the next unit
        } else {
#pragma unroll
            for (int i = 0; i < RPT; i++) {
                const long long r = r0 + (long long)i * RSTRIDE;
                if (r >= nrp) continue;
                if constexpr (AccKind<AGG>::minmax) {
                    const bool f = track ? found[i] : (mm[i] != MM0);
                    if (f) {
                        if (AGG == MIN) atomicMin(&A.acc[r], (long long)mm[i]);
                        else atomicMax(&A.acc[r], (long long)mm[i]);
                        A.cnt[r] = 1;
                    }
                } else if constexpr (AccKind<AGG>::sum) {
                    if (c[i]) {
                        atomicAdd((unsigned long long *)&A.acc[r], (unsigned long long)sm[i]);
                        atomicAdd((unsigned long long *)&A.cnt[r], (unsigned long long)c[i]);
                        if (VB == 8 && track) atomicAdd((unsigned long long *)&A.acc_hi[r], (unsigned long long)mm[i]);
                    }
                } else if constexpr (AccKind<AGG>::count) {
                    if (c[i]) atomicAdd((unsigned long long *)&A.cnt[r], (unsigned long long)c[i]);
                } else {
                    if (found[i]) A.cnt[r] = 1;
                }
            }
        }
    }
}

template <typename K, int VB, int OP, int AGG>
__global__ void __launch_bounds__(B_THREADS, 2) bnl_kernel(BnlArgs A)
{
    constexpr int TILE = BnlTile<K, VB>::TILE;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ __align__(8) unsigned long long full_bar[B_STAGES];
    __shared__ long long s_unit;
    if (threadIdx.x == 0) {
        for (int s = 0; s < B_STAGES; s++) mbar_init(&full_bar[s], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const long long nrp = *A.d_nrp, nsp = *A.d_nsp;
    // Uniform choice of the R-block shape.  Full blocks (2048 tuples) unless
    // they (a) leave fewer than two (R block x S' tile) units per CTA, or (b)
    // pad |R'| by more than 20 % over the warp-split blocks (256 tuples): the
    // padded tuple slots are compared against every S' element like real
    // ones (SF1 Q17 cached: 210 tuples in a 2048-slot block).
    constexpr long long FULL = (long long)B_THREADS * B_RPT, SPL = 32LL * B_RPT;
    const long long n_rb_full = (nrp + FULL - 1) / FULL;
    const long long units_big = n_rb_full * ((nsp + TILE - 1) / TILE);
    const long long slots_full = n_rb_full * FULL, slots_split = (nrp + SPL - 1) / SPL * SPL;
    const bool split = A.shape ? A.shape == 2 : (units_big < 2LL * gridDim.x || 5 * slots_full > 6 * slots_split);
    if (split)
        bnl_body<B_RPT, true, K, VB, OP, AGG>(A, smem, full_bar, s_unit, nrp, nsp);
    else
        bnl_body<B_RPT, false, K, VB, OP, AGG>(A, smem, full_bar, s_unit, nrp, nsp);
}

// Host-side launchers, one per (key width, payload width) family, each in
// its own translation unit (k_bnl_<key>_v<payload>.cu).
#define NG_BNL_FAMILY_DECL(name) \
    cudaError_t name(int op, int agg, const BnlArgs &a, long long n_rp_max, long long ns_max, void *scratch, \
                     int num_sms, cudaStream_t st)
NG_BNL_FAMILY_DECL(bnl_family_u32_v0);
NG_BNL_FAMILY_DECL(bnl_family_u32_v4);
NG_BNL_FAMILY_DECL(bnl_family_u32_v8);
NG_BNL_FAMILY_DECL(bnl_family_u64_v0);
NG_BNL_FAMILY_DECL(bnl_family_u64_v4);
NG_BNL_FAMILY_DECL(bnl_family_u64_v8);

}  // namespace ng
