// k_filter.cu -- a2 / a3: local predicates over R (outer) or S (inner), and
// compaction of the surviving rows into R' (row ids + encoded keys) or
// S' (encoded keys + payload).
//
// PAPER.md P:235 (§III-C): a Selection is "scan -> 0-1 vector -> prefix-sum ->
// materialize" over several primitive kernels with inter-kernel results in a
// memory pool.  On B200 it is ONE pass:
//  * persistent CTAs take 256*ITEMS-row tiles from an atomic counter;
//  * every column segment the tile needs (predicate operands, validity
//    bytes, key, payload) is staged global -> shared by cp.async.bulk (TMA
//    bulk engine) into a double-buffered stage, completed on an mbarrier --
//    the next tile's copies are in flight while this tile is compacted;
//  * predicates are evaluated from shared memory (conflict-free), the 0-1
//    vector lives in a register bitmask, warp ballots + popc give ranks;
//  * the tile's output offset: S' (re-ordered by the sort anyway, order-free
//    for the nested loop) claims its range with one atomicAdd -- no
//    dependency between tiles; R' (whose order is the result's order) is
//    written in row order by two passes -- a count-only pass over just the
//    predicate columns, an exclusive scan of the tile counts, then the
//    writing pass at known offsets (a decoupled look-back chain across
//    thousands of tiles measured 3x slower at TPC-H SF10).
// The S' pass also reduces AND / OR over the encoded keys (radix digits on
// which all keys agree need no sort pass) and flags payloads equal to the
// MIN/MAX identity.
#include <climits>
#include <cstdlib>
#include <cstring>
#include <type_traits>

#include "internal.h"
#include "scan.cuh"

namespace ng {

#ifndef NG_RP_BATCH
#define NG_RP_BATCH 4   // ordered R' filter, phase 2: rounds of key loads in flight per warp
#endif
constexpr int RP_BATCH = NG_RP_BATCH;
#ifndef NG_RP_ITEMS
#define NG_RP_ITEMS 8   // ordered R' filter: rows per thread per staged tile
#endif
constexpr int T_THREADS = 256;
// scratch of the ordered one-launch R' filter: [0, 1024) the barrier word
// (zeroed), then the per-chunk counts, then the ballot words (n / 8 bytes)
constexpr size_t RP_COUNTS_OFF = 1024;
constexpr size_t RP_BITS_OFF = 1024 + 16384;
constexpr int T_WARPS = T_THREADS / 32;
constexpr int MAX_SRC = 40;
constexpr int STAGE_MAX = 49152;  // bytes per stage (2 stages per CTA)

struct SrcCols {
    int n;
    int stage_bytes;
    const void *ptr[MAX_SRC];
    int w[MAX_SRC];    // 1, 4 or 8 bytes per row
    int off[MAX_SRC];  // byte offset of the column's segment inside a stage
};

// A column segment inside a stage: byte offset and width (1, 4, 8);
// off < 0 = absent.  Resolved on the host so the kernel never indexes the
// source table (nor takes a kernel parameter's address) in its item loops.
struct Col {
    int off, w;
};

struct TPred {
    Col x, xv, y, yv;  // operand, its validity, rhs column (y.off < 0: literal), its validity
    int op;
    long long lit;
};

struct TPlan {
    int n_preds;
    TPred p[MAX_PREDS];
    Col key0, key0v, key1, key1v, val, valv;
    int n_key;
    int drop_null_key, drop_null_val;
};

__device__ __forceinline__ long long ld_col(const unsigned char *sb, const Col c, int li)
{
    const unsigned char *a = sb + c.off;
    return c.w == 4 ? (long long)reinterpret_cast<const int *>(a)[li]
                    : (c.w == 8 ? reinterpret_cast<const long long *>(a)[li] : (long long)a[li]);
}

template <int ITEMS>
__device__ __forceinline__ void load_items(const unsigned char *sb, const Col c, int tid, long long (&x)[ITEMS])
{
    const unsigned char *a = sb + c.off;
    if (c.w == 4) {
#pragma unroll
        for (int j = 0; j < ITEMS; j++) x[j] = reinterpret_cast<const int *>(a)[j * T_THREADS + tid];
    } else if (c.w == 8) {
#pragma unroll
        for (int j = 0; j < ITEMS; j++) x[j] = reinterpret_cast<const long long *>(a)[j * T_THREADS + tid];
    } else {
#pragma unroll
        for (int j = 0; j < ITEMS; j++) x[j] = a[j * T_THREADS + tid];
    }
}

template <int ITEMS>
__device__ __forceinline__ unsigned nonnull(const unsigned char *sb, const Col c, unsigned live, int tid)
{
    if (c.off < 0) return live;
    unsigned out = 0;
#pragma unroll
    for (int j = 0; j < ITEMS; j++)
        if ((live >> j & 1u) && sb[c.off + j * T_THREADS + tid]) out |= 1u << j;
    return out;
}

// Encoded keys of a tile's items (column widths dispatched once):
// composite (two int32-storage columns, reading R9), one int32 column, or
// one int64 column (with KB == 4: the low word of its code -- the caller
// knows the high word is constant).
template <int KB, int ITEMS>
__device__ __forceinline__ void load_keys(const unsigned char *sb, const TPlan &tp, int tid,
                                          typename std::conditional<KB == 8, uint64_t, uint32_t>::type (&k)[ITEMS])
{
    using K = typename std::conditional<KB == 8, uint64_t, uint32_t>::type;
    if (tp.n_key == 2) {
        const int *a = reinterpret_cast<const int *>(sb + tp.key0.off);
        const int *b = reinterpret_cast<const int *>(sb + tp.key1.off);
#pragma unroll
        for (int j = 0; j < ITEMS; j++)
            k[j] = (K)(((uint64_t)enc32(a[j * T_THREADS + tid]) << 32) | enc32(b[j * T_THREADS + tid]));
    } else if (tp.key0.w == 4) {
        const int *a = reinterpret_cast<const int *>(sb + tp.key0.off);
#pragma unroll
        for (int j = 0; j < ITEMS; j++)
            k[j] = KB == 4 ? (K)enc32(a[j * T_THREADS + tid]) : (K)enc64((long long)a[j * T_THREADS + tid]);
    } else {
        const long long *a = reinterpret_cast<const long long *>(sb + tp.key0.off);
#pragma unroll
        for (int j = 0; j < ITEMS; j++) k[j] = (K)enc64(a[j * T_THREADS + tid]);
    }
}

template <int ITEMS, int OP, typename T>
__device__ __forceinline__ unsigned cmp_items(const T (&x)[ITEMS], const T (&y)[ITEMS])
{
    unsigned m = 0;
#pragma unroll
    for (int j = 0; j < ITEMS; j++)
        if (cmp_ct<OP>(x[j], y[j])) m |= 1u << j;
    return m;
}

// Output offset of a tile: tile_base[tile] if given (ordered pass 2), else
// an atomic claim on *out_count.  tile_count (pass 1): write the tile's
// survivor count and nothing else.
template <int KB, int VB, int ITEMS>
__global__ void __launch_bounds__(T_THREADS)
filter_tma_kernel(long long n, SrcCols sc, TPlan tp, int *__restrict__ out_ids, void *__restrict__ out_keys,
                  uint8_t *__restrict__ out_kvalid, void *__restrict__ out_vals,
                  unsigned long long *__restrict__ keymask, unsigned *__restrict__ extreme,
                  const unsigned long long *__restrict__ tile_base, unsigned *__restrict__ tile_count,
                  unsigned *__restrict__ counter, long long *__restrict__ out_count,
                  unsigned *__restrict__ live_bits, const unsigned long long *__restrict__ chunk_off)
{
    // live_bits (ordered two-pass mode): pass 1 (tile_count) writes each
    // (tile, item, warp)'s survivor ballot; pass 2 takes its survivors from
    // them instead of re-reading and re-evaluating the predicate columns
    using K = typename std::conditional<KB == 8, uint64_t, uint32_t>::type;
    using V = typename std::conditional<VB == 8, long long, int>::type;
    constexpr int TILE = T_THREADS * ITEMS;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ __align__(8) unsigned long long bar[2];
    __shared__ unsigned s_cnt[ITEMS][T_WARPS];
    __shared__ long long s_tile[2];
    __shared__ unsigned long long s_claim;

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const long long num_tiles = (n + TILE - 1) / TILE;

    auto issue = [&](long long tile, int stage) {
        const long long rows = min((long long)TILE, n - tile * TILE);
        unsigned total = 0;
        for (int c = 0; c < sc.n; c++) total += ((unsigned)rows * sc.w[c] + 15u) & ~15u;
        unsigned char *dst = smem + stage * sc.stage_bytes;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_expect_tx(&bar[stage], total);
        for (int c = 0; c < sc.n; c++)
            bulk_g2s(dst + sc.off[c], (const char *)sc.ptr[c] + tile * TILE * sc.w[c],
                     ((unsigned)rows * sc.w[c] + 15u) & ~15u, &bar[stage]);
    };

    if (tid == 0) {
        mbar_init(&bar[0], 1);
        mbar_init(&bar[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        const long long t0 = atomicAdd(counter, 1u);
        s_tile[0] = t0;
        if (t0 < num_tiles) issue(t0, 0);
    }
    __syncthreads();

    unsigned phase = 0u;  // bit s: parity of the next completion of stage s
    int stage = 0;
    bool ext_max = false, ext_min = false;
    unsigned long long vabs = 0;  // max |payload| over the survivors
    unsigned long long kand = ~0ull, kor = 0ull;
    while (true) {
        const long long tile = s_tile[stage];
        if (tile >= num_tiles) break;
        if (tid == 0) {  // prefetch the next tile into the other stage
            const long long nt = atomicAdd(counter, 1u);
            s_tile[stage ^ 1] = nt;
            if (nt < num_tiles) issue(nt, stage ^ 1);
        }
        mbar_wait(&bar[stage], (phase >> stage) & 1u);
        phase ^= 1u << stage;
        const long long base = tile * TILE;
        const long long rows = min((long long)TILE, n - base);

        unsigned live = 0;
        if (live_bits && !tile_count) {
#pragma unroll
            for (int j = 0; j < ITEMS; j++)
                live |= ((__ldcg(live_bits + (tile * ITEMS + j) * T_WARPS + warp) >> lane) & 1u) << j;
        } else {
#pragma unroll
            for (int j = 0; j < ITEMS; j++)
                if (j * T_THREADS + tid < rows) live |= 1u << j;
        }
        // local predicates (NULL operands are not TRUE, reading R2)
        const unsigned char *sb = smem + stage * sc.stage_bytes;
        for (int k = 0; k < tp.n_preds; k++) {
            const TPred p = tp.p[k];
            live = nonnull<ITEMS>(sb, p.xv, live, tid);
            live = nonnull<ITEMS>(sb, p.yv, live, tid);
#define NG_CMP_ALL(X, Y)                                                                              \
            switch (p.op) {                                                                           \
            case EQ: live &= cmp_items<ITEMS, EQ>(X, Y); break;                                       \
            case NE: live &= cmp_items<ITEMS, NE>(X, Y); break;                                       \
            case LT: live &= cmp_items<ITEMS, LT>(X, Y); break;                                       \
            case LE: live &= cmp_items<ITEMS, LE>(X, Y); break;                                       \
            case GT: live &= cmp_items<ITEMS, GT>(X, Y); break;                                       \
            default: live &= cmp_items<ITEMS, GE>(X, Y); break;                                       \
            }
            if (p.x.w == 4 && (p.y.off >= 0 ? p.y.w == 4 : p.lit == (long long)(int)p.lit)) {
                // int32 operands (the common case): 32-bit compares
                int x[ITEMS], y[ITEMS];
                const int *xa = reinterpret_cast<const int *>(sb + p.x.off);
#pragma unroll
                for (int j = 0; j < ITEMS; j++) x[j] = xa[j * T_THREADS + tid];
                if (p.y.off >= 0) {
                    const int *ya = reinterpret_cast<const int *>(sb + p.y.off);
#pragma unroll
                    for (int j = 0; j < ITEMS; j++) y[j] = ya[j * T_THREADS + tid];
                } else {
#pragma unroll
                    for (int j = 0; j < ITEMS; j++) y[j] = (int)p.lit;
                }
                NG_CMP_ALL(x, y)
            } else {
                long long x[ITEMS], y[ITEMS];
                load_items<ITEMS>(sb, p.x, tid, x);
                if (p.y.off >= 0) {
                    load_items<ITEMS>(sb, p.y, tid, y);
                } else {
#pragma unroll
                    for (int j = 0; j < ITEMS; j++) y[j] = p.lit;
                }
                NG_CMP_ALL(x, y)
            }
#undef NG_CMP_ALL
        }
        unsigned kvalid = live;
        if constexpr (KB > 0) {
            kvalid = nonnull<ITEMS>(sb, tp.key1v, nonnull<ITEMS>(sb, tp.key0v, live, tid), tid);
            if (tp.drop_null_key) live = kvalid;
        }
        if constexpr (VB > 0) {
            const unsigned vv = nonnull<ITEMS>(sb, tp.valv, live, tid);
            if (tp.drop_null_val) live = vv;
        }
        unsigned rank[ITEMS];
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const unsigned m = __ballot_sync(FULL, live >> j & 1u);
            if (lane == 0) {
                s_cnt[j][warp] = __popc(m);
                if (live_bits && tile_count) live_bits[(tile * ITEMS + j) * T_WARPS + warp] = m;
            }
            rank[j] = __popc(m & lanemask_lt());
        }
        __syncthreads();
        if (tid < 32) {  // exclusive scan of the (item, warp) counts; the tile's base
            unsigned *flat = &s_cnt[0][0];
            constexpr int E = ITEMS * T_WARPS, PER = (E + 31) / 32;
            unsigned c[PER], sum = 0;
#pragma unroll
            for (int q = 0; q < PER; q++) {
                c[q] = PER * lane + q < E ? flat[PER * lane + q] : 0u;
                sum += c[q];
            }
            unsigned incl = sum;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const unsigned t = __shfl_up_sync(FULL, incl, o);
                if (lane >= o) incl += t;
            }
            unsigned run = incl - sum;
#pragma unroll
            for (int q = 0; q < PER; q++) {
                if (PER * lane + q < E) flat[PER * lane + q] = run;
                run += c[q];
            }
            if (lane == 31) {
                if (tile_count) tile_count[tile] = incl;
                else if (tile_base) s_claim = tile_base[tile] + (chunk_off ? __ldcg(chunk_off + (tile >> 10)) : 0ull);
                else s_claim = incl ? atomicAdd((unsigned long long *)out_count, (unsigned long long)incl) : 0ull;
            }
        }
        __syncthreads();
        if (tile_count) {  // pass 1 of the ordered mode: counts only
            stage ^= 1;
            continue;
        }
        const unsigned long long tb = s_claim;
        // keys and payloads of the tile's items, loaded with the column
        // widths resolved ONCE per tile (uniform branches) -- per item only
        // the stores and the optional reductions remain
        K keys[ITEMS];
        if constexpr (KB > 0) load_keys<KB, ITEMS>(sb, tp, tid, keys);
        V vals[ITEMS];
        if constexpr (VB > 0) {
#pragma unroll
            for (int j = 0; j < ITEMS; j++) vals[j] = reinterpret_cast<const V *>(sb + tp.val.off)[j * T_THREADS + tid];
        }
        const bool want_ext = extreme != nullptr, want_mask = keymask != nullptr;
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            if (!(live >> j & 1u)) continue;
            const int li = j * T_THREADS + tid;
            const long long pos = (long long)tb + s_cnt[j][warp] + rank[j];
            if (out_ids) out_ids[pos] = (int)(base + li);
            if constexpr (KB > 0) {
                if (out_keys) ((K *)out_keys)[pos] = keys[j];
                if (out_kvalid) out_kvalid[pos] = (kvalid >> j) & 1u;
                if (want_mask) {
                    kand &= (unsigned long long)keys[j];
                    kor |= (unsigned long long)keys[j];
                }
            }
            if constexpr (VB > 0) {
                const V v = vals[j];
                if (out_vals) ((V *)out_vals)[pos] = v;
                if (want_ext) {
                    ext_max |= v == (VB == 8 ? (V)LLONG_MAX : (V)INT_MAX);
                    ext_min |= v == (VB == 8 ? (V)LLONG_MIN : (V)INT_MIN);
                    const unsigned long long a = v < 0 ? 0ull - (unsigned long long)(long long)v
                                                       : (unsigned long long)v;
                    vabs = a > vabs ? a : vabs;
                }
            }
        }
        __syncthreads();  // stage fully read before it is refilled; s_tile visible
        stage ^= 1;
    }
    if constexpr (KB > 0) {
        if (keymask) {  // bits shared by every survivor key
            const unsigned alo = __reduce_and_sync(FULL, (unsigned)kand);
            const unsigned ahi = __reduce_and_sync(FULL, (unsigned)(kand >> 32));
            const unsigned olo = __reduce_or_sync(FULL, (unsigned)kor);
            const unsigned ohi = __reduce_or_sync(FULL, (unsigned)(kor >> 32));
            if (lane == 0) {
                atomicAnd(&keymask[0], ((unsigned long long)ahi << 32) | alo);
                atomicOr(&keymask[1], ((unsigned long long)ohi << 32) | olo);
            }
        }
    }
    if constexpr (VB > 0) {
        if (extreme) {
            if (__any_sync(FULL, ext_max) && lane == 0) atomicOr(&extreme[0], 1u);
            if (__any_sync(FULL, ext_min) && lane == 0) atomicOr(&extreme[1], 1u);
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                const unsigned long long b = __shfl_xor_sync(FULL, vabs, o);
                vabs = b > vabs ? b : vabs;
            }
            if (lane == 0 && vabs) atomicMax((unsigned long long *)(extreme + 2), vabs);
        }
    }
}

// ------------------------------------------------------------------ ordered R'
// One launch, no chained look-back (P:235's scan -> 0-1 vector -> prefix sum
// -> materialize): a persistent cooperative grid, CTA c owns a contiguous
// chunk of rows.
//  phase 1: the chunk's predicate columns stream through a double-buffered
//           cp.async.bulk stage; the 0-1 vector is written as one 32-bit
//           ballot word per 32 consecutive rows (n / 8 bytes, L2-resident)
//           and the chunk's survivor count is published;
//  barrier: one grid-wide barrier (every CTA is resident: cooperative
//           launch), then each CTA sums the counts of the chunks before it;
//  phase 2: warps read 32 ballot words at a time, rank survivors with popc
//           and a warp scan, load the survivors' keys (+ validity) straight
//           from global memory and write ids / encoded keys / key-valid in
//           row order.
// The predicate columns are read once and the key column only where rows
// survive (a selective date window reads a fraction of it); with no outer
// predicate phase 1 and the barrier are skipped (every row survives, the
// chunk offset is its first row).  The round-1 count pass + scan + write
// pass read the predicate columns twice and staged every key; a decoupled
// look-back chain over the tiles measured slower than both.
#ifndef NG_RP_MINB
#define NG_RP_MINB 2   // ordered R' filter: CTAs per SM the register budget must allow (latency hiding)
#endif
template <int KB, int ITEMS>
__global__ void __launch_bounds__(T_THREADS, NG_RP_MINB)
filter_rp_kernel(long long n, long long chunk, SrcCols sc, TPlan tp, KeySrc ks, int *__restrict__ out_ids,
                 void *__restrict__ out_keys, uint8_t *__restrict__ out_kvalid,
                 unsigned long long *__restrict__ keymask, unsigned *__restrict__ bits,
                 unsigned long long *__restrict__ counts, unsigned *__restrict__ barrier,
                 long long *__restrict__ out_count)
{
    using K = typename std::conditional<KB == 8, uint64_t, uint32_t>::type;
    constexpr int TILE = T_THREADS * ITEMS;
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ __align__(8) unsigned long long bar[2];
    __shared__ unsigned long long s_red[T_WARPS];
    __shared__ unsigned s_wtot[T_WARPS];
    __shared__ unsigned long long s_base;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const long long c0 = blockIdx.x * chunk;
    const long long c1 = min(n, c0 + chunk);
    const bool preds = sc.n > 0;
    unsigned long long mycount = 0;

    if (preds) {
        // ---- phase 1: predicates -> ballot words, chunk count
        const long long ntile = c1 > c0 ? (c1 - c0 + TILE - 1) / TILE : 0;
        auto issue = [&](long long t, int stage) {
            const long long r0 = c0 + t * TILE;
            const long long rows = min((long long)TILE, c1 - r0);
            unsigned total = 0;
            for (int c = 0; c < sc.n; c++) total += ((unsigned)rows * sc.w[c] + 15u) & ~15u;
            unsigned char *dst = smem + stage * sc.stage_bytes;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            mbar_expect_tx(&bar[stage], total);
            for (int c = 0; c < sc.n; c++)
                bulk_g2s(dst + sc.off[c], (const char *)sc.ptr[c] + r0 * sc.w[c], ((unsigned)rows * sc.w[c] + 15u) & ~15u,
                         &bar[stage]);
        };
        if (tid == 0) {
            mbar_init(&bar[0], 1);
            mbar_init(&bar[1], 1);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
            if (ntile > 0) issue(0, 0);
        }
        __syncthreads();
        for (long long t = 0; t < ntile; t++) {
            const int stage = (int)(t & 1);
            if (tid == 0 && t + 1 < ntile) issue(t + 1, stage ^ 1);   // the next tile streams in meanwhile
            mbar_wait(&bar[stage], (unsigned)((t >> 1) & 1));
            const unsigned char *sb = smem + stage * sc.stage_bytes;
            const long long r0 = c0 + t * TILE;
            const long long rows = min((long long)TILE, c1 - r0);
            unsigned live = 0;
#pragma unroll
            for (int j = 0; j < ITEMS; j++)
                if (j * T_THREADS + tid < rows) live |= 1u << j;
            for (int k = 0; k < tp.n_preds; k++) {   // local predicates, NULL is not TRUE (R2)
                const TPred p = tp.p[k];
                live = nonnull<ITEMS>(sb, p.xv, live, tid);
                live = nonnull<ITEMS>(sb, p.yv, live, tid);
#define NG_CMP_ALL(X, Y)                                                                              \
                switch (p.op) {                                                                       \
                case EQ: live &= cmp_items<ITEMS, EQ>(X, Y); break;                                   \
                case NE: live &= cmp_items<ITEMS, NE>(X, Y); break;                                   \
                case LT: live &= cmp_items<ITEMS, LT>(X, Y); break;                                   \
                case LE: live &= cmp_items<ITEMS, LE>(X, Y); break;                                   \
                case GT: live &= cmp_items<ITEMS, GT>(X, Y); break;                                   \
                default: live &= cmp_items<ITEMS, GE>(X, Y); break;                                   \
                }
                if (p.x.w == 4 && (p.y.off >= 0 ? p.y.w == 4 : p.lit == (long long)(int)p.lit)) {
                    int x[ITEMS], y[ITEMS];
                    const int *xa = reinterpret_cast<const int *>(sb + p.x.off);
#pragma unroll
                    for (int j = 0; j < ITEMS; j++) x[j] = xa[j * T_THREADS + tid];
                    if (p.y.off >= 0) {
                        const int *ya = reinterpret_cast<const int *>(sb + p.y.off);
#pragma unroll
                        for (int j = 0; j < ITEMS; j++) y[j] = ya[j * T_THREADS + tid];
                    } else {
#pragma unroll
                        for (int j = 0; j < ITEMS; j++) y[j] = (int)p.lit;
                    }
                    NG_CMP_ALL(x, y)
                } else {
                    long long x[ITEMS], y[ITEMS];
                    load_items<ITEMS>(sb, p.x, tid, x);
                    if (p.y.off >= 0) {
                        load_items<ITEMS>(sb, p.y, tid, y);
                    } else {
#pragma unroll
                        for (int j = 0; j < ITEMS; j++) y[j] = p.lit;
                    }
                    NG_CMP_ALL(x, y)
                }
#undef NG_CMP_ALL
            }
            // row r0 + j*256 + warp*32 + lane -> bit lane of word (r0 + j*256)/32 + warp
#pragma unroll
            for (int j = 0; j < ITEMS; j++) {
                const unsigned m = __ballot_sync(FULL, live >> j & 1u);
                if (j * T_THREADS + warp * 32 < rows && lane == 0) {
                    bits[(r0 + j * T_THREADS) / 32 + warp] = m;
                    mycount += __popc(m);
                }
            }
            __syncthreads();   // the stage is refilled two tiles later
        }
        // chunk count -> counts[block]; grid barrier; this chunk's offset
        if (lane == 0) s_red[warp] = mycount;
        __syncthreads();
        if (tid == 0) {
            unsigned long long t = 0;
            for (int w = 0; w < T_WARPS; w++) t += s_red[w];
            st_relaxed_u64(counts + blockIdx.x, t);
            __threadfence();
            atomicAdd(barrier, 1u);
            while (ld_relaxed_u32(barrier) < gridDim.x) __nanosleep(64);
            __threadfence();
        }
        __syncthreads();
        unsigned long long pre = 0;
        for (int b = tid; b < (int)blockIdx.x; b += T_THREADS) pre += ld_relaxed_u64(counts + b);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) pre += __shfl_xor_sync(FULL, pre, o);
        if (lane == 0) s_red[warp] = pre;
        __syncthreads();
        if (tid == 0) {
            unsigned long long t = 0;
            for (int w = 0; w < T_WARPS; w++) t += s_red[w];
            s_base = t;
            if (blockIdx.x == gridDim.x - 1) {   // the grand total
                unsigned long long mine = ld_relaxed_u64(counts + blockIdx.x);
                *out_count = (long long)(t + mine);
            }
        }
        __syncthreads();
    } else {
        if (tid == 0) {
            s_base = (unsigned long long)min(c0, n);   // every row before the chunk survives
            if (blockIdx.x == gridDim.x - 1) *out_count = n;
        }
        __syncthreads();
    }

    // ---- phase 2: ballot words -> ordered ids / keys / key-valid
    unsigned long long run = s_base;
    unsigned long long kand = ~0ull, kor = 0ull;
    const long long w0 = c0 / 32, w1 = (c1 + 31) / 32;
    for (long long g = w0; g < w1; g += 32 * T_WARPS) {
        const long long wi = g + warp * 32 + lane;
        unsigned word = 0;
        if (wi < w1) {
            if (preds) {
                word = __ldcg(bits + wi);
            } else {
                const long long r = wi * 32;
                word = (c1 - r >= 32) ? FULL : ((1u << (unsigned)(c1 - r)) - 1u);
            }
        }
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
        for (int w = 0; w < T_WARPS; w++) {
            const unsigned t = s_wtot[w];
            woff += w < warp ? t : 0;
            btot += t;
        }
        const unsigned excl = incl - c;
        // survivors of the warp's 1024 rows, 32 at a time: lane j takes the
        // survivor of warp-local rank r = b + j, finds its word by a binary
        // search over the lanes' exclusive counts (shuffles) and its row by
        // the rank within the word (__fns) -- every lane loads a key whatever
        // the selectivity, RP_BATCH batches of loads in flight per warp
        const unsigned wtotal = __shfl_sync(FULL, incl, 31);
        for (unsigned b = 0; b < wtotal; b += 32 * RP_BATCH) {
            long long row[RP_BATCH];
            uint64_t raw[RP_BATCH];
            bool kvl[RP_BATCH];
#pragma unroll
            for (int q = 0; q < RP_BATCH; q++) {
                const unsigned r = b + q * 32 + lane;
                int w = 0;   // the last lane whose exclusive count is <= r
#pragma unroll
                for (int step = 16; step > 0; step >>= 1) {
                    const unsigned e = __shfl_sync(FULL, excl, w + step);
                    if (e <= r) w += step;
                }
                const unsigned ew = __shfl_sync(FULL, excl, w);
                const unsigned wv = __shfl_sync(FULL, word, w);
                row[q] = -1;
                raw[q] = 0;
                kvl[q] = true;
                if (r < wtotal) {
                    const int bit = (int)__fns(wv, 0, (int)(r - ew) + 1);
                    const long long rw = (g + warp * 32 + w) * 32 + bit;
                    row[q] = rw;
                    if (ks.n_key == 2)
                        raw[q] = ((uint64_t)(uint32_t)__ldg((const int *)ks.c0 + rw) << 32) |
                                 (uint32_t)__ldg((const int *)ks.c1 + rw);
                    else if (ks.w0 == 4)
                        raw[q] = (uint32_t)__ldg((const int *)ks.c0 + rw);
                    else
                        raw[q] = (uint64_t)__ldg((const long long *)ks.c0 + rw);
                    kvl[q] = !((ks.v0 && !__ldg(ks.v0 + rw)) || (ks.v1 && !__ldg(ks.v1 + rw)));
                }
            }
#pragma unroll
            for (int q = 0; q < RP_BATCH; q++) {
                if (row[q] < 0) continue;
                const long long pos = (long long)run + woff + b + q * 32 + lane;
                K key;
                if (ks.n_key == 2)
                    key = (K)(((uint64_t)enc32((int)(uint32_t)(raw[q] >> 32)) << 32) | enc32((int)(uint32_t)raw[q]));
                else if (ks.w0 == 4)
                    key = KB == 4 ? (K)enc32((int)(uint32_t)raw[q]) : (K)enc64((long long)(int)(uint32_t)raw[q]);
                else
                    key = (K)enc64((long long)raw[q]);
                out_ids[pos] = (int)row[q];
                if (out_keys) ((K *)out_keys)[pos] = key;
                if (out_kvalid) out_kvalid[pos] = kvl[q] ? 1 : 0;
                kand &= (unsigned long long)key;
                kor |= (unsigned long long)key;
            }
        }
        run += btot;
        __syncthreads();   // s_wtot is rewritten next round
    }
    if (keymask) {   // bits shared by every survivor key (dedup sort planning)
        const unsigned alo = __reduce_and_sync(FULL, (unsigned)kand);
        const unsigned ahi = __reduce_and_sync(FULL, (unsigned)(kand >> 32));
        const unsigned olo = __reduce_or_sync(FULL, (unsigned)kor);
        const unsigned ohi = __reduce_or_sync(FULL, (unsigned)(kor >> 32));
        if (lane == 0) {
            atomicAnd(&keymask[0], ((unsigned long long)ahi << 32) | alo);
            atomicOr(&keymask[1], ((unsigned long long)ohi << 32) | olo);
        }
    }
}

// R' without outer predicates (every row survives, in order): a pure
// transform ids[i] = i, keys[i] = enc(key[i]), kvalid[i] -- 4 rows per thread
// with 16-byte loads / stores (a 4-byte access per lane keeps too few bytes
// in flight per SM to approach HBM bandwidth).
template <int KB>
__global__ void __launch_bounds__(256) rp_dense_kernel(long long n, KeySrc ks, int *__restrict__ out_ids,
                                                       void *__restrict__ out_keys, uint8_t *__restrict__ out_kvalid,
                                                       unsigned long long *__restrict__ keymask,
                                                       long long *__restrict__ out_count)
{
    using K = typename std::conditional<KB == 8, uint64_t, uint32_t>::type;
    unsigned long long kand = ~0ull, kor = 0ull;
    const long long n4 = n / 4;
    const long long t0 = blockIdx.x * 256LL + threadIdx.x, nt = (long long)gridDim.x * 256;
    for (long long q = t0; q <= n4; q += nt) {   // q == n4: the ragged tail (n % 4 rows)
        const long long r0 = q * 4;
        const int m = (int)min(4LL, n - r0);
        if (m <= 0) break;
        K k[4];
        if (m == 4 && ks.n_key == 1 && ks.w0 == 4) {
            const int4 v = __ldg(reinterpret_cast<const int4 *>((const int *)ks.c0 + r0));
            const int x[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
            for (int j = 0; j < 4; j++) k[j] = KB == 4 ? (K)enc32(x[j]) : (K)enc64((long long)x[j]);
        } else {
#pragma unroll
            for (int j = 0; j < 4; j++) {
                k[j] = 0;
                if (j >= m) continue;
                const long long row = r0 + j;
                if (ks.n_key == 2)
                    k[j] = (K)(((uint64_t)enc32(__ldg((const int *)ks.c0 + row)) << 32) |
                               enc32(__ldg((const int *)ks.c1 + row)));
                else if (ks.w0 == 4)
                    k[j] = KB == 4 ? (K)enc32(__ldg((const int *)ks.c0 + row))
                                   : (K)enc64((long long)__ldg((const int *)ks.c0 + row));
                else
                    k[j] = (K)enc64(__ldg((const long long *)ks.c0 + row));
            }
        }
        if (m == 4) {
            reinterpret_cast<int4 *>(out_ids)[q] = make_int4((int)r0, (int)r0 + 1, (int)r0 + 2, (int)r0 + 3);
            if (out_keys) {
                if constexpr (KB == 4) {
                    reinterpret_cast<uint4 *>(out_keys)[q] = make_uint4(k[0], k[1], k[2], k[3]);
                } else {
                    reinterpret_cast<ulonglong2 *>(out_keys)[2 * q] = make_ulonglong2(k[0], k[1]);
                    reinterpret_cast<ulonglong2 *>(out_keys)[2 * q + 1] = make_ulonglong2(k[2], k[3]);
                }
            }
        } else {
            for (int j = 0; j < m; j++) {
                out_ids[r0 + j] = (int)(r0 + j);
                if (out_keys) ((K *)out_keys)[r0 + j] = k[j];
            }
        }
        if (out_kvalid)
            for (int j = 0; j < m; j++) {
                const long long row = r0 + j;
                out_kvalid[row] = ((ks.v0 && !__ldg(ks.v0 + row)) || (ks.v1 && !__ldg(ks.v1 + row))) ? 0 : 1;
            }
        for (int j = 0; j < m; j++) {
            kand &= (unsigned long long)k[j];
            kor |= (unsigned long long)k[j];
        }
    }
    if (keymask) {
        const unsigned alo = __reduce_and_sync(FULL, (unsigned)kand);
        const unsigned ahi = __reduce_and_sync(FULL, (unsigned)(kand >> 32));
        const unsigned olo = __reduce_or_sync(FULL, (unsigned)kor);
        const unsigned ohi = __reduce_or_sync(FULL, (unsigned)(kor >> 32));
        if ((threadIdx.x & 31) == 0) {
            atomicAnd(&keymask[0], ((unsigned long long)ahi << 32) | alo);
            atomicOr(&keymask[1], ((unsigned long long)ohi << 32) | olo);
        }
    }
    if (t0 == 0) *out_count = n;
}

// ------------------------------------------------------------------ host side
// Exclusive scan of the per-tile counts (ordered mode) over many CTAs:
// CTA c scans tiles [1024c, 1024c + 1024)
// (one coalesced load each, a block scan) into base[] as chunk-local
// exclusive prefixes and its total into ctot[c]; the last CTA to finish
// scans the chunk totals into coff[] (and *out_count).  A tile's offset is
// base[t] + coff[t >> 10] (29k tiles: one round trip instead of ~29).
__global__ void __launch_bounds__(1024) tile_scan_chunks_kernel(const unsigned *__restrict__ cnt, long long tiles,
                                                                unsigned long long *__restrict__ base,
                                                                unsigned long long *__restrict__ ctot,
                                                                unsigned long long *__restrict__ coff,
                                                                long long *__restrict__ out_count,
                                                                unsigned *__restrict__ done)
{
    __shared__ unsigned long long s_w[32];
    __shared__ bool s_last;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const long long i = blockIdx.x * 1024ll + tid;
    const unsigned long long x = i < tiles ? __ldg(cnt + i) : 0ull;
    unsigned long long incl = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) s_w[warp] = incl;
    __syncthreads();
    unsigned long long pre = incl - x, total = 0;
    for (int w = 0; w < 32; w++) {
        if (w < warp) pre += s_w[w];
        total += s_w[w];
    }
    if (i < tiles) base[i] = pre;
    if (tid == 0) ctot[blockIdx.x] = total;
    __threadfence();
    __syncthreads();
    if (tid == 0) s_last = atomicAdd(done, 1u) == gridDim.x - 1;
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    // the last CTA: exclusive scan of the chunk totals (<= 1024 chunks)
    const unsigned long long c = tid < (int)gridDim.x ? __ldcg(ctot + tid) : 0ull;
    unsigned long long ci = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long y = __shfl_up_sync(FULL, ci, o);
        if (lane >= o) ci += y;
    }
    __syncthreads();
    if (lane == 31) s_w[warp] = ci;
    __syncthreads();
    unsigned long long cp = ci - c, ct = 0;
    for (int w = 0; w < 32; w++) {
        if (w < warp) cp += s_w[w];
        ct += s_w[w];
    }
    if (tid < (int)gridDim.x) coff[tid] = cp;
    if (tid == 0) *out_count = (long long)ct;
}

namespace {

int add_src(SrcCols &sc, const void *p, int w)
{
    if (!p) return -1;
    for (int c = 0; c < sc.n; c++)
        if (sc.ptr[c] == p && sc.w[c] == w) return c;
    sc.ptr[sc.n] = p;
    sc.w[sc.n] = w;
    return sc.n++;
}

// tile size: the largest 256*ITEMS whose stage fits STAGE_MAX bytes; lays
// out the stage.  Returns ITEMS (0 if even 256 rows do not fit).
int layout(SrcCols &sc, int max_items)
{
    int row_bytes = 0;
    for (int c = 0; c < sc.n; c++) row_bytes += sc.w[c];
    int items = max_items;
    while (items > 1 && T_THREADS * items * row_bytes + 16 * sc.n > STAGE_MAX) items >>= 1;
    if (T_THREADS * items * row_bytes + 16 * sc.n > STAGE_MAX) return 0;
    int off = 0;
    for (int c = 0; c < sc.n; c++) {
        sc.off[c] = off;
        off += (T_THREADS * items * sc.w[c] + 15) & ~15;
    }
    sc.stage_bytes = (off + 127) & ~127;
    if (sc.stage_bytes == 0) sc.stage_bytes = 128;
    return items;
}

struct FilterOut {
    int *ids;
    void *keys;
    uint8_t *kvalid;
    void *vals;
    unsigned long long *keymask;
    unsigned *extreme;
    const unsigned long long *tile_base;
    unsigned *tile_count;
    unsigned *counter;
    long long *count;
    unsigned *live_bits;   // ordered two-pass mode: survivor ballots of pass 1 (nullable)
    const unsigned long long *chunk_off = nullptr;   // + offset of the tile's 1024-tile chunk (nullable)
};

template <int KB, int VB, int ITEMS>
cudaError_t launch_t(long long n, const SrcCols &sc, const TPlan &tp, const FilterOut &o, int num_sms,
                     cudaStream_t st)
{
    auto kern = filter_tma_kernel<KB, VB, ITEMS>;
    const int smem = 2 * sc.stage_bytes;
    int occ = 0;
    cudaError_t e0 = per_device_setup((const void *)kern, smem, &occ, [&](int, int *v) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * STAGE_MAX);
        if (e != cudaSuccess) return e;
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(v, kern, T_THREADS, smem);
    });
    if (e0 != cudaSuccess) return e0;
    const long long tiles = (n + T_THREADS * ITEMS - 1) / (T_THREADS * ITEMS);
    long long grid = (long long)num_sms * (occ > 0 ? occ : 1);
    if (grid > tiles) grid = tiles;
    kern<<<(unsigned)grid, T_THREADS, smem, st>>>(n, sc, tp, o.ids, o.keys, o.kvalid, o.vals, o.keymask, o.extreme,
                                                  o.tile_base, o.tile_count, o.counter, o.count, o.live_bits, o.chunk_off);
    return cudaGetLastError();
}

template <int KB, int VB>
cudaError_t launch_items(int items, long long n, const SrcCols &sc, const TPlan &tp, const FilterOut &o, int num_sms,
                         cudaStream_t st)
{
    switch (items) {
    case 16: return launch_t<KB, VB, 16>(n, sc, tp, o, num_sms, st);
    case 8: return launch_t<KB, VB, 8>(n, sc, tp, o, num_sms, st);
    case 4: return launch_t<KB, VB, 4>(n, sc, tp, o, num_sms, st);
    case 2: return launch_t<KB, VB, 2>(n, sc, tp, o, num_sms, st);
    default: return launch_t<KB, VB, 1>(n, sc, tp, o, num_sms, st);
    }
}

cudaError_t dispatch(int k, int v, int items, long long n, const SrcCols &sc, const TPlan &tp, const FilterOut &o,
                     int num_sms, cudaStream_t st)
{
    if (k == 0 && v == 0) return launch_items<0, 0>(items, n, sc, tp, o, num_sms, st);
    if (k == 4 && v == 0) return launch_items<4, 0>(items, n, sc, tp, o, num_sms, st);
    if (k == 4 && v == 4) return launch_items<4, 4>(items, n, sc, tp, o, num_sms, st);
    if (k == 4 && v == 8) return launch_items<4, 8>(items, n, sc, tp, o, num_sms, st);
    if (k == 8 && v == 0) return launch_items<8, 0>(items, n, sc, tp, o, num_sms, st);
    if (k == 8 && v == 4) return launch_items<8, 4>(items, n, sc, tp, o, num_sms, st);
    return launch_items<8, 8>(items, n, sc, tp, o, num_sms, st);
}

}  // namespace

size_t filter_scratch_bytes(long long n)
{
    // counters + per-tile counts / offsets (two-pass mode), or the ordered
    // filter's chunk counts + ballot words
    const size_t two_pass = 1024 + 1024 + (size_t)(n / T_THREADS + 2) * 12 + (size_t)(n / 32 + 2) * 4 + 64 * 16 * 4 +
                            (size_t)(n / T_THREADS / 1024 + 2) * 16;
    const size_t one_launch = RP_BITS_OFF + (size_t)(n / 32 + 2) * 4 + 256;
    return two_pass > one_launch ? two_pass : one_launch;
}

// the counter words (the ordered filter's grid barrier among them)
size_t filter_zero_bytes(long long, bool) { return 1024; }

// ---- one kernel filling a list of small regions (FillList)
__global__ void fill_list_kernel(FillList f)
{
    for (int r = 0; r < f.n; r++) {
        unsigned char *p = (unsigned char *)f.p[r];
        const unsigned long long b = f.bytes[r];
        if (f.word[r]) {   // 64-bit pattern (e.g. the MIN/MAX identity of the partials)
            unsigned long long *w = (unsigned long long *)p;
            for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < (long long)(b / 8);
                 i += (long long)gridDim.x * blockDim.x)
                w[i] = f.pat[r];
            continue;
        }
        const unsigned v = (unsigned)f.pat[r];
        // aligned 16-B body, byte head / tail
        const unsigned long long head = (16 - ((unsigned long long)p & 15)) & 15;
        const unsigned long long h = head < b ? head : b;
        const unsigned long long body = (b - h) / 16;
        const long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x;
        const long long nt = (long long)gridDim.x * blockDim.x;
        for (long long i = t; i < (long long)h; i += nt) p[i] = (unsigned char)v;
        uint4 *q = (uint4 *)(p + h);
        for (long long i = t; i < (long long)body; i += nt) q[i] = make_uint4(v, v, v, v);
        for (long long i = (long long)(h + body * 16) + t; i < (long long)b; i += nt) p[i] = (unsigned char)v;
    }
}

cudaError_t launch_fill(const FillList &f, cudaStream_t st, long long *launches)
{
    if (f.n == 0) return cudaSuccess;
    unsigned long long mx = 0;
    for (int r = 0; r < f.n; r++) mx = f.bytes[r] > mx ? f.bytes[r] : mx;
    long long blocks = (long long)((mx / 16 + 255) / 256);
    if (blocks < 1) blocks = 1;
    if (blocks > 148 * 4) blocks = 148 * 4;
    fill_list_kernel<<<(unsigned)blocks, 256, 0, st>>>(f);
    ++*launches;
    return cudaGetLastError();
}

namespace {
// NESTGPU_FILTER_TWO_PASS=1: the round-1 count + scan + write R' filter
// (kept for side-by-side measurement)
bool getenv_two_pass()
{
    static const bool v = [] {
        const char *s = getenv("NESTGPU_FILTER_TWO_PASS");
        return s && s[0] == '1';
    }();
    return v;
}

template <int KB, int ITEMS>
cudaError_t launch_rp_t(long long n, const SrcCols &sc, const TPlan &tp, const KeySrc &ks, int *ids, void *keys,
                        uint8_t *kvalid, unsigned long long *keymask, void *scratch, long long *count, int num_sms,
                        cudaStream_t st)
{
    auto kern = filter_rp_kernel<KB, ITEMS>;
    const bool preds = sc.n > 0;
    const int smem = preds ? 2 * sc.stage_bytes : 0;
    int occ = 0;
    cudaError_t e0 = per_device_setup((const void *)kern, smem, &occ, [&](int, int *v) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * STAGE_MAX);
        if (e != cudaSuccess) return e;
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(v, kern, T_THREADS, smem);
    });
    if (e0 != cudaSuccess) return e0;
    if (occ < 1) return cudaErrorInvalidConfiguration;
    // every CTA resident (the grid barrier): SMs x occupancy, chunks of whole
    // 256-row groups (ballot words never straddle two chunks)
    long long grid = (long long)num_sms * occ;
    if (grid > 2048) grid = 2048;   // counts area: 16 KB
    long long chunk = (n + grid - 1) / grid;
    chunk = (chunk + T_THREADS - 1) / T_THREADS * T_THREADS;
    const long long used = (n + chunk - 1) / chunk;
    if (!preds) grid = used;   // no barrier: only CTAs with rows
    unsigned *barrier = (unsigned *)scratch;
    unsigned long long *counts = (unsigned long long *)((char *)scratch + RP_COUNTS_OFF);
    unsigned *bits = (unsigned *)((char *)scratch + RP_BITS_OFF);
    if (!preds) {   // every row survives: the vectorised transform
        long long blocks = (n / 4 + 1 + 255) / 256;
        if (blocks > (long long)num_sms * 16) blocks = (long long)num_sms * 16;
        rp_dense_kernel<KB><<<(unsigned)blocks, 256, 0, st>>>(n, ks, ids, keys, kvalid, keymask, count);
        return cudaGetLastError();
    }
    void *args[] = {(void *)&n, (void *)&chunk, (void *)&sc, (void *)&tp, (void *)&ks, (void *)&ids, (void *)&keys,
                    (void *)&kvalid, (void *)&keymask, (void *)&bits, (void *)&counts, (void *)&barrier,
                    (void *)&count};
    return cudaLaunchCooperativeKernel((const void *)kern, dim3((unsigned)grid), dim3(T_THREADS), args, (size_t)smem, st);
}

template <int KB>
cudaError_t launch_rp_items(int items, long long n, const SrcCols &sc, const TPlan &tp, const KeySrc &ks, int *ids,
                            void *keys, uint8_t *kvalid, unsigned long long *keymask, void *scratch, long long *count,
                            int num_sms, cudaStream_t st)
{
    switch (items) {
    case 32: return launch_rp_t<KB, 32>(n, sc, tp, ks, ids, keys, kvalid, keymask, scratch, count, num_sms, st);
    case 16: return launch_rp_t<KB, 16>(n, sc, tp, ks, ids, keys, kvalid, keymask, scratch, count, num_sms, st);
    case 8: return launch_rp_t<KB, 8>(n, sc, tp, ks, ids, keys, kvalid, keymask, scratch, count, num_sms, st);
    case 4: return launch_rp_t<KB, 4>(n, sc, tp, ks, ids, keys, kvalid, keymask, scratch, count, num_sms, st);
    case 2: return launch_rp_t<KB, 2>(n, sc, tp, ks, ids, keys, kvalid, keymask, scratch, count, num_sms, st);
    default: return launch_rp_t<KB, 1>(n, sc, tp, ks, ids, keys, kvalid, keymask, scratch, count, num_sms, st);
    }
}

cudaError_t launch_rp(int kb, int items, long long n, const SrcCols &sc, const TPlan &tp, const KeySrc &ks, int *ids,
                      void *keys, uint8_t *kvalid, unsigned long long *keymask, void *scratch, long long *count,
                      int num_sms, cudaStream_t st)
{
    if (kb == 8) return launch_rp_items<8>(items, n, sc, tp, ks, ids, keys, kvalid, keymask, scratch, count, num_sms, st);
    return launch_rp_items<4>(items, n, sc, tp, ks, ids, keys, kvalid, keymask, scratch, count, num_sms, st);
}
}  // namespace

// Source indices of a plan (host side), resolved into stage offsets by
// resolve() once the tile size / stage layout is known.
struct SrcPlan {
    int x[MAX_PREDS], xv[MAX_PREDS], y[MAX_PREDS], yv[MAX_PREDS];
    int key0, key0v, key1, key1v, val, valv;
};

static Col col_of(const SrcCols &sc, int s)
{
    return s < 0 ? Col{-1, 0} : Col{sc.off[s], sc.w[s]};
}

static void resolve(const SrcCols &sc, const SrcPlan &sp, TPlan &tp)
{
    for (int k = 0; k < tp.n_preds; k++) {
        tp.p[k].x = col_of(sc, sp.x[k]);
        tp.p[k].xv = col_of(sc, sp.xv[k]);
        tp.p[k].y = col_of(sc, sp.y[k]);
        tp.p[k].yv = col_of(sc, sp.yv[k]);
    }
    tp.key0 = col_of(sc, sp.key0);
    tp.key0v = col_of(sc, sp.key0v);
    tp.key1 = col_of(sc, sp.key1);
    tp.key1v = col_of(sc, sp.key1v);
    tp.val = col_of(sc, sp.val);
    tp.valv = col_of(sc, sp.valv);
}

cudaError_t launch_filter(long long n, const PredSet &preds, const KeySrc &key, int kb, const ValSrc &val, int vb,
                          int drop_null_key, int drop_null_val, int *out_ids, void *out_keys, uint8_t *out_kvalid,
                          void *out_vals, unsigned long long *keymask, unsigned *extreme, void *scratch,
                          long long *out_count, cudaStream_t st, long long *launches, bool prezeroed,
                          int ordered_phase)
{
    cudaError_t e = prezeroed || ordered_phase == 2 ? cudaSuccess : cudaMemsetAsync(out_count, 0, sizeof(long long), st);
    if (e != cudaSuccess || n <= 0) return e;
    // the column segments a tile needs, deduplicated
    SrcCols sc;
    memset(&sc, 0, sizeof sc);
    SrcPlan sp;
    TPlan tp;
    memset(&tp, 0, sizeof tp);
    tp.n_preds = preds.n;
    for (int k = 0; k < preds.n; k++) {
        const DevPred &p = preds.p[k];
        sp.x[k] = add_src(sc, p.col, p.w);
        sp.xv[k] = add_src(sc, p.valid, 1);
        sp.y[k] = add_src(sc, p.rhs, p.rhs_w);
        sp.yv[k] = add_src(sc, p.rhs_valid, 1);
        tp.p[k].op = p.op;
        tp.p[k].lit = p.lit;
    }
    const int n_pred_src = sc.n;
    const int k = kb == 8 ? 8 : (kb == 4 ? 4 : 0);
    const int v = val.c ? (vb == 8 ? 8 : 4) : 0;
    sp.key0 = sp.key0v = sp.key1 = sp.key1v = sp.val = sp.valv = -1;
    tp.n_key = key.n_key;
    if (k) {
        sp.key0 = add_src(sc, key.c0, key.n_key == 2 ? 4 : key.w0);
        sp.key0v = add_src(sc, key.v0, 1);
        if (key.n_key == 2) {
            sp.key1 = add_src(sc, key.c1, 4);
            sp.key1v = add_src(sc, key.v1, 1);
        }
    }
    if (v) {
        sp.val = add_src(sc, val.c, val.w);
        sp.valv = add_src(sc, val.v, 1);
    }
    tp.drop_null_key = drop_null_key;
    tp.drop_null_val = drop_null_val;
    const int items = layout(sc, 16);
    if (!items) return cudaErrorInvalidValue;
    resolve(sc, sp, tp);
    const bool ordered = out_ids || ordered_phase;
    const bool one_pass = out_ids && !ordered_phase && !out_vals && !extreme && !drop_null_key && !drop_null_val && k &&
                          !getenv_two_pass();
    if (ordered_phase != 2 && (!prezeroed || (out_ids && !one_pass))) {
        e = cudaMemsetAsync(scratch, 0, 1024, st);
        if (e != cudaSuccess) return e;
    }
    int dev = 0, num_sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&num_sms, cudaDevAttrMultiProcessorCount, dev);
    FilterOut o{out_ids, out_keys, out_kvalid, out_vals, keymask, extreme, nullptr, nullptr,
                (unsigned *)scratch, out_count};
    if (one_pass) {
        // ordered R': one launch, predicate columns read once, survivors'
        // keys gathered (filter_rp_kernel)
        SrcCols sc1 = sc;
        sc1.n = n_pred_src;   // predicate columns come first in the source list
        const int it1 = layout(sc1, NG_RP_ITEMS);
        if (!it1) return cudaErrorInvalidValue;
        SrcPlan sp1 = sp;
        sp1.key0 = sp1.key0v = sp1.key1 = sp1.key1v = sp1.val = sp1.valv = -1;
        TPlan tp1 = tp;
        resolve(sc1, sp1, tp1);
        e = launch_rp(k, it1, n, sc1, tp1, key, out_ids, out_keys, out_kvalid, keymask, scratch, out_count, num_sms,
                      st);
        ++*launches;
        return e;
    }
    if (ordered) {
        // Ordered (R', or S' of a key-ordered column): pass 1 counts
        // survivors per tile reading only the predicate columns (same tile
        // size as pass 2), then an exclusive scan.  ordered_phase 1 stops
        // after the scan (*out_count is final: the caller sizes the output),
        // 2 runs only pass 2 with the same scratch.
        if (drop_null_key || drop_null_val) return cudaErrorInvalidValue;
        const long long tiles = (n + T_THREADS * items - 1) / (T_THREADS * items);
        unsigned *tcount = (unsigned *)((char *)scratch + 1024);
        unsigned long long *tbase = (unsigned long long *)((char *)scratch + 1024 + ((tiles * 4 + 255) & ~255ll));
        const long long nchunks = (tiles + 1023) / 1024;
        unsigned long long *ctot = (unsigned long long *)((char *)tbase + ((tiles * 8 + 255) & ~255ll));
        unsigned long long *coff = ctot + nchunks;
        unsigned *cdone = (unsigned *)scratch + 128;   // a zeroed counter word (scratch bytes 512..515)
        // the two-call mode keeps pass 1's survivor ballots for pass 2
        unsigned *bits = ordered_phase ? (unsigned *)((char *)ctot + ((nchunks * 16 + 255) & ~255ll)) : nullptr;
        if (ordered_phase == 2) {
            // pass 2 streams only the key / payload columns: the predicate
            // columns are not read again
            SrcCols sc2;
            memset(&sc2, 0, sizeof sc2);
            SrcPlan sp2 = sp;
            sp2.key0 = sp2.key0v = sp2.key1 = sp2.key1v = sp2.val = sp2.valv = -1;
            if (k) {
                sp2.key0 = add_src(sc2, key.c0, key.n_key == 2 ? 4 : key.w0);
                sp2.key0v = add_src(sc2, key.v0, 1);
                if (key.n_key == 2) {
                    sp2.key1 = add_src(sc2, key.c1, 4);
                    sp2.key1v = add_src(sc2, key.v1, 1);
                }
            }
            if (v) {
                sp2.val = add_src(sc2, val.c, val.w);
                sp2.valv = add_src(sc2, val.v, 1);
            }
            int off2 = 0;
            for (int c = 0; c < sc2.n; c++) {
                sc2.off[c] = off2;
                off2 += (T_THREADS * items * sc2.w[c] + 15) & ~15;
            }
            sc2.stage_bytes = off2 ? ((off2 + 127) & ~127) : 128;
            TPlan tp2 = tp;
            tp2.n_preds = 0;
            resolve(sc2, sp2, tp2);
            o.tile_base = tbase;
            o.chunk_off = coff;
            o.live_bits = bits;
            e = dispatch(k, v, items, n, sc2, tp2, o, num_sms, st);
            ++*launches;
            return e;
        }
        SrcCols sc1 = sc;
        sc1.n = n_pred_src;   // predicate columns come first in the source list
        int off = 0;
        for (int c = 0; c < sc1.n; c++) {
            sc1.off[c] = off;
            off += (T_THREADS * items * sc1.w[c] + 15) & ~15;
        }
        sc1.stage_bytes = off ? ((off + 127) & ~127) : 128;
        SrcPlan sp1 = sp;
        sp1.key0 = sp1.key0v = sp1.key1 = sp1.key1v = sp1.val = sp1.valv = -1;
        TPlan tp1 = tp;
        resolve(sc1, sp1, tp1);
        FilterOut o1{nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, tcount,
                     (unsigned *)scratch + 64, out_count, bits};
        e = launch_items<0, 0>(items, n, sc1, tp1, o1, num_sms, st);
        if (e != cudaSuccess) return e;
        tile_scan_chunks_kernel<<<(unsigned)nchunks, 1024, 0, st>>>(tcount, tiles, tbase, ctot, coff, out_count,
                                                                    cdone);
        o.tile_base = tbase;
        o.chunk_off = coff;
        *launches += 2;
        if (ordered_phase == 1) return cudaGetLastError();
    }
    e = dispatch(k, v, items, n, sc, tp, o, num_sms, st);
    ++*launches;
    return e;
}

}  // namespace ng
