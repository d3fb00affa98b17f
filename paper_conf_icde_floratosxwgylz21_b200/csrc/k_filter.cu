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
//    vector lives in a register bitmask, warp ballots + popc give ranks,
//    and a CTA-wide decoupled look-back gives the tile's global offset;
//  * survivors are written in row order.
// The S' pass also reduces AND / OR over the encoded keys (radix digits on
// which all keys agree need no sort pass) and flags payloads equal to the
// MIN/MAX identity.
#include <climits>
#include <cstring>
#include <type_traits>

#include "internal.h"
#include "scan.cuh"

namespace ng {

constexpr int T_THREADS = 256;
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

struct TPred {
    int col, valid, rhs, rhs_valid;  // source indices, -1 = none
    int op;
    long long lit;
};

struct TPlan {
    int n_preds;
    TPred p[MAX_PREDS];
    int key0, key0v, key1, key1v, n_key;
    int val, valv;
    int drop_null_key, drop_null_val;
};

size_t filter_scratch_bytes(long long n) { return (size_t)(n / T_THREADS + 2) * 8 + 256; }

template <int ITEMS>
struct Stage {
    const unsigned char *base;
    const SrcCols *sc;
    template <typename T>
    __device__ __forceinline__ T at(int c, int li) const
    {
        return reinterpret_cast<const T *>(base + sc->off[c])[li];
    }
    __device__ __forceinline__ long long val(int c, int li) const
    {
        const int w = sc->w[c];
        return w == 4 ? (long long)at<int>(c, li) : (w == 8 ? at<long long>(c, li) : (long long)at<uint8_t>(c, li));
    }
    __device__ __forceinline__ unsigned nonnull(int c, unsigned live, int tid) const
    {
        if (c < 0) return live;
        unsigned out = 0;
#pragma unroll
        for (int j = 0; j < ITEMS; j++)
            if ((live >> j & 1u) && at<uint8_t>(c, j * T_THREADS + tid)) out |= 1u << j;
        return out;
    }
};

template <int ITEMS, int OP>
__device__ __forceinline__ unsigned cmp_items(const Stage<ITEMS> &S, const TPred &p, unsigned live, int tid)
{
    unsigned m = 0;
#pragma unroll
    for (int j = 0; j < ITEMS; j++) {
        const int li = j * T_THREADS + tid;
        const long long x = S.val(p.col, li);
        const long long y = p.rhs >= 0 ? S.val(p.rhs, li) : p.lit;
        if ((live >> j & 1u) && cmp_ct<OP>(x, y)) m |= 1u << j;
    }
    return m;
}

// ORDERED: survivors keep row order (R', whose order is the result's order)
// via the decoupled look-back; otherwise (S', re-ordered by the sort anyway
// and order-free for the nested loop) a tile claims its output range with
// one atomicAdd on the survivor counter -- no dependency between tiles.
template <int KB, int VB, int ITEMS, bool ORDERED>
__global__ void __launch_bounds__(T_THREADS)
filter_tma_kernel(long long n, SrcCols sc, TPlan tp, int *__restrict__ out_ids, void *__restrict__ out_keys,
                  uint8_t *__restrict__ out_kvalid, void *__restrict__ out_vals,
                  unsigned long long *__restrict__ keymask, unsigned *__restrict__ extreme,
                  unsigned long long *__restrict__ status, unsigned *__restrict__ counter,
                  long long *__restrict__ out_count)
{
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
        const Stage<ITEMS> S{smem + stage * sc.stage_bytes, &sc};
        const long long base = tile * TILE;
        const long long rows = min((long long)TILE, n - base);

        unsigned live = 0;
#pragma unroll
        for (int j = 0; j < ITEMS; j++)
            if (j * T_THREADS + tid < rows) live |= 1u << j;
        // local predicates (NULL operands are not TRUE, reading R2)
        for (int k = 0; k < tp.n_preds; k++) {
            const TPred &p = tp.p[k];
            live = S.nonnull(p.valid, live, tid);
            live = S.nonnull(p.rhs_valid, live, tid);
            switch (p.op) {
            case EQ: live &= cmp_items<ITEMS, EQ>(S, p, live, tid); break;
            case NE: live &= cmp_items<ITEMS, NE>(S, p, live, tid); break;
            case LT: live &= cmp_items<ITEMS, LT>(S, p, live, tid); break;
            case LE: live &= cmp_items<ITEMS, LE>(S, p, live, tid); break;
            case GT: live &= cmp_items<ITEMS, GT>(S, p, live, tid); break;
            default: live &= cmp_items<ITEMS, GE>(S, p, live, tid); break;
            }
        }
        unsigned kvalid = live;
        if constexpr (KB > 0) {
            kvalid = S.nonnull(tp.key1v, S.nonnull(tp.key0v, live, tid), tid);
            if (tp.drop_null_key) live = kvalid;
        }
        if constexpr (VB > 0) {
            const unsigned vv = S.nonnull(tp.valv, live, tid);
            if (tp.drop_null_val) live = vv;
        }
        unsigned rank[ITEMS];
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            const unsigned m = __ballot_sync(FULL, live >> j & 1u);
            if (lane == 0) s_cnt[j][warp] = __popc(m);
            rank[j] = __popc(m & lanemask_lt());
        }
        unsigned long long tb;
        if constexpr (ORDERED) {
            tb = tile_offsets<ITEMS, T_THREADS>(s_cnt, status, tile, num_tiles, out_count);
        } else {
            __syncthreads();
            if (tid < 32) {  // exclusive scan of the (item, warp) counts + one atomic claim
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
                if (lane == 31)
                    s_claim = incl ? atomicAdd((unsigned long long *)out_count, (unsigned long long)incl) : 0ull;
            }
            __syncthreads();
            tb = s_claim;
        }
#pragma unroll
        for (int j = 0; j < ITEMS; j++) {
            if (!(live >> j & 1u)) continue;
            const int li = j * T_THREADS + tid;
            const long long pos = (long long)tb + s_cnt[j][warp] + rank[j];
            if (out_ids) out_ids[pos] = (int)(base + li);
            if constexpr (KB > 0) {
                K key;
                if (tp.n_key == 2)
                    key = (K)(((uint64_t)enc32(S.template at<int>(tp.key0, li)) << 32) |
                              enc32(S.template at<int>(tp.key1, li)));
                else if constexpr (KB == 4)
                    key = (K)enc32(S.template at<int>(tp.key0, li));
                else
                    key = (K)enc64(S.val(tp.key0, li));
                if (out_keys) ((K *)out_keys)[pos] = key;
                if (out_kvalid) out_kvalid[pos] = (kvalid >> j) & 1u;
                kand &= (unsigned long long)key;
                kor |= (unsigned long long)key;
            }
            if constexpr (VB > 0) {
                const V v = (V)S.val(tp.val, li);
                if (out_vals) ((V *)out_vals)[pos] = v;
                ext_max |= v == (VB == 8 ? (V)LLONG_MAX : (V)INT_MAX);
                ext_min |= v == (VB == 8 ? (V)LLONG_MIN : (V)INT_MIN);
                const unsigned long long a = v < 0 ? 0ull - (unsigned long long)(long long)v : (unsigned long long)v;
                vabs = a > vabs ? a : vabs;
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

// ------------------------------------------------------------------ host side
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

template <int KB, int VB, int ITEMS, bool ORDERED>
cudaError_t launch_t(long long n, const SrcCols &sc, const TPlan &tp, int *out_ids, void *out_keys,
                     uint8_t *out_kvalid, void *out_vals, unsigned long long *keymask, unsigned *extreme,
                     void *scratch, long long *out_count, int num_sms, cudaStream_t st)
{
    auto kern = filter_tma_kernel<KB, VB, ITEMS, ORDERED>;
    const int smem = 2 * sc.stage_bytes;
    static int occ_for = -1, occ = 0;
    if (occ_for != smem) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * STAGE_MAX);
        if (e != cudaSuccess) return e;
        e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, T_THREADS, smem);
        if (e != cudaSuccess) return e;
        occ_for = smem;
    }
    const long long tiles = (n + T_THREADS * ITEMS - 1) / (T_THREADS * ITEMS);
    long long grid = (long long)num_sms * (occ > 0 ? occ : 1);
    if (grid > tiles) grid = tiles;
    unsigned *counter = (unsigned *)scratch;
    unsigned long long *status = (unsigned long long *)((char *)scratch + 256);
    kern<<<(unsigned)grid, T_THREADS, smem, st>>>(n, sc, tp, out_ids, out_keys, out_kvalid, out_vals, keymask,
                                                  extreme, status, counter, out_count);
    return cudaGetLastError();
}

template <int KB, int VB, bool ORDERED>
cudaError_t launch_items(int items, long long n, const SrcCols &sc, const TPlan &tp, int *out_ids, void *out_keys,
                         uint8_t *out_kvalid, void *out_vals, unsigned long long *keymask, unsigned *extreme,
                         void *scratch, long long *out_count, int num_sms, cudaStream_t st)
{
#define NG_LT(I) launch_t<KB, VB, I, ORDERED>(n, sc, tp, out_ids, out_keys, out_kvalid, out_vals, keymask, extreme, scratch, \
                                     out_count, num_sms, st)
    switch (items) {
    case 16: return NG_LT(16);
    case 8: return NG_LT(8);
    case 4: return NG_LT(4);
    case 2: return NG_LT(2);
    default: return NG_LT(1);
    }
#undef NG_LT
}

}  // namespace

cudaError_t launch_filter(long long n, const PredSet &preds, const KeySrc &key, int kb, const ValSrc &val, int vb,
                          int drop_null_key, int drop_null_val, int *out_ids, void *out_keys, uint8_t *out_kvalid,
                          void *out_vals, unsigned long long *keymask, unsigned *extreme, void *scratch,
                          long long *out_count, cudaStream_t st, long long *launches)
{
    cudaError_t e = cudaMemsetAsync(out_count, 0, sizeof(long long), st);
    if (e != cudaSuccess || n <= 0) return e;
    // the column segments a tile needs, deduplicated
    SrcCols sc;
    memset(&sc, 0, sizeof sc);
    TPlan tp;
    memset(&tp, 0, sizeof tp);
    tp.n_preds = preds.n;
    for (int k = 0; k < preds.n; k++) {
        const DevPred &p = preds.p[k];
        tp.p[k].col = add_src(sc, p.col, p.w);
        tp.p[k].valid = add_src(sc, p.valid, 1);
        tp.p[k].rhs = add_src(sc, p.rhs, p.rhs_w);
        tp.p[k].rhs_valid = add_src(sc, p.rhs_valid, 1);
        tp.p[k].op = p.op;
        tp.p[k].lit = p.lit;
    }
    const int k = kb == 8 ? 8 : (kb == 4 ? 4 : 0);
    const int v = val.c ? (vb == 8 ? 8 : 4) : 0;
    tp.key0 = tp.key0v = tp.key1 = tp.key1v = tp.val = tp.valv = -1;
    tp.n_key = key.n_key;
    if (k) {
        tp.key0 = add_src(sc, key.c0, key.n_key == 2 ? 4 : key.w0);
        tp.key0v = add_src(sc, key.v0, 1);
        if (key.n_key == 2) {
            tp.key1 = add_src(sc, key.c1, 4);
            tp.key1v = add_src(sc, key.v1, 1);
        }
    }
    if (v) {
        tp.val = add_src(sc, val.c, val.w);
        tp.valv = add_src(sc, val.v, 1);
    }
    tp.drop_null_key = drop_null_key;
    tp.drop_null_val = drop_null_val;
    // tile size: the largest 256*ITEMS whose stage fits STAGE_MAX bytes
    int row_bytes = 0;
    for (int c = 0; c < sc.n; c++) row_bytes += sc.w[c];
    int items = 16;
    while (items > 1 && T_THREADS * items * row_bytes + 16 * sc.n > STAGE_MAX) items >>= 1;
    if (T_THREADS * items * row_bytes + 16 * sc.n > STAGE_MAX) return cudaErrorInvalidValue;
    int off = 0;
    for (int c = 0; c < sc.n; c++) {
        sc.off[c] = off;
        off += (T_THREADS * items * sc.w[c] + 15) & ~15;
    }
    sc.stage_bytes = (off + 127) & ~127;
    if (sc.stage_bytes == 0) sc.stage_bytes = 128;
    e = cudaMemsetAsync(scratch, 0, filter_scratch_bytes(n), st);
    if (e != cudaSuccess) return e;
    int dev = 0, num_sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&num_sms, cudaDevAttrMultiProcessorCount, dev);
#define NG_F(KB_, VB_) e = out_ids ? launch_items<KB_, VB_, true>(items, n, sc, tp, out_ids, out_keys, out_kvalid,  \
                                                                   out_vals, keymask, extreme, scratch, out_count, \
                                                                   num_sms, st)                                     \
                              : launch_items<KB_, VB_, false>(items, n, sc, tp, out_ids, out_keys, out_kvalid, out_vals, keymask, \
                                                 extreme, scratch, out_count, num_sms, st)
    if (k == 0 && v == 0) NG_F(0, 0);
    else if (k == 4 && v == 0) NG_F(4, 0);
    else if (k == 4 && v == 4) NG_F(4, 4);
    else if (k == 4 && v == 8) NG_F(4, 8);
    else if (k == 8 && v == 0) NG_F(8, 0);
    else if (k == 8 && v == 4) NG_F(8, 4);
    else NG_F(8, 8);
#undef NG_F
    ++*launches;
    return e;
}

}  // namespace ng
