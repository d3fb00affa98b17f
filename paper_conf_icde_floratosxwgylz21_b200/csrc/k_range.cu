// k_range.cu -- a5 + a6: the indexed, vectorised subquery.
//
// PAPER.md P:315 (§III-D "Indexing"): "locate a valid range of S.col1 by using
// the binary search on the index and only scan a portion of table S";
// P:317 ("Vectorization"): fuse the per-iteration kernels of many passed-in
// values into one kernel.  One launch evaluates the subquery for every R'
// tuple: each thread binary-searches the sorted S' keys for its tuple's
// encoded key and derives the qualifying range(s) for the correlated operator
// (S' ascending, N = |S'|, predicate r.key OP s.key):
//     '='  [lb, ub)      '<'  [ub, N)     '<=' [lb, N)
//     '>'  [0, lb)       '>=' [0, ub)     '!=' [0, lb) u [ub, N)
// COUNT / EXISTS need only the range length; MIN/MAX/SUM/AVG fold the
// co-sorted payload.  Short ranges are folded by the owning thread; long ones
// are appended to a work list and folded warp-per-range with coalesced loads
// and warp reductions (load balance for skewed / non-equality ranges).
//
// Index-pruned evaluation (extending P:315's "only scan
// a portion of table S"): when the index carries prefix / suffix aggregates
// of its co-sorted payload (built once per index and aggregate kind), a
// range that is a prefix or suffix of S' -- every non-equality operator --
// and any SUM/AVG range is answered in O(1) from them instead of scanned:
//   pre[p] = AGG(payload[0..p)),  suf[p] = AGG(payload[p..N)),  pre[0] =
//   suf[N] = identity;  SUM uses pre only (sum[a,b) = pre[b] - pre[a]).
// '=' MIN/MAX (skew, P:331's hot keys): per-key group aggregates grp[p] =
// AGG(payload[start of p's key run .. p]) (a segmented scan, built once per
// index), passed in `pre`: the group [lb, ub) folds to grp[ub - 1] in O(1),
// so a hot key costs one load per outer tuple instead of its whole run.
#include <type_traits>

#include "internal.h"

namespace ng {

constexpr int R_THREADS = 256;
constexpr int R_SHORT = 32;

struct LongItem {
    int r, lb, ub, pad;
};

// Search samples: every stride-th key of the index, staged in shared memory
// by each CTA, narrow a binary search to one stride-wide window of the keys
// before it touches global memory (the top ~12 levels of the search come from
// shared memory instead of ~12 dependent L2 round trips).
#ifndef NG_SAMP_BYTES
#define NG_SAMP_BYTES 16384
#endif
constexpr int SAMP_BYTES = NG_SAMP_BYTES;

size_t range_scratch_bytes(long long n_rp_max)
{
    return 256 + (size_t)(n_rp_max > 0 ? n_rp_max : 1) * sizeof(LongItem) + SAMP_BYTES;
}

template <typename K>
__global__ void __launch_bounds__(256) sample_kernel(const K *__restrict__ a, int stride, int M, K *__restrict__ samp)
{
    const int j = blockIdx.x * 256 + threadIdx.x;
    if (j < M) samp[j] = a[(long long)j * stride];
}

// first i in [0, N) with a[i] >= k (LOWER) or a[i] > k (!LOWER): samples
// s[j] = a[j * stride], j < M, locate the window ((J-1)*stride, J*stride].
template <bool LOWER, typename K>
__device__ __forceinline__ int bound_sampled(const K *__restrict__ a, int N, const K *s_samp, int M, int stride, K k)
{
    int lo = 0, hi = M;
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (LOWER ? s_samp[mid] < k : s_samp[mid] <= k) lo = mid + 1;
        else hi = mid;
    }
    if (lo == 0) return 0;
    int glo = (lo - 1) * stride + 1;
    int ghi = lo < M ? lo * stride : N;
    while (glo < ghi) {
        const int mid = (int)(((unsigned)glo + (unsigned)ghi) >> 1);
        if (LOWER ? __ldg(a + mid) < k : __ldg(a + mid) <= k) glo = mid + 1;
        else ghi = mid;
    }
    return glo;
}

// upper bound of k given lb = its lower bound: gallop from lb (qualifying
// ranges of '=' are short), then binary search the last doubling step
template <typename K>
__device__ __forceinline__ int upper_from(const K *__restrict__ a, int N, int lb, K k)
{
    if (lb >= N || __ldg(a + lb) > k) return lb;
    int lo = lb + 1, step = 1;   // invariant: a[lo - 1] <= k
    while (lo + step - 1 < N && __ldg(a + lo + step - 1) <= k) {
        lo += step;
        step <<= 1;
    }
    int hi = lo + step - 1 < N ? lo + step - 1 : N;   // a[hi] > k or hi == N
    while (lo < hi) {
        const int mid = (int)(((unsigned)lo + (unsigned)hi) >> 1);
        if (__ldg(a + mid) <= k) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

template <typename K>
__device__ __forceinline__ int lower_bound_g(const K *__restrict__ a, int lo, int hi, K k)
{
    while (lo < hi) {
        int mid = (int)(((unsigned)lo + (unsigned)hi) >> 1);
        if (__ldg(a + mid) < k) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}
template <typename K>
__device__ __forceinline__ int upper_bound_g(const K *__restrict__ a, int lo, int hi, K k)
{
    while (lo < hi) {
        int mid = (int)(((unsigned)lo + (unsigned)hi) >> 1);
        if (__ldg(a + mid) <= k) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

template <int OP>
__device__ __forceinline__ void pieces(int lb, int ub, int N, int &a0, int &b0, int &a1, int &b1)
{
    a1 = b1 = 0;
    if constexpr (OP == EQ) { a0 = lb; b0 = ub; }
    else if constexpr (OP == LT) { a0 = ub; b0 = N; }
    else if constexpr (OP == LE) { a0 = lb; b0 = N; }
    else if constexpr (OP == GT) { a0 = 0; b0 = lb; }
    else if constexpr (OP == GE) { a0 = 0; b0 = ub; }
    else { a0 = 0; b0 = lb; a1 = ub; b1 = N; }
}

template <int AGG, typename V>
__device__ __forceinline__ void fold(long long &acc, V v)
{
    if constexpr (AGG == MIN) acc = min(acc, (long long)v);
    else if constexpr (AGG == MAX) acc = max(acc, (long long)v);
    else acc += (long long)v;
}

template <typename K, int VB, int OP, int AGG>
__global__ void __launch_bounds__(R_THREADS)
range_short_kernel(const long long *__restrict__ d_nrp, const K *__restrict__ rkeys, const K *__restrict__ skeys,
                   const void *__restrict__ svals_, int N, const K *__restrict__ samp, int M, int stride,
                   const long long *__restrict__ pre, const long long *__restrict__ suf, long long *__restrict__ acc,
                   long long *__restrict__ cnt, LongItem *__restrict__ list, unsigned *__restrict__ list_n,
                   const long long *__restrict__ pre_hi, long long *__restrict__ acc_hi)
{
    using V = typename std::conditional<VB == 8, long long, int>::type;
    const V *svals = (const V *)svals_;
    __shared__ K s_samp[SAMP_BYTES / sizeof(K)];
    for (int j = threadIdx.x; j < M; j += R_THREADS) s_samp[j] = samp[j];
    __syncthreads();
    const long long nrp = *d_nrp;
    for (long long i = blockIdx.x * (long long)R_THREADS + threadIdx.x; i < nrp;
         i += (long long)gridDim.x * R_THREADS) {
        const K k = rkeys[i];
        int lb = 0, ub = 0;
        if constexpr (OP == EQ || OP == NE) {
            lb = bound_sampled<true>(skeys, N, s_samp, M, stride, k);
            ub = upper_from(skeys, N, lb, k);
        } else if constexpr (OP == LE || OP == GT) {
            lb = bound_sampled<true>(skeys, N, s_samp, M, stride, k);
        } else {
            ub = bound_sampled<false>(skeys, N, s_samp, M, stride, k);
        }
        int a0, b0, a1, b1;
        pieces<OP>(lb, ub, N, a0, b0, a1, b1);
        const long long L = (long long)(b0 - a0) + (b1 - a1);
        if constexpr (AGG == COUNT || AGG == EXISTS || AGG == NOT_EXISTS) {
            cnt[i] = L;
        } else {
            if constexpr (OP == EQ && (AGG == MIN || AGG == MAX)) {
                if (pre) {   // '=' MIN/MAX: O(1) from the per-key group aggregates (pre = grp)
                    acc[i] = L ? pre[ub - 1] : (AGG == MIN ? LLONG_MAX : LLONG_MIN);
                    cnt[i] = L;
                    continue;
                }
            }
            if (pre && (AGG == SUM || OP != EQ)) {   // O(1) from the prefix / suffix aggregates
                long long a;
                if constexpr (AGG == SUM) {
                    a = (pre[b0] - pre[a0]) + (pre[b1] - pre[a1]);
                    if (pre_hi) acc_hi[i] = (pre_hi[b0] - pre_hi[a0]) + (pre_hi[b1] - pre_hi[a1]);
                } else if constexpr (OP == NE) {
                    a = AGG == MIN ? min(pre[lb], suf[ub]) : max(pre[lb], suf[ub]);
                } else if constexpr (OP == GT || OP == GE) {
                    a = pre[b0];                       // [0, b0)
                } else {
                    a = suf[a0];                       // [a0, N)
                }
                acc[i] = a;
                cnt[i] = L;
            } else if (L <= R_SHORT || N <= (int)RANGE_INLINE_MAX) {
                long long a = AGG == MIN ? LLONG_MAX : (AGG == MAX ? LLONG_MIN : 0);
                for (int s = a0; s < b0; s++) fold<AGG>(a, svals[s]);
                for (int s = a1; s < b1; s++) fold<AGG>(a, svals[s]);
                acc[i] = a;
                cnt[i] = L;
            } else {
                unsigned slot = atomicAdd(list_n, 1u);
                list[slot] = LongItem{(int)i, lb, ub, 0};
            }
        }
    }
}

template <int AGG>
__device__ __forceinline__ long long warp_reduce(long long a)
{
    for (int o = 16; o > 0; o >>= 1) {
        long long b = __shfl_xor_sync(FULL, a, o);
        if constexpr (AGG == MIN) a = min(a, b);
        else if constexpr (AGG == MAX) a = max(a, b);
        else a += b;
    }
    return a;
}

template <int VB, int OP, int AGG>
__global__ void __launch_bounds__(R_THREADS)
range_long_kernel(const void *__restrict__ svals_, int N, const LongItem *__restrict__ list,
                  const unsigned *__restrict__ list_n, long long *__restrict__ acc, long long *__restrict__ cnt)
{
    using V = typename std::conditional<VB == 8, long long, int>::type;
    const V *svals = (const V *)svals_;
    const unsigned lane = threadIdx.x & 31;
    const long long gw = (blockIdx.x * (long long)R_THREADS + threadIdx.x) >> 5;
    const long long nw = ((long long)gridDim.x * R_THREADS) >> 5;
    const long long items = *list_n;
    for (long long it = gw; it < items; it += nw) {
        const LongItem li = list[it];
        int a0, b0, a1, b1;
        pieces<OP>(li.lb, li.ub, N, a0, b0, a1, b1);
        long long a = AGG == MIN ? LLONG_MAX : (AGG == MAX ? LLONG_MIN : 0);
        for (int s = a0 + (int)lane; s < b0; s += 32) fold<AGG>(a, svals[s]);
        for (int s = a1 + (int)lane; s < b1; s += 32) fold<AGG>(a, svals[s]);
        a = warp_reduce<AGG>(a);
        if (lane == 0) {
            acc[li.r] = a;
            cnt[li.r] = (long long)(b0 - a0) + (b1 - a1);
        }
    }
}

template <typename K, int VB, int OP, int AGG>
static void launch_range_t(long long n_rp_max, const long long *d_nrp, const void *rkeys, const void *skeys,
                           const void *svals, long long ns, const long long *pre, const long long *suf,
                           long long *acc, long long *cnt, void *scratch, cudaStream_t st, long long *launches,
                           const long long *pre_hi, long long *acc_hi)
{
    unsigned *list_n = (unsigned *)scratch;
    LongItem *list = (LongItem *)((char *)scratch + 256);
    K *samp = (K *)((char *)scratch + 256 + (size_t)n_rp_max * sizeof(LongItem));
    constexpr int SMAX = SAMP_BYTES / (int)sizeof(K);
    const int N = (int)ns;
    const int stride = N > SMAX ? (N + SMAX - 1) / SMAX : 1;
    const int M = N > 0 ? (N + stride - 1) / stride : 0;
    if (stride == 1) {
        samp = (K *)skeys;   // every key fits the shared-memory sample buffer: the keys are the samples
    } else if (M > 0) {
        sample_kernel<K><<<(M + 255) / 256, 256, 0, st>>>((const K *)skeys, stride, M, samp);
        ++*launches;
    }
    int max_blocks = 148 * 8;   // persistent-ish grid: the samples are staged once per CTA
    per_device_setup((const void *)range_short_kernel<K, VB, OP, AGG>, 0, &max_blocks, [](int dev, int *v) {
        int sms = 0;
        cudaError_t e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        *v = sms * 8;
        return e;
    });
    long long blocks = (n_rp_max + R_THREADS - 1) / R_THREADS;
    if (blocks > max_blocks) blocks = max_blocks;
    range_short_kernel<K, VB, OP, AGG><<<(unsigned)blocks, R_THREADS, 0, st>>>(
        d_nrp, (const K *)rkeys, (const K *)skeys, svals, N, samp, M, stride, pre, suf, acc, cnt, list, list_n,
        pre_hi, acc_hi);
    ++*launches;
    // long ranges exist only when no range is answered in O(1) (prefix /
    // suffix / group aggregates) and the index is too large to fold inline
    if constexpr (AGG != COUNT && AGG != EXISTS && AGG != NOT_EXISTS) {
        if (!pre && ns > RANGE_INLINE_MAX) {
            range_long_kernel<VB, OP, AGG><<<148 * 8, R_THREADS, 0, st>>>(svals, (int)ns, list, list_n, acc, cnt);
            ++*launches;
        }
    }
}

template <typename K, int VB, int OP>
static void dispatch_agg(int agg, long long n_rp_max, const long long *d_nrp, const void *rkeys, const void *skeys,
                         const void *svals, long long ns, const long long *pre, const long long *suf, long long *acc,
                         long long *cnt, void *scratch, cudaStream_t st, long long *launches, const long long *pre_hi,
                         long long *acc_hi)
{
#define NG_R(A) launch_range_t<K, VB, OP, A>(n_rp_max, d_nrp, rkeys, skeys, svals, ns, pre, suf, acc, cnt, scratch, st, \
                                             launches, pre_hi, acc_hi)
    switch (agg) {
    case MIN: NG_R(MIN); break;
    case MAX: NG_R(MAX); break;
    case SUM: NG_R(SUM); break;
    case AVG: NG_R(SUM); break;   // AVG = (sum, nn)
    case COUNT: NG_R(COUNT); break;
    default: NG_R(EXISTS); break; // EXISTS / NOT EXISTS: range length
    }
#undef NG_R
}

template <typename K, int VB>
static void dispatch_op(int op, int agg, long long n_rp_max, const long long *d_nrp, const void *rkeys,
                        const void *skeys, const void *svals, long long ns, const long long *pre, const long long *suf,
                        long long *acc, long long *cnt, void *scratch, cudaStream_t st, long long *launches,
                        const long long *pre_hi, long long *acc_hi)
{
#define NG_O(O) dispatch_agg<K, VB, O>(agg, n_rp_max, d_nrp, rkeys, skeys, svals, ns, pre, suf, acc, cnt, scratch, st, \
                                       launches, pre_hi, acc_hi)
    switch (op) {
    case EQ: NG_O(EQ); break;
    case NE: NG_O(NE); break;
    case LT: NG_O(LT); break;
    case LE: NG_O(LE); break;
    case GT: NG_O(GT); break;
    default: NG_O(GE); break;
    }
#undef NG_O
}

cudaError_t launch_range_agg(int kb, int vb, int op, int agg, long long n_rp_max, const long long *d_nrp,
                             const void *rkeys, const void *skeys, const void *svals, long long ns,
                             const long long *pre, const long long *suf, long long *acc, long long *cnt,
                             void *scratch, cudaStream_t st, long long *launches, const long long *pre_hi,
                             long long *acc_hi, bool prezeroed)
{
    if (n_rp_max <= 0) return cudaSuccess;
    if (agg != SUM && agg != AVG) pre_hi = nullptr, acc_hi = nullptr;
    if (!pre_hi || !acc_hi) pre_hi = nullptr, acc_hi = nullptr;
    cudaError_t e = prezeroed ? cudaSuccess : cudaMemsetAsync(scratch, 0, 256, st);
    if (e != cudaSuccess) return e;
    const bool noval = agg == COUNT || agg == EXISTS || agg == NOT_EXISTS;
    if (kb == 4) {
        if (noval || vb == 4) dispatch_op<uint32_t, 4>(op, agg, n_rp_max, d_nrp, rkeys, skeys, svals, ns, pre, suf, acc, cnt, scratch, st, launches, pre_hi, acc_hi);
        else dispatch_op<uint32_t, 8>(op, agg, n_rp_max, d_nrp, rkeys, skeys, svals, ns, pre, suf, acc, cnt, scratch, st, launches, pre_hi, acc_hi);
    } else {
        if (noval || vb == 4) dispatch_op<uint64_t, 4>(op, agg, n_rp_max, d_nrp, rkeys, skeys, svals, ns, pre, suf, acc, cnt, scratch, st, launches, pre_hi, acc_hi);
        else dispatch_op<uint64_t, 8>(op, agg, n_rp_max, d_nrp, rkeys, skeys, svals, ns, pre, suf, acc, cnt, scratch, st, launches, pre_hi, acc_hi);
    }
    return cudaGetLastError();
}

// ------------------------------------------------------------------ index aggregates
// pre[p] = AGG(v[0..p)) for p in [0, N]; with SUF, suf[p] = AGG(v[p..N)).
// Three passes per direction: per-block aggregate, scan of the block
// aggregates (one CTA), per-block inclusive scan offset by the block prefix.
constexpr int P_THREADS = 256;
constexpr int P_ITEMS = 16;
constexpr int P_BLOCK = P_THREADS * P_ITEMS;

template <int AGG>
__device__ __forceinline__ long long comb(long long a, long long b)
{
    if constexpr (AGG == MIN) return min(a, b);
    else if constexpr (AGG == MAX) return max(a, b);
    else return a + b;
}
template <int AGG>
constexpr long long ident() { return AGG == MIN ? LLONG_MAX : (AGG == MAX ? LLONG_MIN : 0); }

// element e of the direction's sequence: forward v[e], backward v[N-1-e];
// PART 1 / 2: the low 32-bit half (unsigned) / high half (signed) of the
// value, for the split prefix sums of 64-bit payloads (exact SUM)
template <typename V, bool BACK, int PART = 0>
__device__ __forceinline__ long long elem(const V *v, long long N, long long e)
{
    const long long x = (long long)v[BACK ? N - 1 - e : e];
    if constexpr (PART == 1) return (long long)(unsigned long long)(unsigned)x;
    else if constexpr (PART == 2) return x >> 32;
    else return x;
}

template <typename V, int AGG, bool BACK, int PART>
__global__ void __launch_bounds__(P_THREADS) block_agg_kernel(const V *__restrict__ v, long long N,
                                                              long long *__restrict__ bagg)
{
    __shared__ long long s_w[P_THREADS / 32];
    const long long b0 = blockIdx.x * (long long)P_BLOCK;
    long long a = ident<AGG>();
    for (int j = 0; j < P_ITEMS; j++) {
        const long long e = b0 + (long long)j * P_THREADS + threadIdx.x;
        if (e < N) a = comb<AGG>(a, elem<V, BACK, PART>(v, N, e));
    }
    for (int o = 16; o > 0; o >>= 1) a = comb<AGG>(a, __shfl_xor_sync(FULL, a, o));
    if ((threadIdx.x & 31) == 0) s_w[threadIdx.x >> 5] = a;
    __syncthreads();
    if (threadIdx.x == 0) {
        long long t = ident<AGG>();
        for (int w = 0; w < P_THREADS / 32; w++) t = comb<AGG>(t, s_w[w]);
        bagg[blockIdx.x] = t;
    }
}

template <int AGG>
__global__ void __launch_bounds__(1024) block_scan_kernel(long long *__restrict__ bagg, long long nb)
{
    // exclusive scan, one CTA, sequential chunks of 1024
    __shared__ long long s_carry;
    __shared__ long long s_w[32];
    if (threadIdx.x == 0) s_carry = ident<AGG>();
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (long long base = 0; base < nb; base += 1024) {
        const long long i = base + threadIdx.x;
        const long long x = i < nb ? bagg[i] : ident<AGG>();
        long long incl = x;
        for (int o = 1; o < 32; o <<= 1) {
            const long long y = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl = comb<AGG>(incl, y);
        }
        if (lane == 31) s_w[warp] = incl;
        __syncthreads();
        long long wpre = ident<AGG>();
        for (int w = 0; w < warp; w++) wpre = comb<AGG>(wpre, s_w[w]);
        const long long carry = s_carry;
        const long long up = __shfl_up_sync(FULL, incl, 1);
        const long long ex_in_chunk = comb<AGG>(wpre, lane ? up : ident<AGG>());
        __syncthreads();
        if (i < nb) bagg[i] = comb<AGG>(carry, ex_in_chunk);
        if (threadIdx.x == 1023) s_carry = comb<AGG>(carry, comb<AGG>(wpre, incl));
        __syncthreads();
    }
}

template <typename V, int AGG, bool BACK, int PART>
__global__ void __launch_bounds__(P_THREADS) block_prefix_kernel(const V *__restrict__ v, long long N,
                                                                 const long long *__restrict__ bpre,
                                                                 long long *__restrict__ out)
{
    // out has N+1 entries: forward out[e+1] = AGG(v[0..e]); backward
    // out[N-1-e] = AGG(v[N-1-e..N)); the identity entry is written by block 0.
    // The block's rows come in by coalesced loads into shared memory (one
    // padding word per P_ITEMS), each thread scans P_ITEMS consecutive rows in
    // registers, one block scan of the thread totals, and the results leave
    // through shared memory by coalesced stores (round 2, session 2: was 16
    // barrier-separated steps of 256 rows)
    constexpr int PAD = P_ITEMS + 1;
    __shared__ long long s_x[P_THREADS * PAD];
    __shared__ long long s_w[P_THREADS / 32];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const long long b0 = blockIdx.x * (long long)P_BLOCK;
    if (blockIdx.x == 0 && tid == 0) out[BACK ? N : 0] = ident<AGG>();
#pragma unroll
    for (int j = 0; j < P_ITEMS; j++) {
        const int q = j * P_THREADS + tid;   // block-local row, coalesced
        const long long e = b0 + q;
        s_x[(q / P_ITEMS) * PAD + q % P_ITEMS] = e < N ? elem<V, BACK, PART>(v, N, e) : ident<AGG>();
    }
    __syncthreads();
    long long xs[P_ITEMS];
#pragma unroll
    for (int j = 0; j < P_ITEMS; j++) xs[j] = s_x[tid * PAD + j];
#pragma unroll
    for (int j = 1; j < P_ITEMS; j++) xs[j] = comb<AGG>(xs[j - 1], xs[j]);
    long long incl = xs[P_ITEMS - 1];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const long long y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl = comb<AGG>(y, incl);
    }
    if (lane == 31) s_w[warp] = incl;
    __syncthreads();
    long long pre = bpre[blockIdx.x];
    for (int w = 0; w < warp; w++) pre = comb<AGG>(pre, s_w[w]);
    const long long up = __shfl_up_sync(FULL, incl, 1);
    if (lane) pre = comb<AGG>(pre, up);
#pragma unroll
    for (int j = 0; j < P_ITEMS; j++) s_x[tid * PAD + j] = comb<AGG>(pre, xs[j]);
    __syncthreads();
#pragma unroll
    for (int j = 0; j < P_ITEMS; j++) {
        const int q = j * P_THREADS + tid;
        const long long e = b0 + q;
        if (e < N) out[BACK ? N - 1 - e : e + 1] = s_x[(q / P_ITEMS) * PAD + q % P_ITEMS];
    }
}

template <typename V, int AGG, bool BACK, int PART = 0>
static void scan_dir(const void *v, long long N, long long *out, long long *bagg, cudaStream_t st, long long *launches)
{
    const long long nb = (N + P_BLOCK - 1) / P_BLOCK;
    block_agg_kernel<V, AGG, BACK, PART><<<(unsigned)nb, P_THREADS, 0, st>>>((const V *)v, N, bagg);
    block_scan_kernel<AGG><<<1, 1024, 0, st>>>(bagg, nb);
    block_prefix_kernel<V, AGG, BACK, PART><<<(unsigned)nb, P_THREADS, 0, st>>>((const V *)v, N, bagg, out);
    *launches += 3;
}

size_t index_aux_scratch_bytes(long long n) { return (size_t)((n + 1024 - 1) / 1024 + 1) * 16; }

// ---- per-key group aggregates: segmented inclusive scan over the sorted
// index, segments = runs of equal keys.  Pairs (f, v): f = a run starts in
// the span, v = AGG since the span's last run start; combine(earlier, later)
// = (f_e | f_l, f_l ? v_l : AGG(v_e, v_l)) -- associative, applied in order.
template <int AGG>
struct SegPair {
    long long v;
    int f;
};
template <int AGG>
__device__ __forceinline__ SegPair<AGG> seg_comb(SegPair<AGG> e, SegPair<AGG> l)
{
    return SegPair<AGG>{l.f ? l.v : comb<AGG>(e.v, l.v), e.f | l.f};
}
template <int AGG>
__device__ __forceinline__ SegPair<AGG> warp_seg_scan(SegPair<AGG> x, int lane)
{
    for (int o = 1; o < 32; o <<= 1) {
        SegPair<AGG> y{__shfl_up_sync(FULL, x.v, o), __shfl_up_sync(FULL, x.f, o)};
        if (lane >= o) x = seg_comb<AGG>(y, x);
    }
    return x;
}

// Single pass (round 2, session 2): one launch instead of block totals +
// one-CTA scan + rewrite.  CTA b (dynamic id, so its predecessors run)
// scans its 4096 rows (16 consecutive per thread, a sequential segmented
// scan, then a block scan of the thread totals), publishes its block pair
// (f, v) at once, and thread 0 walks back over the predecessors' published
// pairs until one is an inclusive prefix or holds a run start (f = 1:
// nothing before it reaches this block) -- for short runs the walk is one
// step.  status[b]: 0 = not yet, 1 = block pair, 2 = inclusive; bit 2 = f.
constexpr int SG_ITEMS = 16;
constexpr int SG_BLOCK = P_THREADS * SG_ITEMS;
template <typename K, typename V, int AGG>
__global__ void __launch_bounds__(P_THREADS) seg_onepass_kernel(const K *__restrict__ keys, const V *__restrict__ v,
                                                                long long N, long long *__restrict__ grp,
                                                                unsigned *__restrict__ status,
                                                                long long *__restrict__ sagg,
                                                                long long *__restrict__ sinc,
                                                                unsigned *__restrict__ counter)
{
    __shared__ long long s_wv[P_THREADS / 32];
    __shared__ int s_wf[P_THREADS / 32];
    __shared__ SegPair<AGG> s_carry;
    __shared__ long long s_b;
    __shared__ int s_head0;
    __shared__ SegPair<AGG> s_blk;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) s_b = atomicAdd(counter, 1u);
    __syncthreads();
    const long long b = s_b;
    const long long e0 = b * SG_BLOCK + (long long)tid * SG_ITEMS;
    // the block's rows enter through shared memory (coalesced loads, one
    // padding slot per SG_ITEMS) as (payload, run-start flag) pairs
    constexpr int SPAD = SG_ITEMS + 1;
    __shared__ long long s_xv[P_THREADS * SPAD];
    __shared__ unsigned char s_xf[P_THREADS * SPAD];
#pragma unroll
    for (int j = 0; j < SG_ITEMS; j++) {
        const int q = j * P_THREADS + tid;
        const long long e = b * SG_BLOCK + q;
        const int slot = (q / SG_ITEMS) * SPAD + q % SG_ITEMS;
        if (e < N) {
            s_xv[slot] = (long long)v[e];
            s_xf[slot] = (e == 0 || keys[e] != keys[e - 1]) ? 1 : 0;
        } else {
            s_xv[slot] = ident<AGG>();
            s_xf[slot] = 0;
        }
    }
    __syncthreads();
    // this thread's 16 consecutive rows: sequential segmented inclusive scan
    SegPair<AGG> x[SG_ITEMS];
#pragma unroll
    for (int i = 0; i < SG_ITEMS; i++) x[i] = SegPair<AGG>{s_xv[tid * SPAD + i], (int)s_xf[tid * SPAD + i]};
    if (tid == 0) s_head0 = x[0].f;
#pragma unroll
    for (int i = 1; i < SG_ITEMS; i++) x[i] = seg_comb<AGG>(x[i - 1], x[i]);
    // block exclusive scan of the thread totals
    const SegPair<AGG> tot = x[SG_ITEMS - 1];
    const SegPair<AGG> incl = warp_seg_scan<AGG>(tot, lane);
    if (lane == 31) {
        s_wv[warp] = incl.v;
        s_wf[warp] = incl.f;
    }
    __syncthreads();
    SegPair<AGG> wpre{ident<AGG>(), 0};
    for (int w = 0; w < warp; w++) wpre = seg_comb<AGG>(wpre, SegPair<AGG>{s_wv[w], s_wf[w]});
    SegPair<AGG> up{__shfl_up_sync(FULL, incl.v, 1), __shfl_up_sync(FULL, incl.f, 1)};
    if (lane == 0) up = SegPair<AGG>{ident<AGG>(), 0};
    const SegPair<AGG> tex = seg_comb<AGG>(wpre, up);   // the block's rows before this thread's
    if (tid == P_THREADS - 1) s_blk = seg_comb<AGG>(tex, tot);   // the whole block
    __syncthreads();
    if (warp == 0) {
        const SegPair<AGG> blk = s_blk;
        if (lane == 0) {
            if (b == 0 || blk.f) {   // the block's inclusive pair does not depend on its predecessors
                sinc[b] = blk.v;
                __threadfence();
                st_relaxed_u32(status + b, 2u | ((unsigned)blk.f << 2));
            } else {
                sagg[b] = blk.v;
                __threadfence();
                st_relaxed_u32(status + b, 1u);
            }
        }
        SegPair<AGG> carry{ident<AGG>(), 0};
        if (b > 0 && !s_head0) {   // rows before the block's first run start take the carry
            // 32 predecessors per round (lane l: block top - l); the walk stops
            // at the nearest one that is inclusive or holds a run start
            for (long long top = b - 1; top >= 0; top -= 32) {
                const long long p = top - lane;
                unsigned st = 2u;
                long long pv = ident<AGG>();
                if (p >= 0) {
                    while (((st = ld_relaxed_u32(status + p)) & 3u) == 0) {
                    }
                    __threadfence();
                    pv = (st & 3u) == 2u ? ld_relaxed_u64((const unsigned long long *)(sinc + p))
                                         : ld_relaxed_u64((const unsigned long long *)(sagg + p));
                }
                const int pf = (int)((st >> 2) & 1u);
                const unsigned stopm = __ballot_sync(FULL, (st & 3u) == 2u || pf);
                const int stop = stopm ? __ffs(stopm) - 1 : 31;
                // in order: pair[stop] (farthest) ... pair[0] (nearest), then carry
                SegPair<AGG> w{ident<AGG>(), 0};
                for (int l = stop; l >= 0; l--) {
                    const SegPair<AGG> q{__shfl_sync(FULL, pv, l), __shfl_sync(FULL, pf, l)};
                    w = seg_comb<AGG>(w, q);
                }
                carry = seg_comb<AGG>(w, carry);
                if (stopm) break;
            }
            if (lane == 0 && !blk.f) {
                sinc[b] = seg_comb<AGG>(carry, blk).v;
                __threadfence();
                st_relaxed_u32(status + b, 2u);
            }
        }
        if (lane == 0) s_carry = carry;
    }
    __syncthreads();
    const SegPair<AGG> pre = seg_comb<AGG>(s_carry, tex);
#pragma unroll
    for (int i = 0; i < SG_ITEMS; i++) s_xv[tid * SPAD + i] = seg_comb<AGG>(pre, x[i]).v;
    __syncthreads();
#pragma unroll
    for (int j = 0; j < SG_ITEMS; j++) {   // and leave the same way (coalesced stores)
        const int q = j * P_THREADS + tid;
        const long long e = b * SG_BLOCK + q;
        if (e < N) grp[e] = s_xv[(q / SG_ITEMS) * SPAD + q % SG_ITEMS];
    }
    (void)e0;
}

template <typename K, typename V, int AGG>
static void seg_scan(const void *keys, const void *v, long long N, long long *grp, void *scratch, cudaStream_t st,
                     long long *launches)
{
    const long long nb = (N + SG_BLOCK - 1) / SG_BLOCK;
    unsigned *counter = (unsigned *)scratch;
    unsigned *status = counter + 1;
    const size_t zb = ((size_t)(nb + 1) * 4 + 15) & ~(size_t)15;
    long long *sagg = (long long *)((char *)scratch + zb);
    long long *sinc = sagg + nb;
    cudaMemsetAsync(scratch, 0, zb, st);
    seg_onepass_kernel<K, V, AGG><<<(unsigned)nb, P_THREADS, 0, st>>>((const K *)keys, (const V *)v, N, grp, status,
                                                                       sagg, sinc, counter);
    *launches += 1;
}

cudaError_t launch_index_group_agg(int agg, int kb, int vb, const void *keys, const void *payload, long long n,
                                   long long *grp, void *scratch, cudaStream_t st, long long *launches)
{
    if (n <= 0) return cudaSuccess;
#define NG_SEG(K_, V_)                                                                             \
    if (agg == MIN) seg_scan<K_, V_, MIN>(keys, payload, n, grp, scratch, st, launches);           \
    else seg_scan<K_, V_, MAX>(keys, payload, n, grp, scratch, st, launches);
    if (kb == 4) {
        if (vb == 8) { NG_SEG(uint32_t, long long) } else { NG_SEG(uint32_t, int) }
    } else {
        if (vb == 8) { NG_SEG(uint64_t, long long) } else { NG_SEG(uint64_t, int) }
    }
#undef NG_SEG
    return cudaGetLastError();
}

cudaError_t launch_index_aux(int agg, int vb, const void *payload, long long n, long long *pre, long long *suf,
                             void *scratch, cudaStream_t st, long long *launches, long long *pre_hi)
{
    if (n <= 0) {
        const long long id = agg == MIN ? LLONG_MAX : (agg == MAX ? LLONG_MIN : 0);
        cudaError_t e = cudaMemcpyAsync(pre, &id, 8, cudaMemcpyHostToDevice, st);
        if (e == cudaSuccess && suf) e = cudaMemcpyAsync(suf, &id, 8, cudaMemcpyHostToDevice, st);
        if (e == cudaSuccess && pre_hi) e = cudaMemcpyAsync(pre_hi, &id, 8, cudaMemcpyHostToDevice, st);
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);   // &id is a host stack value
        return e;
    }
    long long *bagg = (long long *)scratch;
    if (agg == SUM && pre_hi && vb == 8) {   // exact split prefix sums (no int64 wrap anywhere)
        scan_dir<long long, SUM, false, 1>(payload, n, pre, bagg, st, launches);
        scan_dir<long long, SUM, false, 2>(payload, n, pre_hi, bagg, st, launches);
        return cudaGetLastError();
    }
#define NG_SCAN(V_)                                                                               \
    if (agg == MIN) {                                                                             \
        scan_dir<V_, MIN, false>(payload, n, pre, bagg, st, launches);                            \
        scan_dir<V_, MIN, true>(payload, n, suf, bagg, st, launches);                             \
    } else if (agg == MAX) {                                                                      \
        scan_dir<V_, MAX, false>(payload, n, pre, bagg, st, launches);                            \
        scan_dir<V_, MAX, true>(payload, n, suf, bagg, st, launches);                             \
    } else {                                                                                      \
        scan_dir<V_, SUM, false>(payload, n, pre, bagg, st, launches);                            \
    }
    if (vb == 8) { NG_SCAN(long long) } else { NG_SCAN(int) }
#undef NG_SCAN
    return cudaGetLastError();
}

}  // namespace ng
