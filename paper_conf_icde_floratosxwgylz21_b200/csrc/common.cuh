// common.cuh -- device-side helpers shared by the nestgpu kernels (sm_100a).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace ng {

constexpr int MAX_PREDS = 8;
constexpr unsigned FULL = 0xffffffffu;

enum Op : int { EQ = 0, NE = 1, LT = 2, LE = 3, GT = 4, GE = 5 };
enum Agg : int { MIN = 0, MAX = 1, SUM = 2, COUNT = 3, AVG = 4, EXISTS = 5, NOT_EXISTS = 6 };

// One local predicate ("Selection(op, col, value)"), col OP literal or
// col OP col; widths 4 or 8 bytes (int32 / int64 storage).
struct DevPred {
    const void *col;
    const uint8_t *valid;
    const void *rhs;
    const uint8_t *rhs_valid;
    long long lit;
    int op;
    int w;
    int rhs_w;
    int pad_;
};
struct PredSet {
    int n;
    DevPred p[MAX_PREDS];
};

// Source of the correlated key: one column (int32 or int64 storage) or two
// int32-storage columns packed into an order-preserving 64-bit code
// (reading R9).
struct KeySrc {
    const void *c0;
    const uint8_t *v0;
    const void *c1;
    const uint8_t *v1;
    int w0;      // 4 or 8
    int n_key;   // 1 or 2
};

struct ValSrc {
    const void *c;     // nullptr: no payload
    const uint8_t *v;  // validity (nullptr: NOT NULL)
    int w;             // 4 or 8
};

__device__ __forceinline__ long long load_w(const void *c, int w, long long i)
{
    return w == 4 ? (long long)__ldg((const int *)c + i) : __ldg((const long long *)c + i);
}

template <typename T>
__device__ __forceinline__ bool cmp_rt(T x, int op, T y)
{
    switch (op) {
    case EQ: return x == y;
    case NE: return x != y;
    case LT: return x < y;
    case LE: return x <= y;
    case GT: return x > y;
    default: return x >= y;
    }
}

// Compile-time operator: outer.key OP inner.key (reading R8).
template <int OP, typename T>
__device__ __forceinline__ bool cmp_ct(T x, T y)
{
    if constexpr (OP == EQ) return x == y;
    else if constexpr (OP == NE) return x != y;
    else if constexpr (OP == LT) return x < y;
    else if constexpr (OP == LE) return x <= y;
    else if constexpr (OP == GT) return x > y;
    else return x >= y;
}

// Order-preserving unsigned encodings of signed keys.
__device__ __forceinline__ uint32_t enc32(int32_t k) { return (uint32_t)k ^ 0x80000000u; }
__device__ __forceinline__ uint64_t enc64(long long k) { return (uint64_t)k ^ 0x8000000000000000ull; }

__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ unsigned lanemask_lt()
{
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

// Device-scope relaxed loads/stores for decoupled look-back status words.
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long *p)
{
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_u64(unsigned long long *p, unsigned long long v)
{
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned ld_relaxed_u32(const unsigned *p)
{
    unsigned v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_u32(unsigned *p, unsigned v)
{
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// ---------------------------------------------------------------------------
// Single-pass ordered compaction offsets with decoupled look-back (the
// paper's "0-1 vector -> prefix-sum -> materialize", fused into one
// pass).  Status word: bits 62-63 flag (1 = aggregate, 2 = inclusive), low 62
// bits the count.  `status` must be zeroed before the launch.
constexpr unsigned long long ST_AGG = 1ull << 62;
constexpr unsigned long long ST_INC = 2ull << 62;
constexpr unsigned long long ST_VAL = (1ull << 62) - 1;

// ---------------------------------------------------------------------------
// mbarrier + bulk-copy (TMA bulk engine, SASS UBLKCP / SYNCS) helpers.
__device__ __forceinline__ void mbar_init(unsigned long long *bar, unsigned count)
{
    unsigned a = (unsigned)__cvta_generic_to_shared(bar);
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long *bar, unsigned parity)
{
    unsigned a = (unsigned)__cvta_generic_to_shared(bar);
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "NG_WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra NG_WAIT_%=;\n}" ::"r"(a),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(unsigned long long *bar, unsigned bytes)
{
    unsigned a = (unsigned)__cvta_generic_to_shared(bar);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(a), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, unsigned bytes, unsigned long long *bar)
{
    unsigned d = (unsigned)__cvta_generic_to_shared(dst);
    unsigned b = (unsigned)__cvta_generic_to_shared(bar);
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(d),
        "l"(src), "r"(bytes), "r"(b)
        : "memory");
}

}  // namespace ng
