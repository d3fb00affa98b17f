// api.cpp -- the C ABI (include/nestgpu.h): context, memory pool, columnar
// store, index build, plan validation and the exec pipeline.
//
// Pipeline of nestgpu_exec_correlated (one stream, no device allocation, one
// host synchronisation at the end):
//   a2  filter_kernel(R, outer preds)        -> R' ids + encoded keys
//   a3  filter_kernel(S, inner preds)        -> S' (key, payload)   [BNL path]
//       or the index built by nestgpu_build_index (a3 + a4, once)   [index path]
//   a5+a6 range_short/long kernels            -> per-R' partials     [index path]
//   a7  bnl_kernel                            -> per-R' partials     [BNL path]
//   a8+a9 finalize_kernel                     -> compacted result
//   D2H of the survivor count.
#include <cuda_runtime.h>

#include <algorithm>
#include <climits>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <tuple>
#include <unordered_map>
#include <chrono>
#include <cstdlib>
#include <utility>
#include <vector>

#include "../../include/nestgpu.h"
#include "internal.h"

namespace {

struct Column {
    nestgpu_dtype dtype;
    int32_t scale;
    int64_t n;
    void *d;
    uint8_t *valid;
    size_t off;
    bool alive;
    bool stats;         // host-side min/max known
    long long mn, mx;
    bool sorted;        // (with stats) NOT NULL and stored in ascending key order
    long long band, bor;   // (with stats) AND / OR of the non-NULL (sign-extended) values
    bool caller_filled; // nestgpu_alloc_column: contents may change behind our back (stats not cached)
};

struct IndexRec {
    bool alive;
    size_t off;
    int64_t n;
    int kb, vb;
    void *keys;
    void *payload;
    long long *d_n;     // device copy of n
    int32_t key_cols[2];
    int n_key;
    int32_t payload_col;
    std::vector<nestgpu_pred> inner;
    bool payload_nullable;
    // index-pruned evaluation (NEXT 3): prefix / suffix aggregates of the
    // payload per kind (0 MIN, 1 MAX, 2 SUM, 3 split SUM: pre = low halves,
    // suf = high halves; 4 / 5: per-key group MIN / MAX for '='), built on
    // first use
    long long *aux_pre[6];
    long long *aux_suf[6];
    size_t aux_off[6];
};

constexpr int PIN_WORDS = 8 * 256 + 64;
// Pinned staging for small results: exec copies the first rows of every
// result field into it before its one synchronisation, so a result of at
// most that many rows reaches the host with no further GPU operation.
constexpr size_t STAGE_BYTES = 256 << 10;
// Inputs this small take the latency-oriented shortcuts (fewer launches):
// partial-aggregate init folded into the exec's fill kernel, the whole
// index-build scratch zeroed by one fill before the S' filter.
constexpr long long SMALL_ROWS = 1 << 16;
constexpr size_t ALIGN = 256;

}  // namespace

struct nestgpu_ctx {
    int device;
    char *base;
    size_t size;
    size_t lo;     // persistent tail (grows up)
    size_t hi;     // scratch head (grows down from size)
    size_t peak;
    cudaStream_t stream;
    std::string err;
    long long launches;
    int num_sms;
    std::vector<Column> cols;
    std::vector<IndexRec> idx;
    unsigned *pinned;  // host pinned words for small D2H / H2D
    char *stage;       // STAGE_BYTES of pinned host memory (results staged by exec)
    struct {
        bool ok;
        const void *ids;        // d_row_ids of the staged result
        long long rows;         // rows staged per field
        size_t w8;              // 8-byte fields in the block (2, or 4 with AVG)
    } staged;
    bool profiling;
    // Ablation knob (NESTGPU_OPT_MALLOC_SCRATCH): scratch comes from
    // cudaMalloc per allocation, freed at the next scratch reset -- the
    // pool-less baseline of P:147 / P:233.  Off by default.
    bool malloc_scratch;
    std::vector<void *> mallocs;
    int bnl_shape;   // NESTGPU_OPT_BNL_SHAPE (test knob): 0 automatic, 1 full, 2 warp-split
    int sort_mode;   // NESTGPU_OPT_SORT: 0 / 1 LSD onesweep, 2 MSD bucket sort (experiment)
    bool tiny_on;    // NESTGPU_OPT_TINY: one-launch path for tiny nested-loop queries (default on)
    cudaEvent_t ev[NESTGPU_N_STAGES][2];
    // CUDA graphs of exec launch sequences (NESTGPU_OPT_GRAPHS, default on):
    // key = every argument that determines the sequence (plan, column /
    // index addresses and sizes, arena state); kernels = launches per replay
    // (0 with no exec: seen `seen` times, captured once it keeps repeating;
    // -1: the sequence could not be captured, run it directly)
    struct GraphEntry {
        cudaGraphExec_t exec;
        long long kernels;
        int seen;   // direct runs so far
    };
    bool graphs_on;
    std::unordered_map<std::string, GraphEntry> graphs;
    cudaStream_t cap_stream;   // private stream the sequences are captured on
    // NESTGPU_TRACE=1 (diagnostics): host time of each step of an exec,
    // printed to stderr when the exec returns
    bool trace;
    std::chrono::steady_clock::time_point t0, tl;
    std::string tlog;
    bool ran[NESTGPU_N_STAGES];
};

namespace {

nestgpu_status fail(nestgpu_ctx *c, nestgpu_status code, const char *fmt, ...)
{
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    if (c) c->err = buf;
    return code;
}

#define CUDA_TRY(ctx, expr)                                                                         \
    do {                                                                                            \
        cudaError_t e_ = (expr);                                                                    \
        if (e_ != cudaSuccess)                                                                      \
            return fail(ctx, NESTGPU_ERR_CUDA, "%s: %s (%s:%d)", #expr, cudaGetErrorString(e_),     \
                        __FILE__, __LINE__);                                                        \
    } while (0)

// Radix-pass plan for n encoded keys of kb bytes whose AND / OR over all keys
// are kand / kor: only bits that vary need sorting, so w-bit digit windows
// are placed greedily from the lowest varying bit (the fewest windows that
// cover every varying bit), e.g. keys that are multiples of 32 below 2^26
// take 3 passes of 8 bits instead of 4.  9-bit windows (512 bins) are used
// when they need at most 2/3 of the 8-bit passes (an 18-bit key: 2 instead
// of 3; a 9-bit pass measured 1.3-1.4x an 8-bit one, so 4 -> 3 does not pay).  When every varying bit lies in the low word of a 64-bit key the
// windows stay inside bits 0-31 (start <= 32 - w; overlapping a lower window
// is harmless for a stable LSD sort), so the passes can run on 32-bit keys.
// Returns the number of passes; shifts[] their bit offsets, *rb the width.
static int plan_windows(int kb, unsigned long long var, int w, int *shifts)
{
    const bool low = (var >> 32) == 0;
    int np = 0;
    for (int b = 0; b < kb * 8 && np < 8;) {
        if (!((var >> b) & 1ull)) {
            b++;
            continue;
        }
        const int s = low && b > 32 - w ? 32 - w : b;
        shifts[np++] = s;
        b = s + w;
    }
    return np;
}

static int plan_sort_passes(int kb, unsigned long long kand, unsigned long long kor, long long n, int *shifts,
                            int *rb)
{
    *rb = 8;
    if (n < 2) return 0;
    const unsigned long long var = kand ^ kor;
    int s9[8];
    const int np8 = plan_windows(kb, var, 8, shifts);
    const int np9 = plan_windows(kb, var, 9, s9);
    if (3 * np9 <= 2 * np8) {   // a 9-bit pass costs ~1.3-1.4x an 8-bit one (measured): 3 -> 2 pays, 4 -> 3 not
        for (int p = 0; p < np9; p++) shifts[p] = s9[p];
        *rb = 9;
        return np9;
    }
    return np8;
}

size_t align_up(size_t x) { return (x + ALIGN - 1) / ALIGN * ALIGN; }

// Column / index ids are slots that are reused once their object died
// (release / drop): a loop of load -> query -> release keeps the id set and
// the host tables bounded, and a re-built object gets its old id back.
template <typename T>
int32_t put_slot(std::vector<T> &v, const T &x)
{
    for (size_t i = 0; i < v.size(); i++)
        if (!v[i].alive) {
            v[i] = x;
            return (int32_t)i;
        }
    v.push_back(x);
    return (int32_t)v.size() - 1;
}

// Start a new scratch generation: everything salloc'd before dies here.
void scratch_reset(nestgpu_ctx *c)
{
    c->hi = c->size;
    c->staged.ok = false;
    if (!c->mallocs.empty()) {
        cudaStreamSynchronize(c->stream);
        for (void *p : c->mallocs) cudaFree(p);
        c->mallocs.clear();
    }
}

void *palloc(nestgpu_ctx *c, size_t bytes)
{
    size_t b = align_up(bytes + 16);  // +16: bulk copies / vector loads may read a ragged tail
    if (c->lo + b > c->hi) return nullptr;
    void *p = c->base + c->lo;
    c->lo += b;
    size_t used = c->lo + (c->size - c->hi);
    if (used > c->peak) c->peak = used;
    return p;
}

void *salloc(nestgpu_ctx *c, size_t bytes)
{
    size_t b = align_up(bytes + 16);
    if (c->malloc_scratch) {
        void *p = nullptr;
        if (cudaMalloc(&p, b) != cudaSuccess) return nullptr;
        c->mallocs.push_back(p);
        return p;
    }
    if (c->hi < c->lo + b) return nullptr;
    c->hi -= b;
    size_t used = c->lo + (c->size - c->hi);
    if (used > c->peak) c->peak = used;
    return c->base + c->hi;
}

int dtype_width(nestgpu_dtype t)
{
    switch (t) {
    case NG_INT32: case NG_DATE: case NG_DECIMAL32: return 4;
    case NG_INT64: case NG_DECIMAL: return 8;
    }
    return 0;
}

bool valid_op(int op) { return op >= NG_EQ && op <= NG_GE; }

const Column *col_get(const nestgpu_ctx *c, int32_t id)
{
    if (id < 0 || id >= (int32_t)c->cols.size() || !c->cols[id].alive) return nullptr;
    return &c->cols[id];
}

// Build the device predicate set for a conjunction over a relation of n rows.
nestgpu_status make_preds(nestgpu_ctx *c, const nestgpu_pred *p, int32_t np, int64_t n, ng::PredSet &out,
                          const char *what)
{
    if (np < 0 || np > ng::MAX_PREDS) return fail(c, NESTGPU_ERR_UNSUPPORTED, "%s: at most %d predicates", what, ng::MAX_PREDS);
    if (np > 0 && !p) return fail(c, NESTGPU_ERR_INVALID, "%s: null predicate array", what);
    memset(&out, 0, sizeof out);
    out.n = np;
    for (int k = 0; k < np; k++) {
        const Column *a = col_get(c, p[k].col);
        if (!a) return fail(c, NESTGPU_ERR_INVALID, "%s[%d]: unknown column %d", what, k, p[k].col);
        if (a->n != n) return fail(c, NESTGPU_ERR_INVALID, "%s[%d]: column %d has %lld rows, relation has %lld", what, k, p[k].col, (long long)a->n, (long long)n);
        if (!valid_op(p[k].op)) return fail(c, NESTGPU_ERR_INVALID, "%s[%d]: bad operator", what, k);
        ng::DevPred &d = out.p[k];
        d.col = a->d;
        d.valid = a->valid;
        d.w = dtype_width(a->dtype);
        d.op = p[k].op;
        d.lit = p[k].literal;
        if (p[k].rhs_col >= 0) {
            const Column *b = col_get(c, p[k].rhs_col);
            if (!b) return fail(c, NESTGPU_ERR_INVALID, "%s[%d]: unknown rhs column %d", what, k, p[k].rhs_col);
            if (b->n != n) return fail(c, NESTGPU_ERR_INVALID, "%s[%d]: rhs column row count differs", what, k);
            d.rhs = b->d;
            d.rhs_valid = b->valid;
            d.rhs_w = dtype_width(b->dtype);
        }
    }
    return NESTGPU_OK;
}

bool same_preds(const nestgpu_pred *a, int32_t na, const std::vector<nestgpu_pred> &b)
{
    if ((size_t)na != b.size()) return false;
    for (int i = 0; i < na; i++)
        if (a[i].col != b[i].col || a[i].op != b[i].op || a[i].rhs_col != b[i].rhs_col ||
            (a[i].rhs_col < 0 && a[i].literal != b[i].literal))
            return false;
    return true;
}

// Key source: one column, or two int32-storage columns (composite '=').
nestgpu_status make_key(nestgpu_ctx *c, const int32_t *cols, int32_t nk, int64_t &n, ng::KeySrc &ks, const char *what)
{
    if (nk != 1 && nk != 2) return fail(c, NESTGPU_ERR_INVALID, "%s: 1 or 2 key columns", what);
    const Column *a = col_get(c, cols[0]);
    if (!a) return fail(c, NESTGPU_ERR_INVALID, "%s: unknown key column %d", what, cols[0]);
    memset(&ks, 0, sizeof ks);
    ks.c0 = a->d;
    ks.v0 = a->valid;
    ks.w0 = dtype_width(a->dtype);
    ks.n_key = nk;
    n = a->n;
    if (nk == 2) {
        const Column *b = col_get(c, cols[1]);
        if (!b) return fail(c, NESTGPU_ERR_INVALID, "%s: unknown key column %d", what, cols[1]);
        if (b->n != n) return fail(c, NESTGPU_ERR_INVALID, "%s: key columns differ in row count", what);
        if (dtype_width(a->dtype) != 4 || dtype_width(b->dtype) != 4)
            return fail(c, NESTGPU_ERR_UNSUPPORTED, "%s: composite keys need int32-storage columns", what);
        ks.c1 = b->d;
        ks.v1 = b->valid;
    }
    return NESTGPU_OK;
}

int key_bytes(const nestgpu_ctx *c, const int32_t *cols, int32_t nk)
{
    return (nk == 1 && dtype_width(c->cols[cols[0]].dtype) == 4) ? 4 : 8;
}

void htrace(nestgpu_ctx *c, const char *what)
{
    if (!c->trace) return;
    const auto now = std::chrono::steady_clock::now();
    char buf[64];
    snprintf(buf, sizeof buf, " %s=%.1f", what, std::chrono::duration<double, std::micro>(now - c->tl).count());
    c->tlog += buf;
    c->tl = now;
}
void htrace_begin(nestgpu_ctx *c)
{
    if (!c->trace) return;
    c->t0 = c->tl = std::chrono::steady_clock::now();
    c->tlog.clear();
}
void htrace_end(nestgpu_ctx *c, const char *call)
{
    if (!c->trace) return;
    htrace(c, "tail");
    fprintf(stderr, "[nestgpu trace] %s total=%.1f us:%s\n", call,
            std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - c->t0).count(), c->tlog.c_str());
}

void prof_begin(nestgpu_ctx *c, int s)
{
    if (c->profiling) {
        cudaEventRecord(c->ev[s][0], c->stream);
        c->ran[s] = true;
    }
}
void prof_end(nestgpu_ctx *c, int s)
{
    if (c->profiling) cudaEventRecord(c->ev[s][1], c->stream);
}

// Host-side min/max of a column (lazily, one small D2H) for the SUM/AVG
// overflow pre-check (reading R5).
nestgpu_status column_stats(nestgpu_ctx *c, Column &col);

}  // namespace

namespace ng {
cudaError_t launch_minmax(const void *col, int w, const uint8_t *valid, long long n, long long *out2, cudaStream_t st,
                          long long *launches);
}

namespace {
nestgpu_status column_stats(nestgpu_ctx *c, Column &col)
{
    if (col.stats) return NESTGPU_OK;
    long long *d = (long long *)salloc(c, 40);
    if (!d) return fail(c, NESTGPU_ERR_OOM, "arena exhausted (stats)");
    CUDA_TRY(c, ng::launch_minmax(col.d, dtype_width(col.dtype), col.valid, col.n, d, c->stream, &c->launches));
    CUDA_TRY(c, cudaMemcpyAsync(c->pinned, d, 40, cudaMemcpyDeviceToHost, c->stream));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    long long desc;
    memcpy(&col.mn, c->pinned, 8);
    memcpy(&col.mx, (char *)c->pinned + 8, 8);
    memcpy(&desc, (char *)c->pinned + 16, 8);
    memcpy(&col.band, (char *)c->pinned + 24, 8);
    memcpy(&col.bor, (char *)c->pinned + 32, 8);
    col.sorted = !col.valid && desc == 0;
    col.stats = true;
    return NESTGPU_OK;
}
}  // namespace

// Context accessors for the host-side modules (cost.cpp) -- internal.h.
namespace ng {
namespace {
std::mutex g_launch_mu;
std::map<std::tuple<const void *, long long, int>, int> g_launch_cache;
}  // namespace
bool launch_cache_get(const void *kernel, long long key, int dev, int *value)
{
    std::lock_guard<std::mutex> g(g_launch_mu);
    auto it = g_launch_cache.find(std::make_tuple(kernel, key, dev));
    if (it == g_launch_cache.end()) return false;
    *value = it->second;
    return true;
}
void launch_cache_put(const void *kernel, long long key, int dev, int value)
{
    std::lock_guard<std::mutex> g(g_launch_mu);
    g_launch_cache[std::make_tuple(kernel, key, dev)] = value;
}
void *ctx_scratch_alloc(nestgpu_ctx *c, size_t bytes) { return salloc(c, bytes); }
void ctx_scratch_reset(nestgpu_ctx *c) { scratch_reset(c); }
cudaStream_t ctx_stream(nestgpu_ctx *c) { return c->stream; }
int ctx_num_sms(nestgpu_ctx *c) { return c->num_sms; }
long long *ctx_launches(nestgpu_ctx *c) { return &c->launches; }
unsigned *ctx_pinned(nestgpu_ctx *c) { return c->pinned; }
int ctx_device(nestgpu_ctx *c) { return c->device; }
nestgpu_status ctx_fail(nestgpu_ctx *c, nestgpu_status code, const char *msg) { return fail(c, code, "%s", msg); }
}  // namespace ng

extern "C" {

nestgpu_status nestgpu_create(int device, void *d_arena, size_t arena_bytes, void *cuda_stream, nestgpu_ctx **out)
{
    if (!out) return NESTGPU_ERR_INVALID;
    *out = nullptr;
    if (!d_arena || arena_bytes < (1u << 20) || ((uintptr_t)d_arena % ALIGN) != 0) return NESTGPU_ERR_INVALID;
    if (cudaSetDevice(device) != cudaSuccess) return NESTGPU_ERR_CUDA;
    nestgpu_ctx *c = new nestgpu_ctx();
    c->device = device;
    c->base = (char *)d_arena;
    c->size = arena_bytes / ALIGN * ALIGN;
    c->lo = 0;
    c->hi = c->size;
    c->peak = 0;
    c->stream = (cudaStream_t)cuda_stream;
    c->launches = 0;
    c->profiling = false;
    c->malloc_scratch = false;
    c->bnl_shape = 0;
    c->sort_mode = 0;
    c->tiny_on = true;
    c->cap_stream = nullptr;
    {
        const char *gr = getenv("NESTGPU_GRAPHS");
        c->graphs_on = !(gr && gr[0] == '0');
    }
    {
        const char *tr = getenv("NESTGPU_TRACE");
        c->trace = tr && tr[0] == '1';
    }
    c->stage = nullptr;
    c->staged.ok = false;
    if (cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess ||
        cudaMallocHost((void **)&c->pinned, PIN_WORDS * sizeof(unsigned)) != cudaSuccess) {
        delete c;
        return NESTGPU_ERR_CUDA;
    }
    if (cudaMallocHost((void **)&c->stage, STAGE_BYTES) != cudaSuccess) {
        cudaFreeHost(c->pinned);
        delete c;
        return NESTGPU_ERR_CUDA;
    }
    for (int s = 0; s < NESTGPU_N_STAGES; s++) {
        cudaEventCreate(&c->ev[s][0]);
        cudaEventCreate(&c->ev[s][1]);
        c->ran[s] = false;
    }
    *out = c;
    return NESTGPU_OK;
}

nestgpu_status nestgpu_destroy(nestgpu_ctx *c)
{
    if (!c) return NESTGPU_OK;
    cudaSetDevice(c->device);
    cudaStreamSynchronize(c->stream);
    scratch_reset(c);
    for (int s = 0; s < NESTGPU_N_STAGES; s++) {
        cudaEventDestroy(c->ev[s][0]);
        cudaEventDestroy(c->ev[s][1]);
    }
    cudaFreeHost(c->pinned);
    cudaFreeHost(c->stage);
    for (auto &kv : c->graphs)
        if (kv.second.exec) cudaGraphExecDestroy(kv.second.exec);
    if (c->cap_stream) cudaStreamDestroy(c->cap_stream);
    delete c;
    return NESTGPU_OK;
}

const char *nestgpu_last_error(const nestgpu_ctx *c) { return c ? c->err.c_str() : "null context"; }
int64_t nestgpu_launch_count(const nestgpu_ctx *c) { return c ? c->launches : 0; }

nestgpu_status nestgpu_set_stream(nestgpu_ctx *c, void *s)
{
    if (!c) return NESTGPU_ERR_INVALID;
    cudaSetDevice(c->device);
    // Work queued on the old stream (e.g. an index build's radix passes) may
    // still write the arena: the new stream waits for it before anything
    // enqueued after the switch (no host synchronisation).
    if ((cudaStream_t)s != c->stream) {
        cudaEvent_t ev;
        CUDA_TRY(c, cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
        cudaError_t e = cudaEventRecord(ev, c->stream);
        if (e == cudaSuccess) e = cudaStreamWaitEvent((cudaStream_t)s, ev, 0);
        cudaEventDestroy(ev);
        if (e != cudaSuccess) return fail(c, NESTGPU_ERR_CUDA, "set_stream: %s", cudaGetErrorString(e));
    }
    c->stream = (cudaStream_t)s;
    return NESTGPU_OK;
}

nestgpu_status nestgpu_mark(nestgpu_ctx *c, uint64_t *m)
{
    if (!c || !m) return NESTGPU_ERR_INVALID;
    *m = c->lo;
    return NESTGPU_OK;
}

nestgpu_status nestgpu_release(nestgpu_ctx *c, uint64_t m)
{
    if (!c) return NESTGPU_ERR_INVALID;
    if (m > c->lo) return fail(c, NESTGPU_ERR_INVALID, "release: mark %llu beyond tail %zu", (unsigned long long)m, c->lo);
    cudaSetDevice(c->device);
    // Work already enqueued may still read the released bytes.
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    c->lo = m;
    scratch_reset(c);
    for (auto &col : c->cols)
        if (col.alive && col.off >= m) col.alive = false;
    for (auto &ix : c->idx) {
        if (ix.alive && ix.off >= m) ix.alive = false;
        for (int k = 0; k < 6; k++)
            if (ix.aux_pre[k] && ix.aux_off[k] >= m) ix.aux_pre[k] = ix.aux_suf[k] = nullptr;
    }
    return NESTGPU_OK;
}

nestgpu_status nestgpu_arena_usage(const nestgpu_ctx *c, size_t *in_use, size_t *peak)
{
    if (!c) return NESTGPU_ERR_INVALID;
    if (in_use) *in_use = c->lo + (c->size - c->hi);
    if (peak) *peak = c->peak;
    return NESTGPU_OK;
}

static nestgpu_status new_column(nestgpu_ctx *c, nestgpu_dtype dtype, int32_t scale, int64_t n, bool with_valid,
                                 int32_t *out)
{
    const int w = dtype_width(dtype);
    if (!w) return fail(c, NESTGPU_ERR_TYPE, "unknown dtype %d", (int)dtype);
    if (n < 0 || n >= (1ll << 31)) return fail(c, NESTGPU_ERR_INVALID, "column length %lld outside [0, 2^31)", (long long)n);
    Column col{};
    col.dtype = dtype;
    col.scale = scale;
    col.n = n;
    col.off = c->lo;
    col.d = palloc(c, (size_t)n * w);
    if (!col.d) return fail(c, NESTGPU_ERR_OOM, "arena exhausted loading a %lld-row column", (long long)n);
    if (with_valid) {
        col.valid = (uint8_t *)palloc(c, (size_t)n);
        if (!col.valid) {
            c->lo = col.off;
            return fail(c, NESTGPU_ERR_OOM, "arena exhausted (validity)");
        }
    }
    col.alive = true;
    *out = put_slot(c->cols, col);
    return NESTGPU_OK;
}

nestgpu_status nestgpu_load_column(nestgpu_ctx *c, nestgpu_dtype dtype, int32_t scale, const void *host_values,
                                   const uint8_t *host_valid, int64_t n, int32_t *out_col)
{
    if (!c || !out_col || (n > 0 && !host_values)) return fail(c, NESTGPU_ERR_INVALID, "load_column: null argument");
    cudaSetDevice(c->device);
    int32_t id;
    nestgpu_status s = new_column(c, dtype, scale, n, host_valid != nullptr, &id);
    if (s) return s;
    Column &col = c->cols[id];
    const size_t bytes = (size_t)n * dtype_width(dtype);
    if (n > 0) {
        CUDA_TRY(c, cudaMemcpyAsync(col.d, host_values, bytes, cudaMemcpyHostToDevice, c->stream));
        if (host_valid) CUDA_TRY(c, cudaMemcpyAsync(col.valid, host_valid, (size_t)n, cudaMemcpyHostToDevice, c->stream));
        CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    }
    *out_col = id;
    return NESTGPU_OK;
}

nestgpu_status nestgpu_alloc_column(nestgpu_ctx *c, nestgpu_dtype dtype, int32_t scale, int64_t n, int32_t with_valid,
                                    int32_t *out_col)
{
    if (!c || !out_col) return fail(c, NESTGPU_ERR_INVALID, "alloc_column: null argument");
    nestgpu_status st = new_column(c, dtype, scale, n, with_valid != 0, out_col);
    if (st == NESTGPU_OK) c->cols[*out_col].caller_filled = true;
    return st;
}

nestgpu_status nestgpu_column_info(const nestgpu_ctx *c, int32_t id, nestgpu_column_desc *out)
{
    if (!c || !out) return NESTGPU_ERR_INVALID;
    const Column *col = col_get(c, id);
    if (!col) return NESTGPU_ERR_INVALID;
    out->dtype = col->dtype;
    out->scale = col->scale;
    out->n = col->n;
    out->d_values = col->d;
    out->d_valid = col->valid;
    return NESTGPU_OK;
}

nestgpu_status nestgpu_gather_column(nestgpu_ctx *c, int32_t src_col, const int64_t *d_row_ids, int64_t n,
                                     int64_t row_id_base, int32_t *out_col)
{
    if (!c || !out_col || (n > 0 && !d_row_ids)) return fail(c, NESTGPU_ERR_INVALID, "gather_column: null argument");
    const Column *src = col_get(c, src_col);
    if (!src) return fail(c, NESTGPU_ERR_INVALID, "gather_column: unknown column %d", src_col);
    if (src->valid) return fail(c, NESTGPU_ERR_UNSUPPORTED, "gather_column: source column has NULLs");
    cudaSetDevice(c->device);
    const nestgpu_dtype dt = src->dtype;
    const int32_t scale = src->scale;
    const void *sd = src->d;
    int32_t id;
    nestgpu_status s = new_column(c, dt, scale, n, false, &id);   // may reallocate c->cols
    if (s) return s;
    CUDA_TRY(c, ng::launch_gather(dtype_width(dt), sd, (const long long *)d_row_ids, n, row_id_base, c->cols[id].d,
                                  c->stream, &c->launches));
    *out_col = id;
    return NESTGPU_OK;
}

// Sort-free index build for a key-ordered column (column statistics: NOT
// NULL, every row >= its predecessor -- e.g. TPC-H lineitem stored by
// l_orderkey, partsupp by ps_partkey): the stable sort of S' is then the
// identity, so the index is S' itself, compacted IN ROW ORDER by the ordered
// two-pass filter straight into the index arrays.  The count pass + scan run
// first; one sync reads |S'|; the index is allocated at its exact size and
// the write pass fills it.  Same bytes as the sorting build.
static nestgpu_status build_index_ordered(nestgpu_ctx *c, const int32_t *key_cols, int32_t n_key_cols,
                                          int32_t payload_col, const nestgpu_pred *inner_preds,
                                          int32_t n_inner_preds, const ng::KeySrc &ks, const ng::PredSet &ps,
                                          const ng::ValSrc &vs, int kb, int vb, int64_t n, const Column *pc,
                                          int32_t *out_index)
{
    scratch_reset(c);
    for (int st = 0; st < NESTGPU_N_STAGES; st++) c->ran[st] = false;
    void *fscr = salloc(c, ng::filter_scratch_bytes(n));
    long long *dsmall = (long long *)salloc(c, 64);
    if (!fscr || !dsmall) return fail(c, NESTGPU_ERR_OOM, "arena exhausted building an index over %lld rows", (long long)n);
    {
        ng::FillList fl;
        fl.add(dsmall, 16);
        fl.add(fscr, ng::filter_zero_bytes(n, false));
        CUDA_TRY(c, ng::launch_fill(fl, c->stream, &c->launches));
    }
    prof_begin(c, 1);
    CUDA_TRY(c, ng::launch_filter(n, ps, ks, kb, vs, vb, 0, 0, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr,
                                  fscr, dsmall, c->stream, &c->launches, true, 1));
    CUDA_TRY(c, cudaMemcpyAsync(c->pinned, dsmall, 8, cudaMemcpyDeviceToHost, c->stream));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    htrace(c, "ordered count + sync");
    long long nsp;
    memcpy(&nsp, c->pinned, 8);
    IndexRec ix{};
    ix.off = c->lo;
    ix.n = nsp;
    ix.kb = kb;
    ix.vb = vb;
    ix.d_n = (long long *)palloc(c, 8);
    ix.keys = palloc(c, (size_t)(nsp > 0 ? nsp : 1) * kb);
    ix.payload = vb ? palloc(c, (size_t)(nsp > 0 ? nsp : 1) * vb) : nullptr;
    if (!ix.d_n || !ix.keys || (vb && !ix.payload)) {
        c->lo = ix.off;
        return fail(c, NESTGPU_ERR_OOM, "arena exhausted storing an index of %lld rows", nsp);
    }
    CUDA_TRY(c, cudaMemcpyAsync(ix.d_n, dsmall, 8, cudaMemcpyDeviceToDevice, c->stream));
    if (nsp > 0)
        CUDA_TRY(c, ng::launch_filter(n, ps, ks, kb, vs, vb, 0, 0, nullptr, ix.keys, nullptr, ix.payload, nullptr,
                                      nullptr, fscr, dsmall, c->stream, &c->launches, true, 2));
    prof_end(c, 1);
    ix.key_cols[0] = key_cols[0];
    ix.key_cols[1] = n_key_cols == 2 ? key_cols[1] : -1;
    ix.n_key = n_key_cols;
    ix.payload_col = payload_col;
    ix.inner.assign(inner_preds, inner_preds + n_inner_preds);
    ix.payload_nullable = pc && pc->valid;
    ix.alive = true;
    *out_index = put_slot(c->idx, ix);
    CUDA_TRY(c, cudaGetLastError());
    htrace_end(c, "build_index (key-ordered column, no sort)");
    return NESTGPU_OK;
}

nestgpu_status nestgpu_build_index(nestgpu_ctx *c, const int32_t *key_cols, int32_t n_key_cols, int32_t payload_col,
                                   const nestgpu_pred *inner_preds, int32_t n_inner_preds, int32_t *out_index)
{
    if (!c || !key_cols || !out_index) return fail(c, NESTGPU_ERR_INVALID, "build_index: null argument");
    cudaSetDevice(c->device);
    htrace_begin(c);
    ng::KeySrc ks;
    int64_t n;
    nestgpu_status s = make_key(c, key_cols, n_key_cols, n, ks, "build_index");
    if (s) return s;
    ng::PredSet ps;
    if ((s = make_preds(c, inner_preds, n_inner_preds, n, ps, "inner_preds"))) return s;
    ng::ValSrc vs{nullptr, nullptr, 0};
    const Column *pc = nullptr;
    if (payload_col >= 0) {
        pc = col_get(c, payload_col);
        if (!pc) return fail(c, NESTGPU_ERR_INVALID, "build_index: unknown payload column %d", payload_col);
        if (pc->n != n) return fail(c, NESTGPU_ERR_INVALID, "build_index: payload row count differs");
        vs.c = pc->d;
        vs.v = pc->valid;
        vs.w = dtype_width(pc->dtype);
    }
    const int kb = key_bytes(c, key_cols, n_key_cols);
    const int vb = pc ? vs.w : 0;
    bool stats_fresh = false;
    if (n_key_cols == 1 && c->sort_mode != 1) {
        Column &kc = c->cols[key_cols[0]];
        if (!kc.valid && !(pc && pc->valid)) {
            if (kc.caller_filled) kc.stats = false;   // recomputed: the caller may have rewritten it
            stats_fresh = true;
            if ((s = column_stats(c, kc))) return s;
            if (kc.sorted)
                return build_index_ordered(c, key_cols, n_key_cols, payload_col, inner_preds, n_inner_preds, ks, ps,
                                           vs, kb, vb, n, pc, out_index);
        }
    }
    // 64-bit keys of one column whose encoded min and max share the high word
    // (column statistics, computed once per column): every key does, so the
    // S' filter already writes 32-bit keys and the whole sort runs on them;
    // the last pass re-attaches the word (Q4's order keys: 152 MB less to
    // write, histogram and read again)
    bool pre_narrow = false;
    unsigned pre_hi = 0;
    if (kb == 8 && n_key_cols == 1) {
        Column &kc = c->cols[key_cols[0]];
        if (kc.caller_filled && !stats_fresh) kc.stats = false;   // recomputed: the caller may have rewritten it
        if ((s = column_stats(c, kc))) return s;
        const unsigned long long emn = (unsigned long long)kc.mn ^ 0x8000000000000000ull;
        const unsigned long long emx = (unsigned long long)kc.mx ^ 0x8000000000000000ull;
        if (kc.mn <= kc.mx && (emn >> 32) == (emx >> 32)) {
            pre_narrow = true;
            pre_hi = (unsigned)(emn >> 32);
        }
    }
    const int fkb = pre_narrow ? 4 : kb;   // key width the S' filter writes
    // an index over all of S (no predicates, NOT NULL key / payload) needs no
    // sync: |S'| = |S| and the radix plan comes from the key column's stats
    bool nosync = false;
    if (n_key_cols == 1 && n_inner_preds == 0 && c->sort_mode != 2) {
        Column &kc = c->cols[key_cols[0]];
        if (!kc.valid && !(pc && pc->valid)) {
            if (kc.caller_filled && !stats_fresh) kc.stats = false;
            if ((s = column_stats(c, kc))) return s;
            stats_fresh = true;
            nosync = true;
        }
    }
    scratch_reset(c);
    for (int st = 0; st < NESTGPU_N_STAGES; st++) c->ran[st] = false;
    void *tk = salloc(c, (size_t)n * kb), *tv = vb ? salloc(c, (size_t)n * vb) : nullptr;
    void *uk = salloc(c, (size_t)n * kb), *uv = vb ? salloc(c, (size_t)n * vb) : nullptr;
    void *fscr = salloc(c, ng::filter_scratch_bytes(n));
    unsigned *hist = (unsigned *)salloc(c, ng::hist_bytes());
    unsigned *dbase = (unsigned *)salloc(c, 8 * 512 * 4);
    long long *dsmall = (long long *)salloc(c, 64);   // [0] |S'|, [2] key AND, [3] key OR
    if (!tk || !uk || !fscr || !hist || !dbase || !dsmall || (vb && (!tv || !uv)))
        return fail(c, NESTGPU_ERR_OOM, "arena exhausted building an index over %lld rows", (long long)n);
    long long *d_count = dsmall;
    unsigned long long *keymask = (unsigned long long *)(dsmall + 2);
    // small S: the scratch of the histogram and of every possible pass is
    // allocated now and zeroed by the same fill (no second fill after the sync)
    const bool small = n <= SMALL_ROWS;
    void *pscr[8] = {};
    if (small)
        for (int p = 0; p < kb; p++)
            if (!(pscr[p] = salloc(c, ng::sort_scratch_bytes(n))))
                return fail(c, NESTGPU_ERR_OOM, "arena exhausted (sort scratch)");
    {   // one fill kernel instead of a memset per scratch region
        ng::FillList fl;
        fl.add(dsmall, 16);
        fl.add(keymask, 8, 0xff);   // AND identity
        fl.add(dsmall + 3, 40);
        fl.add(fscr, ng::filter_zero_bytes(n, false));
        if (small) {
            fl.add(hist, ng::hist_bytes());
            for (int p = 0; p < kb; p++) fl.add(pscr[p], ng::sort_scratch_bytes(n));
        }
        htrace(c, "setup");
        CUDA_TRY(c, ng::launch_fill(fl, c->stream, &c->launches));
        htrace(c, "fill");
    }
    // the encoded key AND / OR the S' filter would report, from the key
    // column's statistics (nosync: S' = S)
    auto stats_mask = [&](unsigned long long &ka_out, unsigned long long &ko_out) {
        const Column &kc = c->cols[key_cols[0]];
        const unsigned long long sb = fkb == 8 ? (1ull << 63) : (kb == 4 ? 0x80000000ull : 0ull);
        unsigned long long ka = (unsigned long long)kc.band, ko = (unsigned long long)kc.bor;
        if (fkb == 4) {   // 4-byte keys: the filter's AND / OR of zero-extended keys
            ka &= 0xffffffffull;
            ko &= 0xffffffffull;
        }
        ka_out = (ka & ~sb) | (~ko & sb);
        ko_out = (ko & ~sb) | (~ka & sb);
        if (fkb == 4) {
            ka_out &= 0xffffffffull;
            ko_out &= 0xffffffffull;
        }
    };
    // with S' = S and at least one radix pass, the first pass and the
    // histogram read the raw key / payload columns and encode keys as they
    // load them: no filter pass at all
    bool raw_input = false;
    if (nosync && n > 1 && n < (1ll << 30)) {
        unsigned long long ka, ko;
        stats_mask(ka, ko);
        int sh0[8], rb0 = 8;
        raw_input = plan_sort_passes(fkb, ka, ko, n, sh0, &rb0) >= 1;
    }
    prof_begin(c, 1);
    if (!raw_input)
        CUDA_TRY(c, ng::launch_filter(n, ps, ks, fkb, vs, vb, 1, pc ? 1 : 0, nullptr, tk, nullptr, tv, keymask, nullptr,
                                      fscr, d_count, c->stream, &c->launches, true));
    prof_end(c, 1);
    htrace(c, "filter");
    long long nsp;
    unsigned long long kand, kor;
    if (nosync) {
        // no predicates, NOT NULL key and payload: S' = S, and the key bits
        // that vary come from the column statistics (AND / OR of the values,
        // encoded as the filter encodes them) -- no host round trip
        stats_mask(kand, kor);
        nsp = n;
        htrace(c, "plan from stats");
    } else {
        CUDA_TRY(c, cudaMemcpyAsync(c->pinned, dsmall, 32, cudaMemcpyDeviceToHost, c->stream));
        CUDA_TRY(c, cudaStreamSynchronize(c->stream));
        htrace(c, "sync");
        memcpy(&nsp, c->pinned, 8);
        memcpy(&kand, c->pinned + 4, 8);
        memcpy(&kor, c->pinned + 6, 8);
    }
    if (nsp >= (1ll << 30))   // radix-pass look-back words carry 30-bit counts
        return fail(c, NESTGPU_ERR_UNSUPPORTED, "build_index: |S'| = %lld >= 2^30 rows to sort", nsp);
    int shifts[8], rb = 8;
    int np = plan_sort_passes(fkb, kand, kor, nsp, shifts, &rb);
    if (pre_narrow && np == 0 && nsp > 0) {   // equal keys: one pass still widens them to 64 bits
        np = 1;
        shifts[0] = 0;
    }
    // 64-bit keys whose high words all agree (AND == OR there, e.g. Q4's
    // order keys) travel as 32-bit keys between the first and the last
    // pass: the first pass drops the high word, the last re-attaches it.
    const bool narrow = pre_narrow || (kb == 8 && np >= 2 && ((kand ^ kor) >> 32) == 0);
    const unsigned hi = pre_narrow ? pre_hi : (unsigned)(kand >> 32);
    IndexRec ix{};
    ix.off = c->lo;
    ix.n = nsp;
    ix.kb = kb;
    ix.vb = vb;
    ix.d_n = (long long *)palloc(c, 8);
    ix.keys = palloc(c, (size_t)nsp * kb);
    ix.payload = vb ? palloc(c, (size_t)nsp * vb) : nullptr;
    if (!ix.d_n || !ix.keys || (vb && !ix.payload)) {
        c->lo = ix.off;
        return fail(c, NESTGPU_ERR_OOM, "arena exhausted storing an index of %lld rows", nsp);
    }
    c->pinned[8 * 256 + 4] = (unsigned)(nsp & 0xffffffffu);
    c->pinned[8 * 256 + 5] = (unsigned)((unsigned long long)nsp >> 32);
    CUDA_TRY(c, cudaMemcpyAsync(ix.d_n, c->pinned + 8 * 256 + 4, 8, cudaMemcpyHostToDevice, c->stream));
    prof_begin(c, 2);
    // Two-round-trip MSD bucket sort (k_bsort.cu, NESTGPU_OPT_SORT = 2 only:
    // measured 1.2-1.9x slower than the LSD onesweep on every shape, DESIGN
    // §18): partition by the top D varying bits, finish every bucket in
    // shared memory.  Its histograms report the largest bucket; one more sync
    // reads it, and skewed keys (a bucket past the finish capacity) fall
    // through to the LSD onesweep below.
    bool sorted = false;
    if (c->sort_mode == 2 && np >= 1 && (kand ^ kor) != 0) {
        const int kmid = narrow ? 4 : kb;
        const unsigned long long var = kand ^ kor;
        const int top = 63 - __builtin_clzll(var), low = __builtin_ctzll(var);
        const long long cap = ng::bsort_capacity(kmid, vb);
        int D = 1;
        while (D < 12 && (double)nsp / (double)(1ll << D) > 0.6 * (double)cap) D++;
        const int s1 = top - D + 1;
        // finish passes: <= 6-bit windows over the varying bits below s1
        int sh2[12], bt2[12], np2 = 0;
        for (int b = low; b < s1 && np2 < 12;) {
            if (!((var >> b) & 1ull)) {
                b++;
                continue;
            }
            const int w = s1 - b < 6 ? s1 - b : 6;
            sh2[np2] = b;
            bt2[np2++] = w;
            b += w;
        }
        bool fits = (double)nsp / (double)(1ll << D) <= 0.9 * (double)cap && s1 > low && np2 > 0 && np2 <= 12;
        if (fits) {
            const int nb = 1 << D;
            void *hs = salloc(c, ng::bsort_hist_bytes(nsp, nb));
            unsigned *zs = (unsigned *)salloc(c, ng::bsort_zero_bytes(nb));
            unsigned *bbase = (unsigned *)salloc(c, (size_t)(nb + 1) * 4);
            unsigned *maxb = (unsigned *)(dsmall + 4);
            if (!hs || !zs || !bbase) return fail(c, NESTGPU_ERR_OOM, "arena exhausted (bucket sort scratch)");
            ng::FillList fl;
            fl.add(zs, ng::bsort_zero_bytes(nb));
            CUDA_TRY(c, ng::launch_fill(fl, c->stream, &c->launches));
            CUDA_TRY(c, ng::launch_bsort_hist(fkb, tk, nsp, s1, nb, hs, zs, bbase, maxb, c->stream, &c->launches));
            CUDA_TRY(c, cudaMemcpyAsync(c->pinned + 16, maxb, 4, cudaMemcpyDeviceToHost, c->stream));
            CUDA_TRY(c, cudaStreamSynchronize(c->stream));
            htrace(c, "bsort hist + sync");
            if ((long long)c->pinned[16] <= cap) {
                CUDA_TRY(c, ng::launch_bsort_sort(fkb, kmid, kb, vb, tk, tv, uk, uv, ix.keys, ix.payload, nsp, s1, D,
                                                  sh2, bt2, np2, hs, bbase, hi, c->stream, &c->launches));
                sorted = true;
                htrace(c, "bsort");
            }
        }
    }
    // one scratch region per pass, all zeroed with the digit histograms by
    // one fill kernel
    if (!sorted && !small) {
        ng::FillList fl;
        fl.add(hist, ng::hist_bytes());
        for (int p = 0; p < np; p++) {
            const int kin = raw_input && p == 0 ? kb : (pre_narrow || (narrow && p > 0) ? 4 : kb);
            const size_t zb = ng::sort_pass_zero_bytes(nsp, kin, vb, rb);
            pscr[p] = salloc(c, zb);
            if (!pscr[p]) return fail(c, NESTGPU_ERR_OOM, "arena exhausted (sort scratch)");
            fl.add(pscr[p], zb);
        }
        CUDA_TRY(c, ng::launch_fill(fl, c->stream, &c->launches));
    }
    htrace(c, "fill2");
    if (!sorted) {
        const Column &kcol = c->cols[key_cols[0]];
        const unsigned long long rencx = kb == 8 ? (1ull << 63) : 0x80000000ull;   // raw column -> encoded key
        if (raw_input)
            CUDA_TRY(c, ng::launch_digit_hist(kb, kcol.d, nsp, shifts, np, hist, dbase, c->num_sms, c->stream,
                                              &c->launches, rb, true, rencx));
        else
            CUDA_TRY(c, ng::launch_digit_hist(fkb, tk, nsp, shifts, np, hist, dbase, c->num_sms, c->stream,
                                              &c->launches, rb, true));
        htrace(c, "hist");
    }
    if (sorted) {
    } else if (np == 0) {
        if (nsp > 0) {
            CUDA_TRY(c, cudaMemcpyAsync(ix.keys, tk, (size_t)nsp * kb, cudaMemcpyDeviceToDevice, c->stream));
            if (vb) CUDA_TRY(c, cudaMemcpyAsync(ix.payload, tv, (size_t)nsp * vb, cudaMemcpyDeviceToDevice, c->stream));
        }
    } else {
        // T -> ... -> P with ping-pong so that the last pass writes P (the
        // first pass reads the raw columns when the filter was skipped)
        const Column &kcol = c->cols[key_cols[0]];
        const void *ik = raw_input ? kcol.d : tk, *iv = raw_input ? (pc ? pc->d : nullptr) : tv;
        for (int p = 0; p < np; p++) {
            const bool to_final = ((np - 1 - p) % 2) == 0;
            void *ok = to_final ? ix.keys : uk;
            void *ov = to_final ? ix.payload : uv;
            if (ok == ik) { ok = tk; ov = tv; }
            const bool rawp = raw_input && p == 0;
            const int kin = rawp ? kb : (pre_narrow || (narrow && p > 0) ? 4 : kb), kout = narrow && p < np - 1 ? 4 : kb;
            const unsigned long long encx = rawp ? (kb == 8 ? (1ull << 63) : 0x80000000ull) : 0ull;
            CUDA_TRY(c, ng::launch_radix_pass_x(kin, kout, vb, ik, ok, iv, ov, nsp, shifts[p], dbase + p * (1 << rb),
                                                pscr[p], hi, c->stream, &c->launches, rb, true, encx));
            ik = ok;
            iv = ov;
        }
    }
    prof_end(c, 2);
    htrace(c, "passes");
    ix.key_cols[0] = key_cols[0];
    ix.key_cols[1] = n_key_cols == 2 ? key_cols[1] : -1;
    ix.n_key = n_key_cols;
    ix.payload_col = payload_col;
    ix.inner.assign(inner_preds, inner_preds + n_inner_preds);
    ix.payload_nullable = pc && pc->valid;
    ix.alive = true;
    *out_index = put_slot(c->idx, ix);
    CUDA_TRY(c, cudaGetLastError());
    htrace_end(c, "build_index");
    return NESTGPU_OK;
}

nestgpu_status nestgpu_drop_index(nestgpu_ctx *c, int32_t index)
{
    if (!c || index < 0 || index >= (int32_t)c->idx.size() || !c->idx[index].alive)
        return fail(c, NESTGPU_ERR_INVALID, "drop_index: unknown index %d", index);
    c->idx[index].alive = false;
    return NESTGPU_OK;
}

nestgpu_status nestgpu_index_info(const nestgpu_ctx *c, int32_t index, nestgpu_index_desc *out)
{
    if (!c || !out || index < 0 || index >= (int32_t)c->idx.size() || !c->idx[index].alive) return NESTGPU_ERR_INVALID;
    const IndexRec &ix = c->idx[index];
    out->n = ix.n;
    out->key_bytes = ix.kb;
    out->payload_bytes = ix.vb;
    out->d_keys = ix.keys;
    out->d_payload = ix.payload;
    return NESTGPU_OK;
}

nestgpu_status nestgpu_index_create_empty(nestgpu_ctx *c, int64_t n, int32_t key_bytes_, int32_t payload_bytes,
                                          const int32_t *key_cols, int32_t n_key_cols, int32_t payload_col,
                                          const nestgpu_pred *inner_preds, int32_t n_inner_preds,
                                          nestgpu_index_desc *out, int32_t *out_index)
{
    if (!c || !out || !out_index || !key_cols) return fail(c, NESTGPU_ERR_INVALID, "index_create_empty: null argument");
    if (n < 0 || n >= (1ll << 31) || (key_bytes_ != 4 && key_bytes_ != 8) ||
        (payload_bytes != 0 && payload_bytes != 4 && payload_bytes != 8))
        return fail(c, NESTGPU_ERR_INVALID, "index_create_empty: bad shape");
    ng::KeySrc ks;
    int64_t ns;
    nestgpu_status s = make_key(c, key_cols, n_key_cols, ns, ks, "index_create_empty");
    if (s) return s;
    if (key_bytes(c, key_cols, n_key_cols) != key_bytes_)
        return fail(c, NESTGPU_ERR_TYPE, "index_create_empty: key width does not match the key columns");
    if (n_inner_preds < 0 || (n_inner_preds > 0 && !inner_preds)) return fail(c, NESTGPU_ERR_INVALID, "bad inner preds");
    {
        const Column *pcol = payload_col >= 0 ? col_get(c, payload_col) : nullptr;
        if (payload_col >= 0 && !pcol) return fail(c, NESTGPU_ERR_INVALID, "index_create_empty: unknown payload column %d", payload_col);
        if (payload_bytes != (pcol ? dtype_width(pcol->dtype) : 0))
            return fail(c, NESTGPU_ERR_INVALID, "index_create_empty: payload_bytes must equal the payload column's width (0 without payload)");
        if (pcol && pcol->n != ns) return fail(c, NESTGPU_ERR_INVALID, "index_create_empty: payload row count differs");
    }
    cudaSetDevice(c->device);
    IndexRec ix{};
    ix.off = c->lo;
    ix.n = n;
    ix.kb = key_bytes_;
    ix.vb = payload_bytes;
    ix.d_n = (long long *)palloc(c, 8);
    ix.keys = palloc(c, (size_t)n * key_bytes_);
    ix.payload = payload_bytes ? palloc(c, (size_t)n * payload_bytes) : nullptr;
    if (!ix.d_n || !ix.keys || (payload_bytes && !ix.payload)) {
        c->lo = ix.off;
        return fail(c, NESTGPU_ERR_OOM, "arena exhausted (index_create_empty)");
    }
    long long nn = n;
    memcpy(c->pinned, &nn, 8);
    CUDA_TRY(c, cudaMemcpyAsync(ix.d_n, c->pinned, 8, cudaMemcpyHostToDevice, c->stream));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    ix.key_cols[0] = key_cols[0];
    ix.key_cols[1] = n_key_cols == 2 ? key_cols[1] : -1;
    ix.n_key = n_key_cols;
    ix.payload_col = payload_col;
    ix.inner.assign(inner_preds, inner_preds + n_inner_preds);
    const Column *pc = payload_col >= 0 ? col_get(c, payload_col) : nullptr;
    ix.payload_nullable = pc && pc->valid;
    ix.alive = true;
    *out_index = put_slot(c->idx, ix);
    out->n = n;
    out->key_bytes = key_bytes_;
    out->payload_bytes = payload_bytes;
    out->d_keys = ix.keys;
    out->d_payload = ix.payload;
    return NESTGPU_OK;
}

// ---------------------------------------------------------------- exec graphs
}  // extern "C"
namespace {
template <typename T>
void kput(std::string &k, const T &v)
{
    k.append((const char *)&v, sizeof v);
}

bool graph_ok(const nestgpu_ctx *c, const nestgpu_plan *P, const IndexRec *)
{
    // dedup synchronises mid-sequence; profiling / tracing record host-side
    // state per call; the malloc ablation allocates per call
    return c->graphs_on && !P->dedup && !c->profiling && !c->malloc_scratch;
}

// Everything the exec's launch sequence depends on: the plan (predicates by
// value), every referenced column's address / validity / rows / type, the
// index record (arrays, size, widths, aux arrays), the arena state (scratch
// addresses follow from it) and the knobs.  Equal keys => identical launches.
std::string exec_graph_key(const nestgpu_ctx *c, const nestgpu_plan *P, const IndexRec *ix, bool wide)
{
    std::string k;
    k.reserve(512);
    nestgpu_plan q = *P;
    q.outer_preds = nullptr;
    q.inner_preds = nullptr;
    kput(k, q);
    for (int i = 0; i < P->n_outer_preds; i++) kput(k, P->outer_preds[i]);
    for (int i = 0; i < P->n_inner_preds; i++) kput(k, P->inner_preds[i]);
    auto col = [&](int32_t id) {
        kput(k, id);
        if (id < 0 || id >= (int32_t)c->cols.size() || !c->cols[id].alive) return;
        const Column &x = c->cols[id];
        kput(k, x.d);
        kput(k, x.valid);
        kput(k, x.n);
        kput(k, x.dtype);
    };
    for (int i = 0; i < P->n_key_cols; i++) {
        col(P->outer_key_cols[i]);
        col(P->inner_key_cols[i]);
    }
    col(P->outer_cmp_col);
    col(P->agg_col);
    for (int i = 0; i < P->n_outer_preds; i++) {
        col(P->outer_preds[i].col);
        col(P->outer_preds[i].rhs_col);
    }
    for (int i = 0; i < P->n_inner_preds; i++) {
        col(P->inner_preds[i].col);
        col(P->inner_preds[i].rhs_col);
    }
    if (ix) {
        kput(k, ix->keys);
        kput(k, ix->payload);
        kput(k, ix->n);
        kput(k, ix->kb);
        kput(k, ix->vb);
        for (int i = 0; i < 6; i++) {
            kput(k, ix->aux_pre[i]);
            kput(k, ix->aux_suf[i]);
        }
    }
    kput(k, c->lo);
    kput(k, c->size);
    kput(k, c->base);
    kput(k, c->bnl_shape);
    kput(k, wide);
    return k;
}

// Replay the captured launch sequence for `key`: the first GRAPH_AFTER
// sightings of a key run directly, the next captures the sequence (and runs
// it once through the graph), later ones replay it.  A sequence that cannot
// be captured (e.g. a launch kind the graph API refuses) is remembered and
// run directly.
constexpr int GRAPH_AFTER = 8;
template <typename F>
nestgpu_status run_graph(nestgpu_ctx *c, const std::string &key, F &enqueue)
{
    auto it = c->graphs.find(key);
    if (it == c->graphs.end()) {
        // first sighting: run directly and remember the key -- a sequence is
        // captured only when it repeats, so one-off execs (fresh tables, a
        // per-tuple drive program) never pay for a capture
        if (c->graphs.size() >= 256) {
            for (auto &kv : c->graphs)
                if (kv.second.exec) cudaGraphExecDestroy(kv.second.exec);
            c->graphs.clear();
        }
        c->graphs.emplace(key, nestgpu_ctx::GraphEntry{nullptr, 0, 1});
        htrace(c, "graph:first");
        return enqueue();
    }
    if (!it->second.exec && it->second.kernels == 0 && it->second.seen < GRAPH_AFTER) {
        // capturing + instantiating costs ~1-3 ms: only sequences that keep
        // repeating are worth it
        it->second.seen++;
        htrace(c, "graph:direct");
        return enqueue();
    }
    if (!it->second.exec && it->second.kernels == 0) {
        const long long l0 = c->launches;
        const std::string err0 = c->err;
        // capture on the context's private stream (the caller's may be the
        // legacy default stream, which cannot be captured); the graph is
        // then launched on the caller's stream
        if (!c->cap_stream && cudaStreamCreateWithFlags(&c->cap_stream, cudaStreamNonBlocking) != cudaSuccess) {
            cudaGetLastError();
            c->cap_stream = nullptr;
            c->graphs_on = false;
            return enqueue();
        }
        cudaStream_t user = c->stream;
        c->stream = c->cap_stream;
        if (cudaStreamBeginCapture(c->stream, cudaStreamCaptureModeThreadLocal) != cudaSuccess) {
            cudaGetLastError();
            c->stream = user;
            it->second = nestgpu_ctx::GraphEntry{nullptr, -1, 0};
            return enqueue();
        }
        const nestgpu_status st = enqueue();
        cudaGraph_t g = nullptr;
        cudaError_t e = cudaStreamEndCapture(c->stream, &g);
        c->stream = user;
        cudaGraphExec_t ge = nullptr;
        if (st == NESTGPU_OK && e == cudaSuccess && g) e = cudaGraphInstantiate(&ge, g, 0);
        if (g) cudaGraphDestroy(g);
        const long long kernels = c->launches - l0;
        c->launches = l0;
        if (st != NESTGPU_OK || e != cudaSuccess || !ge) {
            if (c->trace)
                fprintf(stderr, "[nestgpu trace] graph capture failed: status %d, %s, %s\n", (int)st,
                        cudaGetErrorString(e), c->err.c_str());
            cudaGetLastError();   // clear the capture error; run this sequence directly from now on
            c->err = err0;
            it->second = nestgpu_ctx::GraphEntry{nullptr, -1, 0};
            return enqueue();
        }
        it->second = nestgpu_ctx::GraphEntry{ge, kernels, 0};
    }
    if (!it->second.exec) {
        htrace(c, "graph:direct");
        return enqueue();
    }
    htrace(c, "graph:replay");
    CUDA_TRY(c, cudaGraphLaunch(it->second.exec, c->stream));
    c->launches += it->second.kernels;
    return NESTGPU_OK;
}
}  // namespace
extern "C" {

nestgpu_status nestgpu_exec_correlated(nestgpu_ctx *c, const nestgpu_plan *P, nestgpu_result *out)
{
    if (!c || !P || !out) return fail(c, NESTGPU_ERR_INVALID, "exec: null argument");
    cudaSetDevice(c->device);
    htrace_begin(c);
    memset(out, 0, sizeof *out);
    // ------------------------------------------------------------ validation
    if (P->agg < NG_MIN || P->agg > NG_NOT_EXISTS) return fail(c, NESTGPU_ERR_INVALID, "exec: bad aggregate");
    if (!valid_op(P->corr_op)) return fail(c, NESTGPU_ERR_INVALID, "exec: bad correlated operator");
    if (P->n_key_cols == 2 && P->corr_op != NG_EQ)
        return fail(c, NESTGPU_ERR_UNSUPPORTED, "exec: composite correlation supports '=' only");
    const bool is_exists = P->agg == NG_EXISTS || P->agg == NG_NOT_EXISTS;
    const bool value_agg = P->agg == NG_MIN || P->agg == NG_MAX || P->agg == NG_SUM || P->agg == NG_AVG;
    if (!is_exists && !valid_op(P->outer_op)) return fail(c, NESTGPU_ERR_INVALID, "exec: bad outer operator");
    if (!is_exists && (P->lhs_mult < 1 || P->lhs_mult >= (1ll << 31) || P->rhs_mult < 1 || P->rhs_mult >= (1ll << 31)))
        return fail(c, NESTGPU_ERR_INVALID, "exec: lhs_mult / rhs_mult must be in [1, 2^31)");
    ng::KeySrc rks, sks;
    int64_t nR, nS;
    nestgpu_status s;
    if ((s = make_key(c, P->outer_key_cols, P->n_key_cols, nR, rks, "outer key"))) return s;
    if ((s = make_key(c, P->inner_key_cols, P->n_key_cols, nS, sks, "inner key"))) return s;
    ng::PredSet ops, ips;
    if ((s = make_preds(c, P->outer_preds, P->n_outer_preds, nR, ops, "outer_preds"))) return s;
    if ((s = make_preds(c, P->inner_preds, P->n_inner_preds, nS, ips, "inner_preds"))) return s;
    const Column *xc = nullptr;
    if (!is_exists) {
        xc = col_get(c, P->outer_cmp_col);
        if (!xc) return fail(c, NESTGPU_ERR_INVALID, "exec: unknown outer comparison column %d", P->outer_cmp_col);
        if (xc->n != nR) return fail(c, NESTGPU_ERR_INVALID, "exec: outer comparison column row count differs from R");
    }
    Column *ac = nullptr;
    if (value_agg) {
        ac = (P->agg_col >= 0 && P->agg_col < (int32_t)c->cols.size() && c->cols[P->agg_col].alive) ? &c->cols[P->agg_col] : nullptr;
        if (!ac) return fail(c, NESTGPU_ERR_INVALID, "exec: unknown aggregate column %d", P->agg_col);
        if (ac->n != nS) return fail(c, NESTGPU_ERR_INVALID, "exec: aggregate column row count differs from S");
    }
    const int rkb = key_bytes(c, P->outer_key_cols, P->n_key_cols);
    const int skb = key_bytes(c, P->inner_key_cols, P->n_key_cols);
    int kb = (rkb == 8 || skb == 8) ? 8 : 4;
    IndexRec *ix = nullptr;
    if (P->index >= 0) {
        if (P->index >= (int32_t)c->idx.size() || !c->idx[P->index].alive)
            return fail(c, NESTGPU_ERR_INVALID, "exec: unknown index %d", P->index);
        ix = &c->idx[P->index];
        if (ix->n_key != P->n_key_cols || ix->key_cols[0] != P->inner_key_cols[0] ||
            (P->n_key_cols == 2 && ix->key_cols[1] != P->inner_key_cols[1]))
            return fail(c, NESTGPU_ERR_INVALID, "exec: index %d is on different key columns", P->index);
        if (!same_preds(P->inner_preds, P->n_inner_preds, ix->inner))
            return fail(c, NESTGPU_ERR_INVALID, "exec: index %d was built with different inner predicates", P->index);
        if (value_agg && ix->payload_col != P->agg_col)
            return fail(c, NESTGPU_ERR_INVALID, "exec: index %d carries column %d, plan aggregates %d", P->index, ix->payload_col, P->agg_col);
        if (!value_agg && ix->payload_nullable)
            return fail(c, NESTGPU_ERR_INVALID, "exec: index %d dropped NULL-payload rows; COUNT/EXISTS need an index without payload", P->index);
        if (ix->kb != kb)
            return fail(c, NESTGPU_ERR_UNSUPPORTED, "exec: outer key is 64-bit but index %d has 32-bit keys", P->index);
        if (value_agg && (ix->vb != dtype_width(ac->dtype) || (ix->n > 0 && !ix->payload)))
            return fail(c, NESTGPU_ERR_INVALID, "exec: index %d carries %d-byte payloads, column %d has %d-byte values",
                        P->index, ix->vb, P->agg_col, dtype_width(ac->dtype));
    }
    const int vb = value_agg ? dtype_width(ac->dtype) : 0;
    // Exact SUM/AVG (reading R5): 32-bit payloads cannot overflow (|S| < 2^31);
    // 64-bit payloads whose |S| * max|payload| could reach 2^63 are summed as
    // split halves (low 32 bits unsigned, high 32 bits signed -- neither sum can
    // overflow) and recombined in int128 by finalize, which reports
    // NESTGPU_ERR_OVERFLOW only when an actual result leaves int64.
    bool wide = false;
    if ((P->agg == NG_SUM || P->agg == NG_AVG) && vb == 8) {
        if (ac->caller_filled) ac->stats = false;   // recomputed: the caller may have rewritten it
        if ((s = column_stats(c, *ac))) return s;
        const __int128 m = std::max((__int128)ac->mx, -(__int128)ac->mn);
        wide = (__int128)nS * m >= ((__int128)1 << 63);
    }

    htrace(c, "validate");
    // ------------------------------------------------------------ allocation
    scratch_reset(c);  // previous results die here
    for (int st = 0; st < NESTGPU_N_STAGES; st++) c->ran[st] = false;
    const bool ravalid = rks.v0 || rks.v1;
    int *ids = (int *)salloc(c, (size_t)nR * 4);
    void *rkeys = salloc(c, (size_t)nR * kb);
    uint8_t *rkvalid = ravalid ? (uint8_t *)salloc(c, (size_t)nR) : nullptr;
    long long *acc = (long long *)salloc(c, (size_t)nR * 8);
    long long *cnt = (long long *)salloc(c, (size_t)nR * 8);
    long long *counts = (long long *)salloc(c, 128 + 8 * ng::TINY_G_MAX);  // [0] |R'| [1] |S'| [2] survivors;
                                                                          // [4..5] extreme; [8] overflow; tiny: CTA counts
    long long *acc_hi = wide ? (long long *)salloc(c, (size_t)nR * 8) : nullptr;
    // one scratch per filter / finalize (all zeroed up front by one fill kernel)
    void *fscr = salloc(c, ng::filter_scratch_bytes(nR));
    void *fscr_s = ix ? nullptr : salloc(c, ng::filter_scratch_bytes(nS));
    void *fscr_f = salloc(c, ng::finalize_scratch_bytes(nR));
    void *kscr = salloc(c, ix ? ng::range_scratch_bytes(nR) : ng::bnl_scratch_bytes(nR));
    // result block: ids | values | [AVG sum | AVG nn] | valid | passed, one
    // allocation so its first rows reach the host in two copies (staging)
    const bool is_avg = P->agg == NG_AVG;
    const size_t w8 = is_avg ? 4 : 2;
    char *rblk = (char *)salloc(c, (size_t)nR * (8 * w8 + 2));
    long long *o_ids = rblk ? (long long *)rblk : nullptr;
    long long *o_vals = rblk ? (long long *)(rblk + (size_t)nR * 8) : nullptr;
    long long *o_sum = rblk && is_avg ? (long long *)(rblk + (size_t)nR * 16) : nullptr;
    long long *o_cnt = rblk && is_avg ? (long long *)(rblk + (size_t)nR * 24) : nullptr;
    uint8_t *o_valid = rblk ? (uint8_t *)(rblk + (size_t)nR * 8 * w8) : nullptr;
    uint8_t *o_pass = rblk ? o_valid + nR : nullptr;
    void *skeys = nullptr, *svals = nullptr;
    if (!ix) {
        skeys = salloc(c, (size_t)nS * kb);
        svals = vb ? salloc(c, (size_t)nS * vb) : nullptr;
    }
    if (!ids || !rkeys || (ravalid && !rkvalid) || !acc || !cnt || !counts || !fscr || !fscr_f || !kscr || !rblk ||
        (!ix && (!fscr_s || !skeys || (vb && !svals))) || (wide && !acc_hi))
        return fail(c, NESTGPU_ERR_OOM, "arena exhausted executing a plan over |R|=%lld |S|=%lld", (long long)nR, (long long)nS);
    // counts: [0] |R'| [1] |S'| [2] survivors [3] distinct keys [4] extreme flags (2 x u32)
    //         [6] AND / [7] OR of the R' keys (dedup sort planning) [8] split-SUM overflow flag
    unsigned *extreme = (unsigned *)(counts + 4);
    long long *d_nrp = counts, *d_nsp = counts + 1, *d_out = counts + 2, *d_u = counts + 3;
    unsigned long long *rmask = (unsigned long long *)(counts + 6);
    // caching: sort buffers, distinct keys and the R' -> distinct map
    int *pos = nullptr, *tpos = nullptr, *map = nullptr;
    void *tkeys = nullptr, *ukeys = nullptr, *sscr = nullptr, *gscr = nullptr;
    unsigned *hist = nullptr, *dbase = nullptr;
    if (P->dedup) {
        pos = (int *)salloc(c, (size_t)nR * 4);
        tpos = (int *)salloc(c, (size_t)nR * 4);
        map = (int *)salloc(c, (size_t)nR * 4);
        tkeys = salloc(c, (size_t)nR * kb);
        ukeys = salloc(c, (size_t)nR * kb);
        sscr = salloc(c, ng::sort_scratch_bytes(nR));
        gscr = salloc(c, ng::group_scratch_bytes(nR));
        hist = (unsigned *)salloc(c, ng::hist_bytes());
        dbase = (unsigned *)salloc(c, 8 * 512 * 4);
        if (!pos || !tpos || !map || !tkeys || !ukeys || !sscr || !gscr || !hist || !dbase)
            return fail(c, NESTGPU_ERR_OOM, "arena exhausted (dedup buffers for |R|=%lld)", (long long)nR);
    }

    // Index aux arrays (built on first use and kept with the index) are
    // built here, outside the per-exec launch sequence: that sequence may be
    // a replayed CUDA graph, and a build changes host state (arena tail,
    // the index record) that a replay would not.
    const long long *pre = nullptr, *suf = nullptr;
    if (ix) {
        // Index-pruned evaluation (NEXT 3): prefix / suffix aggregates of the
        // payload make non-equality and SUM/AVG ranges O(1); built once per
        // index and aggregate kind, kept with the index.
        if (value_agg && (P->corr_op != NG_EQ || P->agg == NG_SUM || P->agg == NG_AVG)) {
            const int kind = P->agg == NG_MIN ? 0 : (P->agg == NG_MAX ? 1 : (wide ? 3 : 2));
            const int akind = kind == 0 ? ng::MIN : (kind == 1 ? ng::MAX : ng::SUM);
            if (!ix->aux_pre[kind]) {
                const size_t off = c->lo;
                long long *ap = (long long *)palloc(c, (size_t)(ix->n + 1) * 8);
                long long *as = kind != 2 ? (long long *)palloc(c, (size_t)(ix->n + 1) * 8) : nullptr;
                void *ascr = salloc(c, ng::index_aux_scratch_bytes(ix->n));
                if (!ap || (kind != 2 && !as) || !ascr) {
                    c->lo = off;
                    return fail(c, NESTGPU_ERR_OOM, "arena exhausted (index prefix aggregates)");
                }
                CUDA_TRY(c, ng::launch_index_aux(akind, ix->vb, ix->payload, ix->n, ap, kind == 3 ? nullptr : as, ascr,
                                                 c->stream, &c->launches, kind == 3 ? as : nullptr));
                ix->aux_pre[kind] = ap;
                ix->aux_suf[kind] = as;
                ix->aux_off[kind] = off;
            }
            pre = ix->aux_pre[kind];
            suf = ix->aux_suf[kind];
        } else if ((P->agg == NG_MIN || P->agg == NG_MAX) && ix->n > ng::RANGE_INLINE_MAX) {
            // '=' MIN/MAX: per-key group aggregates (segmented scan), so a hot
            // key's run is folded once per index, not once per outer tuple
            const int kind = P->agg == NG_MIN ? 4 : 5;
            if (!ix->aux_pre[kind]) {
                const size_t off = c->lo;
                long long *gp = (long long *)palloc(c, (size_t)(ix->n + 1) * 8);
                void *gscr2 = salloc(c, ng::index_aux_scratch_bytes(ix->n));
                if (!gp || !gscr2) {
                    c->lo = off;
                    return fail(c, NESTGPU_ERR_OOM, "arena exhausted (index group aggregates)");
                }
                CUDA_TRY(c, ng::launch_index_group_agg(kind == 4 ? ng::MIN : ng::MAX, ix->kb, ix->vb, ix->keys,
                                                       ix->payload, ix->n, gp, gscr2, c->stream, &c->launches));
                ix->aux_pre[kind] = gp;
                ix->aux_off[kind] = off;
            }
            pre = ix->aux_pre[kind];
        }
    }

    const long long krows = std::min<long long>(nR, (long long)(STAGE_BYTES / (8 * w8 + 2)));
    long long n_distinct = -1;
    // Tiny inputs: the nested-loop strategy's whole sequence as one launch of
    // one CTA (k_finalize.cu tiny_exec_kernel; NESTGPU_OPT_TINY, off when a
    // test forces a nested-loop R-block shape)
    const bool tiny = c->tiny_on && !ix && !P->dedup && c->bnl_shape == 0 && nS <= ng::TINY_S_MAX &&
                      nR <= ng::TINY_R_MAX && nR * nS <= ng::TINY_PAIRS_MAX;
    // Everything enqueued from here to the result copies: run directly, or
    // captured once into a CUDA graph and replayed (§17) -- a repeated small
    // query then costs one graph launch instead of one launch per kernel.
    auto enqueue = [&]() -> nestgpu_status {
      if (tiny) {
        prof_begin(c, 5);
        prof_begin(c, 3);
        ng::TinyArgs ta{};
        ta.nR = nR;
        ta.nS = nS;
        ta.rp = ops;
        ta.sp = ips;
        ta.rk = rks;
        ta.sk = sks;
        if (value_agg) ta.v = ng::ValSrc{ac->d, ac->valid, vb};
        ta.corr_op = P->corr_op;
        ng::FinalizeArgs &fa = ta.f;
        fa.x_col = xc ? xc->d : nullptr;
        fa.x_valid = xc ? xc->valid : nullptr;
        fa.x_w = xc ? dtype_width(xc->dtype) : 4;
        fa.agg = P->agg;
        fa.outer_op = P->outer_op;
        fa.a = P->lhs_mult;
        fa.b = P->rhs_mult;
        fa.row_id_base = P->row_id_base;
        fa.emit_all = P->emit_all;
        fa.out_ids = o_ids;
        fa.out_vals = o_vals;
        fa.out_sum = o_sum;
        fa.out_cnt = o_cnt;
        fa.out_valid = o_valid;
        fa.out_passed = o_pass;
        fa.out_count = d_out;
        ta.counts = counts;
        ta.status = (unsigned long long *)(counts + 16);
        CUDA_TRY(c, ng::launch_tiny_exec(ta, c->num_sms, c->stream, &c->launches));
        htrace(c, "tiny");
        prof_end(c, 3);
        prof_end(c, 5);
      } else {
        // ------------------------------------------------------------ a2: R'
        prof_begin(c, 5);
        prof_begin(c, 0);
        ng::ValSrc none{nullptr, nullptr, 0};
        {   // every small scratch region of this exec zeroed by ONE kernel
            ng::FillList fl;
            fl.add(counts, 48);
            fl.add(rmask, 8, 0xff);    // [6] AND identity
            fl.add(counts + 7, 8);     // [7] OR
            fl.add(counts + 8, 64);
            fl.add(fscr, ng::filter_zero_bytes(nR, true));
            if (fscr_s) fl.add(fscr_s, ng::filter_zero_bytes(nS, false));
            fl.add(fscr_f, ng::finalize_zero_bytes());
            fl.add(kscr, ix ? 256 : ng::bnl_scratch_bytes(nR));
            if (wide) fl.add(acc_hi, (size_t)nR * 8);
            if (!ix && nR <= SMALL_ROWS) {   // small R: the partials' identity init rides on the fill
                const long long acc0 = P->agg == NG_MIN ? LLONG_MAX : (P->agg == NG_MAX ? LLONG_MIN : 0);
                fl.add_words(acc, (size_t)nR * 8, (unsigned long long)acc0);
                fl.add(cnt, (size_t)nR * 8);
            }
            // the staged rows (copied to the host even when fewer survive):
            // defined contents for compute-sanitizer's initcheck
            const long long kr = std::min<long long>(nR, (long long)(STAGE_BYTES / (8 * w8 + 2)));
            for (size_t f = 0; f < w8; f++) fl.add(rblk + (size_t)nR * 8 * f, (size_t)kr * 8);
            fl.add(o_valid, (size_t)kr);
            fl.add(o_pass, (size_t)kr);
            htrace(c, "alloc");
            CUDA_TRY(c, ng::launch_fill(fl, c->stream, &c->launches));
            htrace(c, "fill");
        }
        CUDA_TRY(c, ng::launch_filter(nR, ops, rks, kb, none, 0, 0, 0, ids, rkeys, rkvalid, nullptr,
                                      P->dedup ? rmask : nullptr, nullptr, fscr, d_nrp, c->stream, &c->launches, true));
        htrace(c, "rfilter");
        prof_end(c, 0);

        // The keys the subquery kernels evaluate: every R' key, or (dedup) each
        // distinct R' key once -- P:331's cache keyed by the passed-in parameter.
        const void *eval_keys = rkeys;
        const long long *d_neval = d_nrp;
        long long n_eval = nR;
        if (P->dedup) {
            prof_begin(c, 2);
            CUDA_TRY(c, cudaMemcpyAsync(c->pinned, counts, 64, cudaMemcpyDeviceToHost, c->stream));
            CUDA_TRY(c, cudaStreamSynchronize(c->stream));
            long long nrp;
            unsigned long long kand, kor;
            memcpy(&nrp, c->pinned, 8);
            memcpy(&kand, c->pinned + 12, 8);
            memcpy(&kor, c->pinned + 14, 8);
            int shifts[8], rb = 8;
            const int np = plan_sort_passes(kb, kand, kor, nrp, shifts, &rb);
            CUDA_TRY(c, ng::launch_iota(pos, nrp, c->stream, &c->launches));
            CUDA_TRY(c, ng::launch_digit_hist(kb, rkeys, nrp, shifts, np, hist, dbase, c->num_sms, c->stream,
                                              &c->launches, rb));
            void *ck = rkeys, *ok = tkeys;
            int *cv = pos, *ov = tpos;
            const bool narrow = kb == 8 && np >= 2 && ((kand ^ kor) >> 32) == 0;   // as in build_index
            for (int p = 0; p < np; p++) {
                const int kin = narrow && p > 0 ? 4 : kb, kout = narrow && p < np - 1 ? 4 : kb;
                CUDA_TRY(c, ng::launch_radix_pass_x(kin, kout, 4, ck, ok, cv, ov, nrp, shifts[p], dbase + p * (1 << rb),
                                                    sscr, (unsigned)(kand >> 32), c->stream, &c->launches, rb));
                std::swap(ck, ok);
                std::swap(cv, ov);
            }
            CUDA_TRY(c, ng::launch_group(kb, ck, cv, nrp, ukeys, map, d_u, gscr, c->stream, &c->launches));
            CUDA_TRY(c, cudaMemcpyAsync(c->pinned, d_u, 8, cudaMemcpyDeviceToHost, c->stream));
            CUDA_TRY(c, cudaStreamSynchronize(c->stream));
            memcpy(&n_distinct, c->pinned, 8);
            eval_keys = ukeys;
            d_neval = d_u;
            n_eval = n_distinct;
            prof_end(c, 2);
        }

        // ------------------------------------------------------------ a3 / a5-a7
        if (ix) {
            prof_begin(c, 3);
            const bool split = wide && pre && P->agg != NG_MIN && P->agg != NG_MAX;
            CUDA_TRY(c, ng::launch_range_agg(kb, vb, P->corr_op, P->agg, n_eval, d_neval, eval_keys, ix->keys, ix->payload,
                                             ix->n, pre, split ? nullptr : suf, acc, cnt, kscr, c->stream, &c->launches,
                                             split ? suf : nullptr, split ? acc_hi : nullptr, true));
            htrace(c, "range");
            prof_end(c, 3);
        } else {
            prof_begin(c, 1);
            ng::ValSrc vs{nullptr, nullptr, 0};
            if (value_agg) { vs.c = ac->d; vs.v = ac->valid; vs.w = vb; }
            CUDA_TRY(c, ng::launch_filter(nS, ips, sks, kb, vs, vb, 1, value_agg ? 1 : 0, nullptr, skeys, nullptr, svals,
                                          nullptr, value_agg ? extreme : nullptr, fscr_s, d_nsp, c->stream,
                                          &c->launches, true));
            htrace(c, "sfilter");
            if (nR > SMALL_ROWS)
                CUDA_TRY(c, ng::launch_init_partials(n_eval, d_neval, P->agg, acc, cnt, c->stream, &c->launches));
            htrace(c, "init");
            prof_end(c, 1);
            prof_begin(c, 3);
            CUDA_TRY(c, ng::launch_bnl(kb, vb, P->corr_op, P->agg, n_eval, d_neval, eval_keys, nS, d_nsp, skeys, svals,
                                       extreme, acc, cnt, kscr, c->num_sms, c->bnl_shape, c->stream, &c->launches,
                                       wide ? acc_hi : nullptr, true));
            htrace(c, "bnl");
            prof_end(c, 3);
        }

        // ------------------------------------------------------------ a8 + a9
        prof_begin(c, 4);
        ng::FinalizeArgs fa{};
        fa.n_rp_max = nR;
        fa.d_nrp = d_nrp;
        fa.ids = ids;
        fa.map = map;
        fa.kvalid = rkvalid;
        fa.acc = acc;
        fa.cnt = cnt;
        fa.acc_hi = wide ? acc_hi : nullptr;
        fa.overflow = (unsigned long long *)(counts + 8);
        fa.x_col = xc ? xc->d : nullptr;
        fa.x_valid = xc ? xc->valid : nullptr;
        fa.x_w = xc ? dtype_width(xc->dtype) : 4;
        fa.agg = P->agg;
        fa.outer_op = P->outer_op;
        fa.a = P->lhs_mult;
        fa.b = P->rhs_mult;
        fa.row_id_base = P->row_id_base;
        fa.emit_all = P->emit_all;
        fa.out_ids = o_ids;
        fa.out_vals = o_vals;
        fa.out_sum = o_sum;
        fa.out_cnt = o_cnt;
        fa.out_valid = o_valid;
        fa.out_passed = o_pass;
        fa.out_count = d_out;
        fa.scratch = fscr_f;
        CUDA_TRY(c, ng::launch_finalize(fa, c->stream, &c->launches, true));
        htrace(c, "finalize");
        prof_end(c, 4);
        prof_end(c, 5);
      }
        CUDA_TRY(c, cudaMemcpyAsync(c->pinned, counts, 72, cudaMemcpyDeviceToHost, c->stream));
        // the first rows of every result field, staged on the host before the
        // one synchronisation (8-byte fields, then the two byte fields)
        if (krows == nR && krows > 0) {   // the whole result block fits: one copy, same layout
            CUDA_TRY(c, cudaMemcpyAsync(c->stage, rblk, (size_t)nR * (8 * w8 + 2), cudaMemcpyDeviceToHost, c->stream));
        } else if (krows > 0) {
            CUDA_TRY(c, cudaMemcpy2DAsync(c->stage, (size_t)krows * 8, rblk, (size_t)nR * 8, (size_t)krows * 8, w8,
                                          cudaMemcpyDeviceToHost, c->stream));
            CUDA_TRY(c, cudaMemcpy2DAsync(c->stage + (size_t)krows * 8 * w8, (size_t)krows, o_valid, (size_t)nR,
                                          (size_t)krows, 2, cudaMemcpyDeviceToHost, c->stream));
        }
        return NESTGPU_OK;
    };
    if (graph_ok(c, P, ix)) {
        nestgpu_status gs = run_graph(c, exec_graph_key(c, P, ix, wide), enqueue);
        if (gs) return gs;
    } else {
        nestgpu_status es = enqueue();
        if (es) return es;
    }
    htrace(c, "copies");
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    htrace(c, "sync");
    long long cnts[9];
    memcpy(cnts, c->pinned, 72);
    if (cnts[8]) return fail(c, NESTGPU_ERR_OVERFLOW, "exec: a SUM exceeds int64 (reading R5)");
    c->staged.ok = krows > 0;
    c->staged.ids = o_ids;
    c->staged.rows = krows;
    c->staged.w8 = w8;
    out->n_rows = cnts[2];
    out->n_evaluated = P->dedup ? n_distinct : cnts[0];
    out->d_row_ids = (const int64_t *)o_ids;
    out->d_values = (const int64_t *)o_vals;
    out->d_valid = o_valid;
    out->d_passed = o_pass;
    out->d_avg_sum = (const int64_t *)o_sum;
    out->d_avg_cnt = (const int64_t *)o_cnt;
    htrace_end(c, "exec");
    return NESTGPU_OK;
}

nestgpu_status nestgpu_result_to_host(nestgpu_ctx *c, const nestgpu_result *r, int64_t *row_ids, int64_t *values,
                                      uint8_t *valid, uint8_t *passed, int64_t *avg_sum, int64_t *avg_cnt, int64_t cap)
{
    if (!c || !r) return fail(c, NESTGPU_ERR_INVALID, "result_to_host: null argument");
    if (cap < r->n_rows) return fail(c, NESTGPU_ERR_BUFFER, "result_to_host: %lld rows, buffer holds %lld", (long long)r->n_rows, (long long)cap);
    cudaSetDevice(c->device);
    const size_t n = (size_t)r->n_rows;
    if (c->staged.ok && r->d_row_ids == c->staged.ids && r->n_rows <= c->staged.rows) {
        // staged by exec: host copies only, no GPU operation
        const size_t k = (size_t)c->staged.rows;
        const char *s = c->stage;
        if (n) {
            if (row_ids) memcpy(row_ids, s, n * 8);
            if (values) memcpy(values, s + k * 8, n * 8);
            if (avg_sum && r->d_avg_sum) memcpy(avg_sum, s + k * 16, n * 8);
            if (avg_cnt && r->d_avg_cnt) memcpy(avg_cnt, s + k * 24, n * 8);
            if (valid) memcpy(valid, s + k * 8 * c->staged.w8, n);
            if (passed) memcpy(passed, s + k * 8 * c->staged.w8 + k, n);
        }
        return NESTGPU_OK;
    }
    if (n) {
        if (row_ids) CUDA_TRY(c, cudaMemcpyAsync(row_ids, r->d_row_ids, n * 8, cudaMemcpyDeviceToHost, c->stream));
        if (values) CUDA_TRY(c, cudaMemcpyAsync(values, r->d_values, n * 8, cudaMemcpyDeviceToHost, c->stream));
        if (valid) CUDA_TRY(c, cudaMemcpyAsync(valid, r->d_valid, n, cudaMemcpyDeviceToHost, c->stream));
        if (passed) CUDA_TRY(c, cudaMemcpyAsync(passed, r->d_passed, n, cudaMemcpyDeviceToHost, c->stream));
        if (avg_sum && r->d_avg_sum) CUDA_TRY(c, cudaMemcpyAsync(avg_sum, r->d_avg_sum, n * 8, cudaMemcpyDeviceToHost, c->stream));
        if (avg_cnt && r->d_avg_cnt) CUDA_TRY(c, cudaMemcpyAsync(avg_cnt, r->d_avg_cnt, n * 8, cudaMemcpyDeviceToHost, c->stream));
    }
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    return NESTGPU_OK;
}

// ---------------------------------------------------------------- type-J results
nestgpu_status nestgpu_exec_collect(nestgpu_ctx *c, const nestgpu_plan *P, nestgpu_collection *out)
{
    if (!c || !P || !out) return fail(c, NESTGPU_ERR_INVALID, "exec_collect: null argument");
    cudaSetDevice(c->device);
    memset(out, 0, sizeof *out);
    if (!valid_op(P->corr_op)) return fail(c, NESTGPU_ERR_INVALID, "exec_collect: bad correlated operator");
    if (P->n_key_cols == 2 && P->corr_op != NG_EQ)
        return fail(c, NESTGPU_ERR_UNSUPPORTED, "exec_collect: composite correlation supports '=' only");
    if (P->index < 0)
        return fail(c, NESTGPU_ERR_UNSUPPORTED, "exec_collect: type-J results are built from an index (plan.index >= 0)");
    ng::KeySrc rks, sks;
    int64_t nR, nS;
    nestgpu_status s;
    if ((s = make_key(c, P->outer_key_cols, P->n_key_cols, nR, rks, "outer key"))) return s;
    if ((s = make_key(c, P->inner_key_cols, P->n_key_cols, nS, sks, "inner key"))) return s;
    ng::PredSet ops;
    if ((s = make_preds(c, P->outer_preds, P->n_outer_preds, nR, ops, "outer_preds"))) return s;
    if (P->index >= (int32_t)c->idx.size() || !c->idx[P->index].alive)
        return fail(c, NESTGPU_ERR_INVALID, "exec_collect: unknown index %d", P->index);
    IndexRec *ix = &c->idx[P->index];
    if (ix->n_key != P->n_key_cols || ix->key_cols[0] != P->inner_key_cols[0] ||
        (P->n_key_cols == 2 && ix->key_cols[1] != P->inner_key_cols[1]))
        return fail(c, NESTGPU_ERR_INVALID, "exec_collect: index %d is on different key columns", P->index);
    if (!same_preds(P->inner_preds, P->n_inner_preds, ix->inner))
        return fail(c, NESTGPU_ERR_INVALID, "exec_collect: index %d was built with different inner predicates", P->index);
    if (ix->vb == 0 || ix->payload_col != P->agg_col)
        return fail(c, NESTGPU_ERR_INVALID, "exec_collect: index %d must carry the selected column %d as payload",
                    P->index, P->agg_col);
    const int rkb = key_bytes(c, P->outer_key_cols, P->n_key_cols);
    const int kb = (rkb == 8 || ix->kb == 8) ? 8 : 4;
    if (ix->kb != kb)
        return fail(c, NESTGPU_ERR_UNSUPPORTED, "exec_collect: outer key is 64-bit but index %d has 32-bit keys", P->index);

    scratch_reset(c);
    for (int st = 0; st < NESTGPU_N_STAGES; st++) c->ran[st] = false;
    const bool ravalid = rks.v0 || rks.v1;
    int *ids = (int *)salloc(c, (size_t)nR * 4);
    void *rkeys = salloc(c, (size_t)nR * kb);
    uint8_t *rkvalid = ravalid ? (uint8_t *)salloc(c, (size_t)nR) : nullptr;
    long long *counts = (long long *)salloc(c, 64);   // [0] |R'| [1] level-2 total
    void *fscr = salloc(c, ng::filter_scratch_bytes(nR));
    void *cscr = salloc(c, ng::collect_scratch_bytes(nR));
    long long *lens = (long long *)salloc(c, (size_t)nR * 8);
    long long *row_ids = (long long *)salloc(c, (size_t)nR * 8);
    long long *offsets = (long long *)salloc(c, (size_t)(nR + 1) * 8);
    if (!ids || !rkeys || (ravalid && !rkvalid) || !counts || !fscr || !cscr || !lens || !row_ids || !offsets)
        return fail(c, NESTGPU_ERR_OOM, "arena exhausted collecting over |R|=%lld", (long long)nR);
    ng::ValSrc none{nullptr, nullptr, 0};
    prof_begin(c, 5);
    prof_begin(c, 0);
    CUDA_TRY(c, cudaMemsetAsync(counts, 0, 64, c->stream));
    CUDA_TRY(c, ng::launch_filter(nR, ops, rks, kb, none, 0, 0, 0, ids, rkeys, rkvalid, nullptr, nullptr, nullptr,
                                  fscr, counts, c->stream, &c->launches));
    prof_end(c, 0);
    prof_begin(c, 3);
    CUDA_TRY(c, ng::launch_collect_bounds(kb, P->corr_op, nR, counts, ids, rkeys, rkvalid, ix->keys, ix->n,
                                          P->row_id_base, cscr, lens, row_ids, offsets, counts + 1, c->stream,
                                          &c->launches));
    CUDA_TRY(c, cudaMemcpyAsync(c->pinned, counts, 16, cudaMemcpyDeviceToHost, c->stream));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    long long nc[2];
    memcpy(nc, c->pinned, 16);
    long long *vals = (long long *)salloc(c, (size_t)(nc[1] > 0 ? nc[1] : 1) * 8);
    long long *owner = (long long *)salloc(c, (size_t)(nc[1] > 0 ? nc[1] : 1) * 8);
    if (!vals || !owner)
        return fail(c, NESTGPU_ERR_OOM, "arena exhausted: the type-J result has %lld values", nc[1]);
    CUDA_TRY(c, ng::launch_collect_fill(ix->vb, counts, offsets, cscr, row_ids, ix->payload, nc[1], vals, owner,
                                        c->stream, &c->launches));
    prof_end(c, 3);
    prof_end(c, 5);
    CUDA_TRY(c, cudaGetLastError());
    out->n_outer = nc[0];
    out->n_values = nc[1];
    out->d_row_ids = (const int64_t *)row_ids;
    out->d_offsets = (const int64_t *)offsets;
    out->d_values = (const int64_t *)vals;
    out->d_owner = (const int64_t *)owner;
    return NESTGPU_OK;
}

nestgpu_status nestgpu_collection_in(nestgpu_ctx *c, const nestgpu_collection *coll, int32_t x_col,
                                     int64_t row_id_base, int32_t emit_all, nestgpu_result *out)
{
    if (!c || !coll || !out) return fail(c, NESTGPU_ERR_INVALID, "collection_in: null argument");
    cudaSetDevice(c->device);
    memset(out, 0, sizeof *out);
    const long long n = coll->n_outer;
    if (n < 0 || coll->n_values < 0 || (n > 0 && (!coll->d_row_ids || !coll->d_offsets)) ||
        (coll->n_values > 0 && !coll->d_values))
        return fail(c, NESTGPU_ERR_INVALID, "collection_in: malformed collection");
    const Column *xc = col_get(c, x_col);
    if (!xc) return fail(c, NESTGPU_ERR_INVALID, "collection_in: unknown column %d", x_col);
    // scratch grows below the collection (which must stay intact)
    int *ids32 = (int *)salloc(c, (size_t)n * 4);
    long long *cnt = (long long *)salloc(c, (size_t)n * 8);
    long long *acc = (long long *)salloc(c, (size_t)n * 8);
    long long *small = (long long *)salloc(c, 64);   // [0] n  [2] survivors
    void *fscr = salloc(c, ng::filter_scratch_bytes(n));
    long long *o_ids = (long long *)salloc(c, (size_t)n * 8);
    long long *o_vals = (long long *)salloc(c, (size_t)n * 8);
    uint8_t *o_valid = (uint8_t *)salloc(c, (size_t)n);
    uint8_t *o_pass = (uint8_t *)salloc(c, (size_t)n);
    if (!ids32 || !cnt || !acc || !small || !fscr || !o_ids || !o_vals || !o_valid || !o_pass)
        return fail(c, NESTGPU_ERR_OOM, "arena exhausted (collection_in over %lld lists)", n);
    memcpy(c->pinned + 8 * 256 + 8, &n, 8);
    CUDA_TRY(c, cudaMemcpyAsync(small, c->pinned + 8 * 256 + 8, 8, cudaMemcpyHostToDevice, c->stream));
    if (n > 0) CUDA_TRY(c, cudaMemsetAsync(acc, 0, (size_t)n * 8, c->stream));
    CUDA_TRY(c, ng::launch_in_list(n, (const long long *)coll->d_row_ids, (const long long *)coll->d_offsets,
                                   (const long long *)coll->d_values, xc->d, dtype_width(xc->dtype), xc->valid,
                                   row_id_base, ids32, cnt, c->stream, &c->launches));
    ng::FinalizeArgs fa{};
    fa.n_rp_max = n;
    fa.d_nrp = small;
    fa.ids = ids32;
    fa.acc = acc;
    fa.cnt = cnt;
    fa.x_w = 4;
    fa.agg = NG_EXISTS;
    fa.outer_op = NG_EQ;
    fa.a = fa.b = 1;
    fa.row_id_base = row_id_base;
    fa.emit_all = emit_all;
    fa.out_ids = o_ids;
    fa.out_vals = o_vals;
    fa.out_valid = o_valid;
    fa.out_passed = o_pass;
    fa.out_count = small + 2;
    fa.scratch = fscr;
    CUDA_TRY(c, ng::launch_finalize(fa, c->stream, &c->launches));
    CUDA_TRY(c, cudaMemcpyAsync(c->pinned, small + 2, 8, cudaMemcpyDeviceToHost, c->stream));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    long long m;
    memcpy(&m, c->pinned, 8);
    out->n_rows = m;
    out->n_evaluated = n;
    out->d_row_ids = (const int64_t *)o_ids;
    out->d_values = (const int64_t *)o_vals;
    out->d_valid = o_valid;
    out->d_passed = o_pass;
    return NESTGPU_OK;
}

nestgpu_status nestgpu_column_from_device(nestgpu_ctx *c, nestgpu_dtype dtype, int32_t scale, const int64_t *d_src,
                                          const uint8_t *d_valid, int64_t n, int32_t *out_col)
{
    if (!c || !out_col || (n > 0 && !d_src)) return fail(c, NESTGPU_ERR_INVALID, "column_from_device: null argument");
    cudaSetDevice(c->device);
    const int w = dtype_width(dtype);
    const size_t off = c->lo;
    int32_t id;
    nestgpu_status s = new_column(c, dtype, scale, n, d_valid != nullptr, &id);
    if (s) return s;
    unsigned long long *bad = nullptr;
    if (w == 4) {
        bad = (unsigned long long *)salloc(c, 8);
        if (!bad) {
            c->cols[id].alive = false;
            c->lo = off;
            return fail(c, NESTGPU_ERR_OOM, "arena exhausted (column_from_device)");
        }
        CUDA_TRY(c, cudaMemsetAsync(bad, 0, 8, c->stream));
    }
    Column &col = c->cols[id];
    CUDA_TRY(c, ng::launch_materialize(w, (const long long *)d_src, d_valid, n, col.d, col.valid, bad, c->stream,
                                       &c->launches));
    if (w == 4) {
        CUDA_TRY(c, cudaMemcpyAsync(c->pinned, bad, 8, cudaMemcpyDeviceToHost, c->stream));
        CUDA_TRY(c, cudaStreamSynchronize(c->stream));
        unsigned long long nb;
        memcpy(&nb, c->pinned, 8);
        if (nb) {
            c->cols[id].alive = false;
            c->lo = off;
            return fail(c, NESTGPU_ERR_OVERFLOW, "column_from_device: %llu values do not fit a 4-byte column", nb);
        }
    }
    *out_col = id;
    return NESTGPU_OK;
}

// ---------------------------------------------------------------- peer windows
static_assert(sizeof(nestgpu_ipc_handle) == sizeof(cudaIpcMemHandle_t), "IPC handle size");

nestgpu_status nestgpu_window_create(nestgpu_ctx *c, int64_t cap, void **d_window, nestgpu_ipc_handle *out)
{
    if (!c || !d_window || !out || cap < 0) return fail(c, NESTGPU_ERR_INVALID, "window_create: bad argument");
    cudaSetDevice(c->device);
    void *p = nullptr;
    CUDA_TRY(c, cudaMalloc(&p, (size_t)(cap > 0 ? cap : 1) * 16));
    cudaIpcMemHandle_t h;
    cudaError_t e = cudaIpcGetMemHandle(&h, p);
    if (e != cudaSuccess) {
        cudaFree(p);
        return fail(c, NESTGPU_ERR_CUDA, "window_create: cudaIpcGetMemHandle: %s", cudaGetErrorString(e));
    }
    memcpy(out->bytes, &h, sizeof h);
    *d_window = p;
    return NESTGPU_OK;
}

nestgpu_status nestgpu_window_open(nestgpu_ctx *c, const nestgpu_ipc_handle *handle, void **d_peer)
{
    if (!c || !handle || !d_peer) return fail(c, NESTGPU_ERR_INVALID, "window_open: null argument");
    cudaSetDevice(c->device);
    cudaIpcMemHandle_t h;
    memcpy(&h, handle->bytes, sizeof h);
    void *p = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) return fail(c, NESTGPU_ERR_CUDA, "window_open: cudaIpcOpenMemHandle: %s", cudaGetErrorString(e));
    *d_peer = p;
    return NESTGPU_OK;
}

nestgpu_status nestgpu_window_close(nestgpu_ctx *c, void *d_peer)
{
    if (!c || !d_peer) return NESTGPU_ERR_INVALID;
    cudaSetDevice(c->device);
    CUDA_TRY(c, cudaIpcCloseMemHandle(d_peer));
    return NESTGPU_OK;
}

nestgpu_status nestgpu_window_free(nestgpu_ctx *c, void *d_window)
{
    if (!c || !d_window) return NESTGPU_ERR_INVALID;
    cudaSetDevice(c->device);
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    CUDA_TRY(c, cudaFree(d_window));
    return NESTGPU_OK;
}

nestgpu_status nestgpu_result_put(nestgpu_ctx *c, const nestgpu_result *r, void *d_window, int64_t cap, int64_t offset)
{
    if (!c || !r || !d_window || cap < 0 || offset < 0) return fail(c, NESTGPU_ERR_INVALID, "result_put: bad argument");
    if (offset + r->n_rows > cap)
        return fail(c, NESTGPU_ERR_INVALID, "result_put: rows [%lld, %lld) outside the window's %lld", (long long)offset,
                    (long long)(offset + r->n_rows), (long long)cap);
    cudaSetDevice(c->device);
    long long *wi = (long long *)d_window + offset;
    long long *wv = (long long *)d_window + cap + offset;
    CUDA_TRY(c, ng::launch_put_rows((const long long *)r->d_row_ids, (const long long *)r->d_values, r->n_rows, wi,
                                    wv, c->stream, &c->launches));
    CUDA_TRY(c, cudaStreamSynchronize(c->stream));
    return NESTGPU_OK;
}

nestgpu_status nestgpu_set_option(nestgpu_ctx *c, int32_t option, int64_t value)
{
    if (!c) return NESTGPU_ERR_INVALID;
    switch (option) {
    case NESTGPU_OPT_MALLOC_SCRATCH:
        cudaSetDevice(c->device);
        scratch_reset(c);
        c->malloc_scratch = value != 0;
        return NESTGPU_OK;
    case NESTGPU_OPT_BNL_SHAPE:
        if (value < 0 || value > 2) return fail(c, NESTGPU_ERR_INVALID, "set_option: BNL shape 0, 1 or 2");
        c->bnl_shape = (int)value;
        return NESTGPU_OK;
    case NESTGPU_OPT_GRAPHS:
        c->graphs_on = value != 0;
        return NESTGPU_OK;
    case NESTGPU_OPT_TINY:
        c->tiny_on = value != 0;
        return NESTGPU_OK;
    case NESTGPU_OPT_SORT:
        if (value < 0 || value > 2) return fail(c, NESTGPU_ERR_INVALID, "set_option: sort 0, 1 or 2");
        c->sort_mode = (int)value;
        return NESTGPU_OK;
    }
    return fail(c, NESTGPU_ERR_INVALID, "set_option: unknown option %d", option);
}

nestgpu_status nestgpu_set_profiling(nestgpu_ctx *c, int32_t on)
{
    if (!c) return NESTGPU_ERR_INVALID;
    c->profiling = on != 0;
    return NESTGPU_OK;
}

nestgpu_status nestgpu_last_profile(const nestgpu_ctx *c, float *ms, int32_t n)
{
    if (!c || !ms) return NESTGPU_ERR_INVALID;
    cudaSetDevice(c->device);
    for (int s = 0; s < n && s < NESTGPU_N_STAGES; s++) {
        ms[s] = NAN;
        if (c->profiling && c->ran[s]) {
            float t;
            if (cudaEventSynchronize(c->ev[s][1]) == cudaSuccess &&
                cudaEventElapsedTime(&t, c->ev[s][0], c->ev[s][1]) == cudaSuccess)
                ms[s] = t;
        }
    }
    return NESTGPU_OK;
}

}  // extern "C"
