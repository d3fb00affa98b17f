/*
 * nestgpu.h -- C ABI of the B200-native nested-method correlated-subquery
 * engine (libnestgpu.so, sm_100a).
 *
 * The operation (Fig. 2, §II-D; Fig. 4, P:175-183,
 * §III-B): for every outer tuple r of R that passes the outer local
 * predicates, evaluate the subquery over S with r's correlated value bound in
 * ("subquery(r.c1)"), store the scalar result in Res[i],
 * then keep r iff the predicate on Res holds ("Selection(=, R.col1, Res)",
 * P:183) and compact the survivors.  Template (north_star):
 *
 *   SELECT R.* FROM R
 *   WHERE <outer_preds(R)>
 *     AND lhs_mult*R.cmp <outer_op> rhs_mult*(SELECT AGG(S.agg) FROM S
 *            WHERE <inner_preds(S)> AND R.key <corr_op> S.key)
 *   -- or AND [NOT] EXISTS (SELECT * FROM S WHERE ...)
 *
 * The three entry points named by the north star are nestgpu_load_column
 * (LoadToGPU), nestgpu_build_index (the sorted correlated-column
 * index, §III-D "Indexing") and nestgpu_exec_correlated (the
 * vectorised subquery loop, §III-D "Vectorization").  The rest manage
 * the context, the memory pool (§III-C) and results.
 *
 * Conventions
 *  - Every call returns nestgpu_status: 0 = OK, < 0 = error.  The message of
 *    the last error is kept per context (nestgpu_last_error).  No exception,
 *    abort() or CPU fallback ever crosses this boundary: if the device work
 *    cannot be done, the call fails.
 *  - Device memory and the CUDA stream are OWNED BY THE CALLER.  The library
 *    carves every allocation out of the caller's arena (no cudaMalloc on any
 *    path) and enqueues all work on the caller's stream.
 *  - Host buffers passed in are borrowed for the duration of the call only.
 *  - Column / index ids and result pointers belong to the context.  Result
 *    device pointers stay valid until the next exec or release.
 *  - A context is not thread-safe; use one per host thread / GPU.
 *  - Semantics follow SQL-92 where the paper is silent (DESIGN.md readings
 *    R1-R11): NULL compares UNKNOWN (not TRUE); an empty subquery gives
 *    NULL for MIN/MAX/SUM/AVG, 0 for COUNT(*), false for EXISTS.
 */
#ifndef NESTGPU_H
#define NESTGPU_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define NESTGPU_ABI_VERSION 3

typedef int32_t nestgpu_status;
enum {
    NESTGPU_OK = 0,
    NESTGPU_ERR_INVALID = -1,      /* bad argument / id / plan (nothing launched) */
    NESTGPU_ERR_OOM = -2,          /* the caller's arena is exhausted */
    NESTGPU_ERR_TYPE = -3,         /* dtype mismatch */
    NESTGPU_ERR_UNSUPPORTED = -4,  /* valid SQL outside this engine's template */
    NESTGPU_ERR_OVERFLOW = -5,     /* an exact SUM leaves int64 (reading R5) */
    NESTGPU_ERR_CUDA = -6,         /* a CUDA runtime call or launch failed */
    NESTGPU_ERR_BUFFER = -7        /* caller's host buffer too small */
};

/* Column storage types (columnar store).  Decimals are scaled
 * integers; dates are int32 days since 1970-01-01 (reading R11). */
typedef enum {
    NG_INT32 = 0,     /* int32 */
    NG_INT64 = 1,     /* int64 */
    NG_DECIMAL = 2,   /* int64, value * 10^scale */
    NG_DATE = 3,      /* int32 days since 1970-01-01 */
    NG_DECIMAL32 = 4  /* int32, value * 10^scale (fits when |value*10^scale| < 2^31) */
} nestgpu_dtype;

/* Comparison operators.  A correlated predicate always reads
 * outer.key OP inner.key (reading R8). */
typedef enum { NG_EQ = 0, NG_NE = 1, NG_LT = 2, NG_LE = 3, NG_GT = 4, NG_GE = 5 } nestgpu_cmp;

/* Aggregates (type-JA subqueries; EXISTS as semi-join). */
typedef enum {
    NG_MIN = 0, NG_MAX = 1, NG_SUM = 2,
    NG_COUNT = 3,       /* COUNT(*) over qualifying S rows */
    NG_AVG = 4,         /* exact: compared as a*x*nn OP b*sum (reading R6) */
    NG_EXISTS = 5, NG_NOT_EXISTS = 6
} nestgpu_agg;

typedef struct nestgpu_ctx nestgpu_ctx;   /* opaque */

/* Local predicate on one table: col OP literal (rhs_col < 0) or col OP rhs_col.
 * Columns are compared as int64 values (int32 storage is widened). */
typedef struct {
    int32_t col;
    nestgpu_cmp op;
    int64_t literal;
    int32_t rhs_col;
} nestgpu_pred;

/* ---------------------------------------------------------------- context */

/* Create a context on `device` over the caller's device buffer
 * [d_arena, d_arena + arena_bytes) (>= 1 MiB, 256-B aligned) and the
 * caller's cudaStream_t `cuda_stream` (NULL = legacy default stream).
 * The library never frees d_arena.  Errors: INVALID, CUDA. */
nestgpu_status nestgpu_create(int device, void *d_arena, size_t arena_bytes,
                              void *cuda_stream, nestgpu_ctx **out);
/* Destroy the context (waits for its stream).  NULL is a no-op. */
nestgpu_status nestgpu_destroy(nestgpu_ctx *ctx);
/* Message of the last failed call on ctx ("" if none).  Owned by ctx. */
const char *nestgpu_last_error(const nestgpu_ctx *ctx);
/* Number of kernels this context has launched since creation. */
int64_t nestgpu_launch_count(const nestgpu_ctx *ctx);
/* Switch the stream subsequent calls enqueue on.  Work already queued on the
 * old stream is ordered before anything enqueued afterwards (the new stream
 * waits on an event recorded on the old one; no host synchronisation).
 * Errors: INVALID, CUDA. */
nestgpu_status nestgpu_set_stream(nestgpu_ctx *ctx, void *cuda_stream);

/* Memory pool (Fig. 7: "record where to free", then move the
 * tail back).  nestgpu_mark returns the current tail of the persistent side of
 * the arena; nestgpu_release drops every column, index and result created
 * after that mark.  Column and index ids are slots: the id of a dropped /
 * released object is handed to the next object created, so a
 * load -> build -> exec -> release loop keeps reusing the same ids (a plan
 * struct built once stays valid) and the host tables stay bounded; an id
 * kept past its object's release may name a newer object.  Errors: INVALID. */
nestgpu_status nestgpu_mark(nestgpu_ctx *ctx, uint64_t *out_mark);
nestgpu_status nestgpu_release(nestgpu_ctx *ctx, uint64_t mark);
/* Bytes in use (persistent + scratch) and the high-water mark. */
nestgpu_status nestgpu_arena_usage(const nestgpu_ctx *ctx, size_t *in_use, size_t *peak);

/* ---------------------------------------------------------------- columns */

/* LoadToGPU: copy n host values (and optional validity bytes,
 * host_valid[i] == 0 means NULL; NULL pointer = NOT NULL column) into the
 * arena, asynchronously on the context stream; the call returns after the
 * copy has been enqueued AND completed (the host buffers are borrowed for the
 * call only; pinned host memory makes the copy a DMA).  Values are stored in
 * the dtype's width; `scale` is metadata for NG_DECIMAL / NG_DECIMAL32.
 * n must be < 2^31.  Returns the new column id.  Errors: INVALID, OOM, CUDA. */
nestgpu_status nestgpu_load_column(nestgpu_ctx *ctx, nestgpu_dtype dtype, int32_t scale,
                                   const void *host_values, const uint8_t *host_valid,
                                   int64_t n, int32_t *out_col);
/* Reserve an uninitialised column (contents to be filled by the caller on
 * the device, e.g. by an NCCL broadcast into nestgpu_column_info's pointers).
 * with_valid != 0 reserves a validity byte array too. */
nestgpu_status nestgpu_alloc_column(nestgpu_ctx *ctx, nestgpu_dtype dtype, int32_t scale,
                                    int64_t n, int32_t with_valid, int32_t *out_col);
typedef struct {
    nestgpu_dtype dtype;
    int32_t scale;
    int64_t n;
    void *d_values;      /* n * (4|8) bytes */
    uint8_t *d_valid;    /* n bytes or NULL */
} nestgpu_column_desc;
nestgpu_status nestgpu_column_info(const nestgpu_ctx *ctx, int32_t col, nestgpu_column_desc *out);
/* Materialise a NOT NULL column of n values from row ids on the device:
 * out[i] = src_col[d_row_ids[i] - row_id_base].  This is the data flow between
 * the levels of a multi-level nested query (Fig. 6: a level's result
 * vector feeds the block above it): pass a result's d_row_ids / n_rows and the
 * row_id_base its plan used.  d_row_ids is borrowed for the call (it may be a
 * result's pointer, valid until the next exec).  src_col must have no NULLs.
 * Errors: INVALID, OOM, CUDA. */
nestgpu_status nestgpu_gather_column(nestgpu_ctx *ctx, int32_t src_col, const int64_t *d_row_ids, int64_t n,
                                     int64_t row_id_base, int32_t *out_col);

/* ---------------------------------------------------------------- index */

/* Build the correlated-column index of P:315 over S' = rows of S whose
 * inner_preds are all TRUE ("invariant component", executed once):
 * a stable device radix sort of S' by the correlated key, carrying the
 * aggregate payload.  key_cols: 1 column (int32/int64/date/decimal) or 2
 * int32-storage columns (composite '=' key, packed; reading R9).
 * payload_col: the column a MIN/MAX/SUM/AVG plan aggregates, or -1 (COUNT /
 * EXISTS need none).  Rows with a NULL key component are dropped (they
 * satisfy no correlated predicate); rows with a NULL payload are dropped too
 * (MIN/MAX/SUM/AVG skip them), so an index with a nullable payload column
 * cannot serve COUNT/EXISTS plans.  All columns must have S's row count.
 * A NOT NULL single key column stored in ascending order (checked once per
 * column with its min / max statistics; every build for a column created by
 * nestgpu_alloc_column) with a NOT NULL payload needs no sort: S' is
 * compacted in row order straight into the index (the stable sort of a
 * sorted S' is the identity; same bytes).
 * Synchronises the stream once (to size the sort or the index) -- not at
 * all for an index over all of S (no inner predicates, NOT NULL key and
 * payload: the radix plan comes from the key column's statistics) -- plus
 * once when a key column's statistics are computed.  UNSUPPORTED when a sort
 * would see |S'| >= 2^30 rows (columns hold < 2^31).
 * Errors: INVALID, TYPE, UNSUPPORTED, OOM, CUDA. */
nestgpu_status nestgpu_build_index(nestgpu_ctx *ctx, const int32_t *key_cols, int32_t n_key_cols,
                                   int32_t payload_col,
                                   const nestgpu_pred *inner_preds, int32_t n_inner_preds,
                                   int32_t *out_index);
/* Drop an index (its arena bytes are reclaimed at the next release of a
 * mark taken before it was built). */
nestgpu_status nestgpu_drop_index(nestgpu_ctx *ctx, int32_t index);

/* Device layout of an index, for the multi-GPU broadcast (sorted keys are
 * order-preserving unsigned encodings: int32 k -> (uint32)k ^ 0x80000000,
 * int64 k -> (uint64)k ^ 2^63, composite (k1,k2) -> enc32(k1) << 32 | enc32(k2)). */
typedef struct {
    int64_t n;              /* |S'| */
    int32_t key_bytes;      /* 4 or 8 */
    int32_t payload_bytes;  /* 0, 4 or 8 */
    void *d_keys;           /* n * key_bytes, ascending */
    void *d_payload;        /* n * payload_bytes, co-sorted, or NULL */
} nestgpu_index_desc;
nestgpu_status nestgpu_index_info(const nestgpu_ctx *ctx, int32_t index, nestgpu_index_desc *out);
/* Receiving rank of a broadcast: create an index with the given shape whose
 * contents the caller fills on the device (d_keys / d_payload of *out after
 * the call).  key_cols / payload_col / inner_preds describe what it indexes
 * (they are validated against plans exactly as for nestgpu_build_index). */
nestgpu_status nestgpu_index_create_empty(nestgpu_ctx *ctx, int64_t n, int32_t key_bytes,
                                          int32_t payload_bytes,
                                          const int32_t *key_cols, int32_t n_key_cols,
                                          int32_t payload_col,
                                          const nestgpu_pred *inner_preds, int32_t n_inner_preds,
                                          nestgpu_index_desc *out, int32_t *out_index);

/* ---------------------------------------------------------------- exec */

typedef struct {
    const nestgpu_pred *outer_preds; int32_t n_outer_preds;   /* over R, conjunctive */
    int32_t outer_key_cols[2];                                /* correlated outer column(s) */
    int32_t inner_key_cols[2];                                /* correlated inner column(s) */
    int32_t n_key_cols;                                       /* 1, or 2 (composite, '=' only) */
    nestgpu_cmp corr_op;                                      /* outer.key OP inner.key */
    const nestgpu_pred *inner_preds; int32_t n_inner_preds;   /* over S, conjunctive, invariant */
    nestgpu_agg agg;
    int32_t agg_col;                                          /* S column; ignored for COUNT/EXISTS */
    int32_t outer_cmp_col;                                    /* R column x; ignored for EXISTS */
    nestgpu_cmp outer_op;                                     /* lhs_mult*x OP rhs_mult*v */
    int64_t lhs_mult, rhs_mult;                               /* 1 .. 2^31-1 (reading R7) */
    int32_t index;                                            /* -1: tiled nested loop over S'; else index id */
    int64_t row_id_base;                                      /* added to emitted row ids (R shard offset) */
    int32_t emit_all;                                         /* 0: survivors only; 1: every R' tuple */
    int32_t dedup;                                            /* 1: evaluate the subquery once per distinct
                                                                 correlated value and reuse the result for
                                                                 duplicates ("Caching"); 0: once per
                                                                 R' tuple.  Same result either way. */
} nestgpu_plan;

typedef struct {
    int64_t n_rows;               /* survivors, or |R'| if emit_all */
    int64_t n_evaluated;          /* subquery evaluations performed: |R'|, or the number of
                                     distinct correlated values with dedup */
    const int64_t *d_row_ids;     /* ascending R row ids (+ row_id_base) */
    const int64_t *d_values;      /* Res[i]: MIN/MAX/SUM value, COUNT, AVG rounded at
                                     scale+6 (reading R6), EXISTS 0/1 */
    const uint8_t *d_valid;       /* 0: the subquery value is NULL */
    const uint8_t *d_passed;      /* outer predicate TRUE (always 1 unless emit_all) */
    const int64_t *d_avg_sum;     /* AVG only: exact sum of non-NULL payloads */
    const int64_t *d_avg_cnt;     /* AVG only: number of non-NULL payloads (nn) */
} nestgpu_result;

/* Execute one correlated subquery plan.  R is the set of columns the outer_*
 * fields name (all with one row count), S the columns the inner_* / agg
 * fields name.  index >= 0: S' comes from that index (its key columns, payload
 * and inner predicates must match the plan: INVALID otherwise); index == -1:
 * S is filtered here and the tiled block-nested-loop kernel runs.  Work is
 * enqueued on the context stream; the call synchronises once at the end to
 * read the survivor count (dedup adds two synchronisations: to plan the sort
 * of R' keys and to size the evaluation of the distinct keys); before that
 * sync the first rows of every result field (256 KB worth) are copied to
 * pinned host memory, so nestgpu_result_to_host of a result that small is a
 * host copy.  SUM / AVG are exact (reading R5): 64-bit payloads whose
 * |S| * max|payload| could reach 2^63 are accumulated as split 32-bit halves
 * and combined in int128; OVERFLOW only when some R' tuple's sum leaves
 * int64 (as the oracle).  Errors: INVALID, TYPE, UNSUPPORTED, OVERFLOW,
 * OOM, CUDA.  Nothing is launched when validation fails. */
nestgpu_status nestgpu_exec_correlated(nestgpu_ctx *ctx, const nestgpu_plan *plan,
                                       nestgpu_result *out);

/* Copy up to cap rows of a result to host buffers (each pointer may be NULL
 * to skip that field).  BUFFER if cap < n_rows (nothing copied).  Synchronous;
 * a result staged by its exec (see above) is served from pinned host memory
 * without any GPU operation. */
nestgpu_status nestgpu_result_to_host(nestgpu_ctx *ctx, const nestgpu_result *res,
                                      int64_t *row_ids, int64_t *values, uint8_t *valid,
                                      uint8_t *passed, int64_t *avg_sum, int64_t *avg_cnt,
                                      int64_t cap);

/* ---------------------------------------------------------------- type-J results */

/* The result of a type-J (set-valued) correlated subquery
 *     SELECT S.<agg_col> FROM S WHERE <inner_preds> AND R.key <corr_op> S.key
 * for every R' tuple, stored as the paper's two-level arrays (§III-B:
 * "The first level is to store the lengths of variable results for each
 * subquery evaluation and the second is to store the results").  Level 1 is
 * given as offsets (lengths = offsets[i+1] - offsets[i]).  Reading R17
 * (DESIGN.md): level 2 holds the NON-NULL values of the select list (its
 * consumers -- IN under WHERE semantics and equi-joins -- never match NULL).
 * Within one list the order is the index order (ascending key); compare
 * lists as multisets. */
typedef struct {
    int64_t n_outer;            /* level-1 entries = |R'| */
    int64_t n_values;           /* level-2 entries */
    const int64_t *d_row_ids;   /* [n_outer] R row ids (+ row_id_base), ascending */
    const int64_t *d_offsets;   /* [n_outer + 1] exclusive prefix sums of the lengths */
    const int64_t *d_values;    /* [n_values] S.<agg_col> widened to int64 */
    const int64_t *d_owner;     /* [n_values] row id of the level-1 entry owning the slot */
} nestgpu_collection;

/* Evaluate a type-J subquery for every R' tuple into two-level arrays.  Uses
 * the plan's outer_preds, key columns, corr_op, inner_preds, agg_col (the
 * selected column), index and row_id_base; the aggregate and outer
 * comparison fields are ignored.  The plan must name an index (index >= 0,
 * built with payload_col == agg_col and the plan's inner predicates):
 * with the sorted index every list is one run of the co-sorted payload (two
 * for '!='), so the arrays are built by binary search + prefix sum + a
 * load-balanced copy.  index == -1: UNSUPPORTED.  The arrays live in the
 * scratch pool until the next exec / exec_collect / build_index / release.
 * Synchronises once (to size level 2).  Errors: INVALID, UNSUPPORTED, OOM
 * (level 2 does not fit the arena), CUDA. */
nestgpu_status nestgpu_exec_collect(nestgpu_ctx *ctx, const nestgpu_plan *plan, nestgpu_collection *out);

/* The upper-level selection over a type-J result: keep R' tuple i iff
 * R.x_col[row] IN (list i) -- TRUE iff x is not NULL and some element equals
 * it (SQL; "R.col1 IN (...)").  x_col is an R column; rows are
 * d_row_ids[i] - row_id_base (pass the collection plan's row_id_base).
 * Output as nestgpu_exec_correlated's (values = 1 for survivors; emit_all = 1:
 * every level-1 entry with passed = the IN outcome).  The collection must
 * still be valid; the result lives until the next exec.  NOT IN is not
 * offered: its NULL semantics need the NULL elements R17 drops.
 * Errors: INVALID, OOM, CUDA. */
nestgpu_status nestgpu_collection_in(nestgpu_ctx *ctx, const nestgpu_collection *coll, int32_t x_col,
                                     int64_t row_id_base, int32_t emit_all, nestgpu_result *out);

/* Materialise a column from device int64 values: out[i] = src[i], valid[i] =
 * d_valid ? d_valid[i] : 1 (no validity array if d_valid is NULL).  This is
 * "Res[i] = Materialize(...)" (Fig. 4): it turns a result's d_values /
 * d_row_ids or a collection's d_values / d_owner into a column that later
 * plans, indexes and joins read (Fig. 5 join with a subquery;
 * Fig. 6 levels).  dtype NG_INT32 / NG_DATE / NG_DECIMAL32 narrows: OVERFLOW
 * (and no column) if a valid value is outside int32.  d_src / d_valid are
 * borrowed for the call.  Synchronises once when narrowing.
 * Errors: INVALID, TYPE, OVERFLOW, OOM, CUDA. */
nestgpu_status nestgpu_column_from_device(nestgpu_ctx *ctx, nestgpu_dtype dtype, int32_t scale,
                                          const int64_t *d_src, const uint8_t *d_valid, int64_t n,
                                          int32_t *out_col);

/* ---------------------------------------------------------------- cost model */

/* The paper's cost model (§IV), adapted to this engine's
 * vectorised kernels, to predict the latency of one nestgpu_exec_correlated
 * under each execution strategy and pick the fastest ("a cost model to
 * guide subquery processing by selecting the most effective execution
 * path").
 *
 *   Eq. (1)  T_op = sum_i K_i * ceil(D_i / Th_i) + M * D_r * sum(Rs) + C
 *   Eq. (6)  N    = (S - Ch) * [per-evaluation cost] + invariant parts once
 *   Eq. (7)  Nmem = memory-related cost per operation, once
 *   Eq. (8)  U    = outer-block scans / aggregations
 *   Eq. (9)  Q    = N + Nmem + U
 *
 * Every kernel here sizes its grid to its input, so K_i * ceil(D_i / Th_i)
 * becomes a per-element cost K_i * D_i (per row, per sorted byte, per probe
 * step, per (r,s) pair ...).  The K_i are MEASURED on this GPU by running the
 * engine's own kernels once on synthetic data ("One method to estimate
 * Ki is actually running the query once and reusing this value for all
 * predictions").  Vectorisation turns the per-iteration constant C of
 * Eq. (1) into one C per launch, not per outer tuple; caching makes
 * S - Ch the number of distinct correlated values.  Nmem is zero: columns
 * are preloaded and scratch comes from the pool, so there is no
 * per-operation allocation or transfer.  Cardinalities (D_r) are inputs,
 * known in advance as in the paper's evaluation. */
typedef struct {
    double launch_ms;                /* C: one kernel launch with a tiny input */
    double filter_ms_per_row;        /* selection (a2/a3), per input row */
    double hist_ms_per_key_digit;    /* index build digit histogram, per key per digit */
    double sort_ms_per_key;          /* one radix pass: per key ...                      */
    double sort_ms_per_byte;         /* ... plus per (key + payload) byte moved           */
    double probe_ms_per_step;        /* a5 binary search, per outer tuple per log2|S'| step */
    double range_ms_per_elem;        /* a6 fold, per qualifying element (only '=' MIN/MAX scans) */
    double aux_ms_per_elem;          /* prefix/suffix aggregates of an index payload, per element */
    double bnl_ms_per_pair[2][4];    /* a7 per (r,s) pair, [0] 4-byte / [1] 8-byte keys x
                                        [0] MIN/MAX [1] COUNT [2] SUM/AVG [3] EXISTS (no early exit) */
    double final_ms_per_row;         /* a8 aggregate finalize + outer comparison, per R' tuple */
    double materialize_ms_per_byte;  /* M: a9 compaction, per survivor byte written */
    double group_ms_per_key;         /* caching: grouping of sorted R' keys, per key */
    double sync_ms;                  /* one host round trip (small D2H + stream sync): exec reads its
                                        survivor count, an index build its |S'|, caching two more */
    double exec_overhead_ms;         /* host work of one exec beyond the above (validation, launch
                                        calls): a tiny exec's wall time minus its modelled time */
    double build_overhead_ms;        /* the same for one index build */
    double dedup_overhead_ms;        /* the same for the caching steps of an exec */
} nestgpu_cost_params;

typedef struct {
    int64_t n_r, n_s;            /* |R|, |S| */
    int64_t n_rp, n_sp;          /* |R'|, |S'| (after the local predicates) */
    int64_t n_distinct;          /* distinct correlated values among R' (S - Ch of Eq. (6)) */
    int64_t sum_k;               /* sum over R' tuples of their qualifying |S'| rows */
    int64_t survivors;           /* result rows */
    int32_t key_bytes;           /* 4 or 8 */
    int32_t payload_bytes;       /* 0 (COUNT / EXISTS), 4 or 8 */
    int32_t sort_passes;         /* radix passes of the index build (8-bit digits that vary) */
    int32_t dedup_passes;        /* radix passes of the R' key sort when caching */
    int32_t narrow_keys;         /* 1: 8-byte keys whose high words all agree (sorted as 4-byte
                                    keys between the first and the last pass) */
    nestgpu_cmp corr_op;
    nestgpu_agg agg;
} nestgpu_cost_input;

enum { NESTGPU_STRATEGY_NESTED_LOOP = 0, NESTGPU_STRATEGY_INDEX = 1,
       NESTGPU_STRATEGY_NESTED_LOOP_CACHED = 2, NESTGPU_STRATEGY_INDEX_CACHED = 3 };

typedef struct {
    double ms[4];                /* predicted Q per strategy (index strategies include building it) */
    double index_build_ms;       /* the index-build part of ms[1] / ms[3] (invariant, once) */
    double outer_ms;             /* U, Eq. (8): outer selection + finalize + compaction */
    double nested_ms[4];         /* N, Eq. (6), per strategy (index build excluded) */
    int32_t best;                /* argmin of ms[] */
} nestgpu_cost_estimate;

/* Measure the K_i of nestgpu_cost_params on this GPU: runs the engine's
 * filter, radix pass, digit histogram, binary-search range, prefix-aggregate,
 * nested-loop (per aggregate class), finalize and grouping kernels once each
 * (after a warm-up) on synthetic data in the scratch pool (~64 * n_rows bytes;
 * n_rows <= 0 picks 4M and shrinks to fit the arena) and times them with CUDA
 * events; then runs a tiny exec (plain, cached) and index build through this
 * API to measure their fixed host-side overheads (wall clock).  n_rows <= 0
 * picks 16M rows (large sorts amortise their per-tile costs like real ones).
 * Invalidates results of earlier execs; columns / indexes created after
 * nestgpu_mark survive.  Errors: INVALID, OOM, CUDA. */
nestgpu_status nestgpu_cost_calibrate(nestgpu_ctx *ctx, int64_t n_rows, nestgpu_cost_params *out);
/* Evaluate Eqs. (1)-(9) for one plan shape.  Pure host arithmetic (no device
 * work, no context).  Errors: INVALID (negative sizes, bad widths / enums). */
nestgpu_status nestgpu_cost_estimate_plan(const nestgpu_cost_params *params, const nestgpu_cost_input *in,
                                          nestgpu_cost_estimate *out);

/* ---------------------------------------------------------------- multi-GPU
 * Peer-memory survivor gather (north_star: "results are gathered"; the paper
 * is single-GPU).  Outer tuples are independent (Fig. 2),
 * so each rank's survivors are a contiguous block of the global result in
 * rank order.  Rank 0 creates a WINDOW -- device memory other processes map
 * through a CUDA IPC handle (NVLink / NVSwitch peer memory on a multi-GPU
 * box; plain device memory for ranks sharing one GPU) -- and every rank
 * stores its survivors straight into it at its row offset with
 * nestgpu_result_put: the bulk data moves by peer stores from the rank's own
 * kernel, no NCCL on the data path.  The caller exchanges the survivor counts
 * (8 B per rank) to get the offsets and orders the puts before rank 0 reads
 * the window (a barrier).
 *
 * Window layout (cap rows): int64 row ids [cap], then int64 values [cap].
 * The window is allocated with cudaMalloc at creation (setup time, never on
 * the exec path) and owned by the context until nestgpu_window_free. */
typedef struct {
    unsigned char bytes[64];   /* cudaIpcMemHandle_t */
} nestgpu_ipc_handle;
/* Create a window of cap rows; *d_window = its device address on this
 * context's device, *out its IPC handle.  Errors: INVALID, CUDA. */
nestgpu_status nestgpu_window_create(nestgpu_ctx *ctx, int64_t cap, void **d_window, nestgpu_ipc_handle *out);
/* Map a window created by another process; *d_peer is valid in this
 * context until nestgpu_window_close.  Errors: INVALID, CUDA (IPC not
 * available between the two devices). */
nestgpu_status nestgpu_window_open(nestgpu_ctx *ctx, const nestgpu_ipc_handle *handle, void **d_peer);
nestgpu_status nestgpu_window_close(nestgpu_ctx *ctx, void *d_peer);
nestgpu_status nestgpu_window_free(nestgpu_ctx *ctx, void *d_window);
/* Store a result's rows (ids, values) into window rows [offset, offset +
 * n_rows) of a window of cap rows (own or peer).  Synchronous: on return the
 * stores are complete and visible system-wide (__threadfence_system + stream
 * sync), so a host barrier then orders them before the owner's reads.
 * Errors: INVALID (offset + n_rows > cap), CUDA. */
nestgpu_status nestgpu_result_put(nestgpu_ctx *ctx, const nestgpu_result *res, void *d_window, int64_t cap,
                                  int64_t offset);

/* Ablation knobs -- NOT for production use; they exist to measure the
 * paper's design claims against their baselines (tools/ablations.py).
 *   NESTGPU_OPT_MALLOC_SCRATCH (value 0/1): per-exec scratch comes from one
 *     cudaMalloc per allocation, freed (after a stream sync) at the next
 *     exec / build_index / exec_collect / release -- the pool-less baseline
 *     that P:147 ("calling malloc/free ... is unacceptable") and P:233-237
 *     (memory pools) argue against.  Default 0: the arena pool.
 *   NESTGPU_OPT_BNL_SHAPE (value 0/1/2): the nested-loop kernel's R-block
 *     shape -- 0 automatic (from |R'|, |S'|), 1 full blocks, 2 warp-split.
 *     Results are identical; tests use it to cover both shapes on one input.
 *   NESTGPU_OPT_GRAPHS (value 0/1, default 1; env NESTGPU_GRAPHS=0 at
 *     create): exec's launch sequence is captured into a CUDA graph the first
 *     time a (plan, columns, index, arena state) combination is seen and
 *     replayed afterwards (one graph launch instead of one launch per
 *     kernel; not with dedup, profiling or the malloc ablation).  Results
 *     are identical either way.
 *   NESTGPU_OPT_SORT (value 0/1/2): the index build's sort -- 0 (default)
 *     the LSD onesweep, none for a key-ordered column; 1 always the LSD
 *     onesweep (the key-ordered shortcut off); 2 the two-round-trip MSD bucket sort
 *     (partition by the top varying key bits, finish each bucket in shared
 *     memory) wherever it fits, else the LSD onesweep.  An experiment kept
 *     for measurement: 1.2-1.9x slower than the onesweep on every measured
 *     shape.  Both are stable sorts of the same S'.
 *   NESTGPU_OPT_TINY (value 0/1, default 1): a nested-loop exec (index -1,
 *     no dedup) over |S| <= 4096, |R| <= 4096 rows and |R| x |S| <= 2^21 pairs
 *     runs as ONE kernel launch of one CTA (S' in shared memory, a warp per
 *     outer tuple, finalize and ordered compaction in the same kernel)
 *     instead of the fill / filter / nested-loop / finalize sequence; 0
 *     forces the sequence.  Results are identical either way.
 * Errors: INVALID (unknown option). */
enum { NESTGPU_OPT_MALLOC_SCRATCH = 1, NESTGPU_OPT_BNL_SHAPE = 2, NESTGPU_OPT_GRAPHS = 3, NESTGPU_OPT_SORT = 4,
       NESTGPU_OPT_TINY = 5 };
nestgpu_status nestgpu_set_option(nestgpu_ctx *ctx, int32_t option, int64_t value);

/* Per-stage device times (ms, CUDA events on the context stream) of the last
 * exec / build_index when profiling is on (nestgpu_set_profiling(ctx, 1)).
 * Stage order: 0 outer filter, 1 inner filter, 2 sort, 3 subquery kernel
 * (range-agg or nested loop), 4 finalize+compact, 5 total.  NaN if a stage
 * did not run. */
#define NESTGPU_N_STAGES 6
nestgpu_status nestgpu_set_profiling(nestgpu_ctx *ctx, int32_t on);
nestgpu_status nestgpu_last_profile(const nestgpu_ctx *ctx, float *ms, int32_t n);

#ifdef __cplusplus
}
#endif
#endif /* NESTGPU_H */
