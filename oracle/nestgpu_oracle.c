/*
 * nestgpu_oracle.c -- CPU ORACLE for the nested-method correlated subquery.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant with the CUDA path
 * (paper_conf_icde_floratosxwgylz21_b200/, include/) and includes nothing
 * from them.
 *
 * What it computes: the plain definition of the nested method -- PAPER.md
 * Fig. 2 (§II-D): for every outer tuple r, re-evaluate the
 * subquery with r's correlated value bound in, then keep r iff the outer
 * comparison with the subquery result holds; generalised, as the paper does,
 * to any correlated operator (§I) and to the drive-program shape of
 * Fig. 4 (§III-B) where the correlated outer column differs from
 * the compared one.  Nothing is blocked, fused, indexed or reordered: a
 * double loop over R x S in row order.
 *
 * Where the paper is silent this follows the SQL-92 readings listed in
 * DESIGN.md ("Readings of the paper"):
 *   R1 empty subquery: MIN/MAX/SUM/AVG -> NULL, COUNT(*) -> 0,
 *      EXISTS -> false, NOT EXISTS -> true; comparison with NULL is UNKNOWN
 *      and drops r.
 *   R2 NULL inputs: any predicate or correlation on a NULL is UNKNOWN
 *      (not TRUE); MIN/MAX/SUM/AVG skip NULL payloads; COUNT is COUNT(*).
 *   R5 sums are exact (__int128); a sum that does not fit int64 is an error.
 *   R6 AVG compares exactly: a*x OP b*(sum/nn)  <=>  a*x*nn OP b*sum (nn>0);
 *      the materialised AVG is round_half_away_from_zero(sum*10^6 / nn).
 *   R7 the outer comparison is  lhs_mult*x OP rhs_mult*v  (a,b > 0).
 *   R8 correlated predicates read  r.<outer col> OP s.<inner col>.
 *
 * Parity status: pinned (tests/test_oracle_pins.py): SQLite exhaustive
 * single-row instances, Query 1 == Query 2 for '=', closed-form prefix
 * aggregates for '<,<=,>,>=', total-minus-group for '!=', COUNT bug,
 * invariants.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* Operator / aggregate codes private to the oracle (the Python wrapper maps
 * SQL spellings onto them). */
enum { O_EQ = 0, O_NE = 1, O_LT = 2, O_LE = 3, O_GT = 4, O_GE = 5 };
enum { A_MIN = 0, A_MAX = 1, A_SUM = 2, A_COUNT = 3, A_AVG = 4,
       A_EXISTS = 5, A_NOT_EXISTS = 6 };

typedef struct { const int64_t *v; const uint8_t *valid; } ocol;   /* valid==NULL: NOT NULL */
typedef struct { int32_t col; int32_t op; int64_t lit; int32_t rhs_col; } opred;  /* rhs_col<0: literal */
typedef struct { int32_t outer_col; int32_t op; int32_t inner_col; } ocorr;

typedef struct {
    int64_t nR, nS;
    const ocol *R, *S;
    const opred *outer_preds; int32_t n_outer;
    const ocorr *corr; int32_t n_corr;       /* conjunctive; composite key = 2 entries */
    const opred *inner_preds; int32_t n_inner;
    int32_t agg, agg_col;
    int32_t cmp_col, outer_op;
    int64_t a, b;
} oplan;

/* x OP y evaluated on known (non-NULL) values. */
static int cmp_i128(__int128 x, int op, __int128 y)
{
    switch (op) {
    case O_EQ: return x == y;
    case O_NE: return x != y;
    case O_LT: return x < y;
    case O_LE: return x <= y;
    case O_GT: return x > y;
    case O_GE: return x >= y;
    }
    return 0;
}

static int is_null(const ocol *c, int64_t i) { return c->valid != NULL && c->valid[i] == 0; }

/* A local predicate "col OP literal" or "col OP col" on one row of table T:
 * TRUE only if every operand is non-NULL and the comparison holds (R2). */
static int pred_true(const ocol *T, const opred *p, int64_t row)
{
    const ocol *c = &T[p->col];
    if (is_null(c, row)) return 0;
    int64_t rhs;
    if (p->rhs_col >= 0) {
        const ocol *d = &T[p->rhs_col];
        if (is_null(d, row)) return 0;
        rhs = d->v[row];
    } else {
        rhs = p->lit;
    }
    return cmp_i128(c->v[row], p->op, rhs);
}

/* round_half_away_from_zero(num / den), den > 0 (reading R6). */
static __int128 div_round_half_away(__int128 num, __int128 den)
{
    __int128 mag = num < 0 ? -num : num;
    __int128 q = (2 * mag + den) / (2 * den);
    return num < 0 ? -q : q;
}

#define I64_MAX ((__int128)INT64_MAX)
#define I64_MIN ((__int128)INT64_MIN)

/*
 * Evaluate the plan for n_eval outer rows.
 *   rows   : R row numbers to evaluate (NULL => rows 0..nR-1, n_eval = nR)
 *   s_lo/hi: optional per-evaluated-row window of S rows [lo, hi)
 *            (NULL => all of S).  Used by batched tests only.
 * Outputs, one entry per evaluated row (all optional except passed):
 *   in_rp  : 1 if every outer local predicate is TRUE (r is in R')
 *   passed : 1 if r is in R' and the outer comparison / EXISTS is TRUE
 *   valid  : 1 if the subquery value is not NULL
 *   value  : the subquery value (MIN/MAX/SUM: the aggregate; COUNT: n;
 *            AVG: rounded mean at scale+6; EXISTS/NOT EXISTS: 0/1)
 *   sum    : exact sum of non-NULL payloads (SUM/AVG), else 0
 *   cnt    : AVG: nn (non-NULL payloads); otherwise n (qualifying rows)
 * Returns 0, -1 (invalid plan) or -5 (a sum overflows int64; reading R5).
 */
int oracle_eval(const oplan *P, const int64_t *rows, int64_t n_eval,
                const int64_t *s_lo, const int64_t *s_hi,
                uint8_t *in_rp, uint8_t *passed, uint8_t *valid,
                int64_t *value, int64_t *sum_out, int64_t *cnt_out,
                int nthreads)
{
    if (P->a <= 0 || P->b <= 0 || P->n_corr < 1 || P->n_corr > 2) return -1;
    if (rows == NULL) n_eval = P->nR;
    int status = 0;
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#else
    (void)nthreads;
#endif

#pragma omp parallel for schedule(dynamic, 16)
    for (int64_t e = 0; e < n_eval; e++) {
        const int64_t r = rows ? rows[e] : e;
        const int agg = P->agg;

        /* Outer block, local predicates first ("join first, then selection
         * with subquery"). */
        int in = 1;
        for (int k = 0; k < P->n_outer; k++)
            if (!pred_true(P->R, &P->outer_preds[k], r)) { in = 0; break; }

        int64_t n = 0, nn = 0;        /* qualifying rows / non-NULL payloads */
        __int128 acc = 0;             /* MIN/MAX/SUM accumulator */
        int have = 0;

        if (in) {
            /* subquery(r.c1): a full scan of S (Fig. 2, Fig. 4). */
            int64_t lo = s_lo ? s_lo[e] : 0, hi = s_hi ? s_hi[e] : P->nS;
            for (int64_t s = lo; s < hi; s++) {
                int ok = 1;
                for (int k = 0; k < P->n_inner && ok; k++)
                    ok = pred_true(P->S, &P->inner_preds[k], s);
                for (int k = 0; k < P->n_corr && ok; k++) {
                    const ocol *rc = &P->R[P->corr[k].outer_col];
                    const ocol *sc = &P->S[P->corr[k].inner_col];
                    ok = !is_null(rc, r) && !is_null(sc, s) &&
                         cmp_i128(rc->v[r], P->corr[k].op, sc->v[s]);
                }
                if (!ok) continue;
                n += 1;
                if (agg == A_MIN || agg == A_MAX || agg == A_SUM || agg == A_AVG) {
                    const ocol *vc = &P->S[P->agg_col];
                    if (is_null(vc, s)) continue;
                    __int128 v = vc->v[s];
                    nn += 1;
                    if (!have) { acc = v; have = 1; }
                    else if (agg == A_MIN) { if (v < acc) acc = v; }
                    else if (agg == A_MAX) { if (v > acc) acc = v; }
                    else acc += v;
                }
            }
        }

        /* finalize(AGG) -> subquery value (R1, R6) */
        int vvalid = 1;
        __int128 v = 0;
        int64_t sum64 = 0, cnt64 = n;
        switch (agg) {
        case A_MIN: case A_MAX: case A_SUM:
            vvalid = nn > 0; v = acc; break;
        case A_COUNT:
            v = n; break;
        case A_AVG:
            vvalid = nn > 0; cnt64 = nn;
            if (vvalid) v = div_round_half_away(acc * 1000000, nn);
            break;
        case A_EXISTS: v = n > 0; break;
        case A_NOT_EXISTS: v = n == 0; break;
        }
        if ((agg == A_SUM || agg == A_AVG) && (acc > I64_MAX || acc < I64_MIN)) {
#pragma omp atomic write
            status = -5;
            vvalid = 0;
        }
        if (agg == A_SUM || agg == A_AVG) sum64 = (int64_t)acc;

        /* The selection on Res (Fig. 4): a*x OP b*v, NULL => UNKNOWN. */
        int pass = 0;
        if (in) {
            if (agg == A_EXISTS || agg == A_NOT_EXISTS) {
                pass = (int)v;
            } else {
                const ocol *xc = &P->R[P->cmp_col];
                if (vvalid && !is_null(xc, r)) {
                    __int128 x = xc->v[r];
                    if (agg == A_AVG)
                        pass = cmp_i128((__int128)P->a * x * nn, P->outer_op,
                                        (__int128)P->b * acc);
                    else
                        pass = cmp_i128((__int128)P->a * x, P->outer_op,
                                        (__int128)P->b * v);
                }
            }
        }
        if (in_rp) in_rp[e] = (uint8_t)in;
        passed[e] = (uint8_t)pass;
        if (valid) valid[e] = (uint8_t)(in && vvalid);
        if (value) value[e] = (in && vvalid) ? (int64_t)v : 0;
        if (sum_out) sum_out[e] = in ? sum64 : 0;
        if (cnt_out) cnt_out[e] = in ? cnt64 : 0;
    }
    return status;
}

/*
 * Type-J subquery results as two-level arrays (§III-B "For
 * such subqueries, we use a two-level arrays to store the results of
 * subquery evaluations.  The first level is to store the lengths of variable
 * results for each subquery evaluation and the second is to store the
 * results."): for every R row in row order, the multiset
 *     SELECT S.<agg_col> FROM S WHERE <inner_preds> AND r.key OP s.key
 * evaluated by a full scan of S in row order (Fig. 2's loop).
 * Reading R17: the arrays hold the NON-NULL values of the select
 * list -- their consumers are IN under WHERE semantics (a NULL element never
 * makes IN TRUE, R10b) and equi-joins (NULL never joins).  A row that fails
 * the outer predicates (not in R') gets length 0 and in_rp = 0.
 *   lens   : level 1, one length per evaluated row (always written)
 *   vals   : level 2, concatenated in row order; NULL => lengths only
 *   cap    : capacity of vals; -7 if the total exceeds it
 * Aggregate / outer-comparison fields of the plan are ignored.
 * Returns 0, -1 (invalid plan) or -7 (vals too small).
 */
int oracle_collect(const oplan *P, uint8_t *in_rp, int64_t *lens, int64_t *vals, int64_t cap)
{
    if (P->n_corr < 1 || P->n_corr > 2 || P->agg_col < 0) return -1;
    const ocol *vc = &P->S[P->agg_col];
    int64_t pos = 0;
    for (int64_t r = 0; r < P->nR; r++) {
        int in = 1;
        for (int k = 0; k < P->n_outer; k++)
            if (!pred_true(P->R, &P->outer_preds[k], r)) { in = 0; break; }
        int64_t len = 0;
        if (in) {
            for (int64_t s = 0; s < P->nS; s++) {
                int ok = 1;
                for (int k = 0; k < P->n_inner && ok; k++)
                    ok = pred_true(P->S, &P->inner_preds[k], s);
                for (int k = 0; k < P->n_corr && ok; k++) {
                    const ocol *rc = &P->R[P->corr[k].outer_col];
                    const ocol *sc = &P->S[P->corr[k].inner_col];
                    ok = !is_null(rc, r) && !is_null(sc, s) &&
                         cmp_i128(rc->v[r], P->corr[k].op, sc->v[s]);
                }
                if (!ok || is_null(vc, s)) continue;
                if (vals) {
                    if (pos >= cap) return -7;
                    vals[pos] = vc->v[s];
                }
                pos += 1;
                len += 1;
            }
        }
        if (in_rp) in_rp[r] = (uint8_t)in;
        lens[r] = len;
    }
    return 0;
}

int oracle_max_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
