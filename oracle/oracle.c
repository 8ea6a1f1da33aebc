/*
 * oracle/oracle.c -- CPU ORACLE FOR SpGEMM C = A x B on CSR.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  The product path (paper_conf_ipps_xia0ar21_b200/) never
 * imports, links or executes it, and the two share no code, header or table.
 *
 * What it computes (§I, eq. C_ij = sum_k A_ik x B_kj; Alg. 1 L33-50):
 *   structure  S_i = U_{k in I_i(A)} { j : (k,j) in pat(B) }, sorted ascending (§II-A, §II-B);
 *              entries are structural: a sum that cancels to 0.0 is still stored (Alg. 1 L42-44
 *              inserts on first touch regardless of value; reading R1).
 *   values     c_ij accumulated in IEEE binary64 in exactly Alg. 1's order: rows of A in order
 *              (line 2), A_ik ascending (line 3), B_kj ascending (line 4), value = A_ik*B_kj
 *              rounded once (line 5), first touch assigns (lines 6-8), later touches add (line 10).
 *   reference  ref_ij = the same sum carried in x86-64 long double (64-bit significand), and
 *              tol_ij = 1e-12 * sum |A_ik*B_kj| (BASELINE.json north_star bound), both for the
 *              parity comparison.
 *   products   u_i = sum_{k in I_i(A)} nnz(B_k*), the trip count of Alg. 1 line 4 (the "number of
 *              floating-point operations associated with each row", §III-B; reading R4).
 *
 * Two independent accumulators are provided so that each checks the other:
 *   oracle_numeric      -- Alg. 1 with a dense marker array (sparse accumulator) + sort of the
 *                          touched column list;
 *   oracle_numeric_esc  -- expand/sort/compress (the ESC formulation, §VI): all products
 *                          of a row expanded, stably merge-sorted by column, equal columns summed
 *                          left to right.  Stable sorting keeps Alg. 1's order per column, so the
 *                          fp64 sums are bit-identical to oracle_numeric's.
 *
 * Threads: rows are independent (§III-A), so rows are handed out in blocks of 64 to
 * `nthreads` POSIX threads; every row is computed by one thread in the order above, so the
 * result does not depend on the thread count.  Compile with -O2 -ffp-contract=off, never
 * -ffast-math (fp64 products must round exactly once, Alg. 1 line 5).
 *
 * Index widths (reading R3): row_ptr int64, col int32, val fp64.
 *
 * Comparison rule (SURVEY.md §8(c) "Comparison rule"), used by oracle_verify
 * below and, identically, by oracle.compare() in Python:
 *   row_ptr and col_idx bit-identical to the oracle's (sorted, unique columns, §II-B);
 *   each value v against ref = (double) long-double sum and tol = (double)(1e-12 * sum |a*b|):
 *     NaN on either side   -> good iff both are NaN;
 *     Inf on either side   -> good iff v == ref (same infinity);
 *     otherwise            -> good iff |v - ref| <= tol  (tol = 0 -> v must equal ref, +-0.0).
 * oracle_verify checks a candidate's rows while it computes them, without storing the oracle's
 * output (full-size parity of C3 / C4 / C5, whose C is larger than host memory).  Structure:
 * the candidate row must be strictly increasing, every column must be in the oracle's set S_i
 * (the marker array of Alg. 1 line 6) and the counts must agree -- which is the same as
 * col == sorted(S_i) element by element, without sorting S_i.
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
    int64_t nrows, ncols;
    const int64_t *rp;
    const int32_t *col;
    const double *val;
} ocsr;

/* ---------------------------------------------------------------------------------------- */
/* thread pool over a row selection                                                          */

/* verification statistics (oracle_verify) */
typedef struct {
    int64_t rows, entries, products;   /* rows / candidate entries checked, products walked        */
    int64_t bad_rows, bad_row_ptr, bad_col, bad_val, bad_products;
    int64_t first_bad_row;             /* -1 if none (smallest failing row index)                  */
    int32_t first_bad_kind;            /* 0 none, 1 row_ptr (nnz), 2 col, 3 value, 4 products      */
    int32_t pad;
    double worst_ratio;                /* max |v - ref| / tol over good-by-tolerance entries        */
} vstat;

typedef struct job job;
typedef void (*row_fn)(job *, void *scratch, int64_t sel_index, int64_t row);
typedef void *(*scratch_new)(job *);

struct job {
    const ocsr *A, *B;
    const int64_t *rows; /* NULL = rows 0..nsel-1 */
    int64_t nsel;
    int64_t next;        /* atomic cursor */
    row_fn fn;
    scratch_new mk;
    /* outputs */
    int64_t *u, *nnz;
    const int64_t *out_rp;
    int32_t *col;
    double *val, *ref, *tol;
    int status;
    /* oracle_verify: candidate rows (offsets relative to crp[0]) and merged statistics */
    int64_t row0;
    const int64_t *crp;
    const int32_t *ccol;
    const double *cval;
    const int64_t *cprod;  /* optional candidate products per row (NULL: not checked) */
    vstat *vout;
    pthread_mutex_t mu;
    struct spa **pool;  /* optional persistent scratch, one per thread (oracle_verify_ctx) */
    int pool_n, pool_next;
};

static void *worker(void *arg) {
    job *J = (job *)arg;
    void *s = J->mk ? J->mk(J) : NULL;
    if (J->mk && !s) {
        __atomic_store_n(&J->status, -1, __ATOMIC_SEQ_CST);
        return NULL;
    }
    for (;;) {
        int64_t b = __atomic_fetch_add(&J->next, 64, __ATOMIC_RELAXED);
        if (b >= J->nsel) break;
        int64_t e = b + 64 < J->nsel ? b + 64 : J->nsel;
        for (int64_t t = b; t < e; ++t) J->fn(J, s, t, J->rows ? J->rows[t] : t);
    }
    free(s);
    return NULL;
}

static int run(job *J, int nthreads) {
    if (nthreads < 1) nthreads = 1;
    if (nthreads > 256) nthreads = 256;
    J->next = 0;
    J->status = 0;
    if (nthreads == 1) {
        worker(J);
        return J->status;
    }
    pthread_t th[256];
    int started = 0;
    for (int t = 0; t < nthreads; ++t)
        if (pthread_create(&th[t], NULL, worker, J) == 0) started++;
        else break;
    if (started == 0) worker(J);
    for (int t = 0; t < started; ++t) pthread_join(th[t], NULL);
    return J->status;
}

/* ---------------------------------------------------------------------------------------- */
/* products per row: u_i = sum_{k in I_i(A)} (B.rp[k+1] - B.rp[k])                             */

static void products_row(job *J, void *s, int64_t t, int64_t i) {
    (void)s;
    const ocsr *A = J->A, *B = J->B;
    int64_t u = 0;
    for (int64_t p = A->rp[i]; p < A->rp[i + 1]; ++p) {
        int32_t k = A->col[p];
        u += B->rp[k + 1] - B->rp[k];
    }
    J->u[t] = u;
}

int oracle_products(const ocsr *A, const ocsr *B, const int64_t *rows, int64_t nsel, int64_t *u_out,
                    int nthreads) {
    job J;
    memset(&J, 0, sizeof J);
    J.A = A; J.B = B; J.rows = rows; J.nsel = nsel; J.fn = products_row; J.u = u_out;
    return run(&J, nthreads);
}

/* ---------------------------------------------------------------------------------------- */
/* Alg. 1 with a dense marker array                                                          */


typedef struct spa {
    int64_t *mark;      /* mark[j] == gen  <=>  C_ij in C_i* for the row being built (Alg. 1 line 6) */
    int64_t gen;        /* one fresh stamp per row (rows may repeat in a selection) */
    double *acc;        /* fp64 accumulator, Alg. 1 order */
    long double *accL;  /* extended-precision reference sum */
    long double *absL;  /* sum of |products| for the tolerance */
    int32_t *touched;   /* columns inserted in this row (insert(), Alg. 1 line 7) */
    int64_t ntouched;
    vstat vs;           /* oracle_verify: this thread's statistics */
} spa;

static void *spa_alloc(int64_t ncols) {
    int64_t n = ncols > 0 ? ncols : 1;
    spa *s = (spa *)calloc(1, sizeof(spa));
    if (!s) return NULL;
    s->vs.first_bad_row = -1;
    s->mark = (int64_t *)malloc(sizeof(int64_t) * n);
    s->acc = (double *)malloc(sizeof(double) * n);
    s->accL = (long double *)malloc(sizeof(long double) * n);
    s->absL = (long double *)malloc(sizeof(long double) * n);
    s->touched = (int32_t *)malloc(sizeof(int32_t) * n);
    if (!s->mark || !s->acc || !s->accL || !s->absL || !s->touched) return NULL;
    for (int64_t j = 0; j < n; ++j) s->mark[j] = -1;
    return s;
}

static void *spa_new(job *J) { return spa_alloc(J->B->ncols); }

static void spa_free_members(spa *s) {
    free(s->mark); free(s->acc); free(s->accL); free(s->absL); free(s->touched);
}

static int cmp_i32(const void *a, const void *b) {
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

/* Gustavson row i into s: lines 3-12 of Alg. 1 */
static void gustavson_row(const ocsr *A, const ocsr *B, spa *s, int64_t i) {
    const int64_t g = ++s->gen;
    s->ntouched = 0;
    for (int64_t p = A->rp[i]; p < A->rp[i + 1]; ++p) {          /* line 3: A_ik in A_i* */
        int32_t k = A->col[p];
        double a = A->val[p];
        for (int64_t q = B->rp[k]; q < B->rp[k + 1]; ++q) {      /* line 4: B_kj in B_k* */
            int32_t j = B->col[q];
            double value = a * B->val[q];                       /* line 5 */
            long double valueL = (long double)a * (long double)B->val[q];
            if (s->mark[j] != g) {                              /* line 6 */
                s->mark[j] = g;                                 /* line 7: insert */
                s->touched[s->ntouched++] = j;
                s->acc[j] = value;                              /* line 8 */
                s->accL[j] = valueL;
                s->absL[j] = fabsl(valueL);
            } else {
                s->acc[j] = s->acc[j] + value;                  /* line 10 */
                s->accL[j] += valueL;
                s->absL[j] += fabsl(valueL);
            }
        }
    }
    qsort(s->touched, (size_t)s->ntouched, sizeof(int32_t), cmp_i32); /* sorted rows, §II-B */
}

static void nnz_row(job *J, void *sv, int64_t t, int64_t i) {
    spa *s = (spa *)sv;
    /* structure only: same marker walk, no values */
    int64_t c = 0;
    const int64_t g = ++s->gen;
    const ocsr *A = J->A, *B = J->B;
    for (int64_t p = A->rp[i]; p < A->rp[i + 1]; ++p) {
        int32_t k = A->col[p];
        for (int64_t q = B->rp[k]; q < B->rp[k + 1]; ++q) {
            int32_t j = B->col[q];
            if (s->mark[j] != g) { s->mark[j] = g; c++; }
        }
    }
    J->nnz[t] = c;
}

static void numeric_row(job *J, void *sv, int64_t t, int64_t i) {
    spa *s = (spa *)sv;
    gustavson_row(J->A, J->B, s, i);
    int64_t o = J->out_rp[t];
    if (J->out_rp[t + 1] - o != s->ntouched) {                   /* caller sized rows wrongly */
        __atomic_store_n(&J->status, -2, __ATOMIC_SEQ_CST);
        return;
    }
    for (int64_t e = 0; e < s->ntouched; ++e) {
        int32_t j = s->touched[e];
        J->col[o + e] = j;
        J->val[o + e] = s->acc[j];
        if (J->ref) J->ref[o + e] = (double)s->accL[j];
        if (J->tol) J->tol[o + e] = (double)(1e-12L * s->absL[j]);
    }
}

static void vmerge(job *J, const vstat *x);

/* worker wrapper that frees the spa members (scratch is a struct of pointers) */
static void *worker_spa(void *arg) {
    job *J = (job *)arg;
    spa *s = NULL;
    if (J->pool) {  /* persistent scratch: marks stay valid (stamps only grow), stats restart */
        int k = __atomic_fetch_add(&J->pool_next, 1, __ATOMIC_RELAXED);
        if (k < J->pool_n) {
            s = J->pool[k];
            memset(&s->vs, 0, sizeof s->vs);
            s->vs.first_bad_row = -1;
        }
    } else {
        s = (spa *)spa_new(J);
    }
    if (!s) {
        __atomic_store_n(&J->status, -1, __ATOMIC_SEQ_CST);
        return NULL;
    }
    for (;;) {
        int64_t b = __atomic_fetch_add(&J->next, 64, __ATOMIC_RELAXED);
        if (b >= J->nsel) break;
        int64_t e = b + 64 < J->nsel ? b + 64 : J->nsel;
        for (int64_t t = b; t < e; ++t) J->fn(J, s, t, J->rows ? J->rows[t] : t);
    }
    if (J->vout) vmerge(J, &s->vs);
    if (!J->pool) {
        spa_free_members(s);
        free(s);
    }
    return NULL;
}

static int run_spa(job *J, int nthreads) {
    if (nthreads < 1) nthreads = 1;
    if (nthreads > 256) nthreads = 256;
    J->next = 0;
    J->status = 0;
    if (nthreads == 1) {
        worker_spa(J);
        return J->status;
    }
    pthread_t th[256];
    int started = 0;
    for (int t = 0; t < nthreads; ++t)
        if (pthread_create(&th[t], NULL, worker_spa, J) == 0) started++;
        else break;
    if (started == 0) worker_spa(J);
    for (int t = 0; t < started; ++t) pthread_join(th[t], NULL);
    return J->status;
}

/* nnz of C row per selected row (the symbolic count, §II-B) */
int oracle_row_nnz(const ocsr *A, const ocsr *B, const int64_t *rows, int64_t nsel, int64_t *nnz_out,
                   int nthreads) {
    job J;
    memset(&J, 0, sizeof J);
    J.A = A; J.B = B; J.rows = rows; J.nsel = nsel; J.fn = nnz_row; J.nnz = nnz_out;
    return run_spa(&J, nthreads);
}

/* values: out_rp[nsel+1] are offsets (relative) of each selected row into col/val/ref/tol.
 * ref and tol may be NULL (the timed CPU baseline computes only col/val). */
int oracle_numeric(const ocsr *A, const ocsr *B, const int64_t *rows, int64_t nsel, const int64_t *out_rp,
                   int32_t *col, double *val, double *ref, double *tol, int nthreads) {
    job J;
    memset(&J, 0, sizeof J);
    J.A = A; J.B = B; J.rows = rows; J.nsel = nsel; J.fn = numeric_row;
    J.out_rp = out_rp; J.col = col; J.val = val; J.ref = ref; J.tol = tol;
    return run_spa(&J, nthreads);
}

/* ---------------------------------------------------------------------------------------- */
/* ESC cross-check: expand, stable sort by column, compress                                   */

typedef struct {
    int32_t j;
    double v;
} prod;

static void merge_sort_stable(prod *a, prod *tmp, int64_t n) {
    /* bottom-up merge sort: stable (equal keys keep expansion order = Alg. 1 order) */
    for (int64_t w = 1; w < n; w *= 2) {
        for (int64_t lo = 0; lo < n; lo += 2 * w) {
            int64_t mid = lo + w < n ? lo + w : n, hi = lo + 2 * w < n ? lo + 2 * w : n;
            int64_t x = lo, y = mid, k = lo;
            while (x < mid && y < hi) tmp[k++] = (a[y].j < a[x].j) ? a[y++] : a[x++];
            while (x < mid) tmp[k++] = a[x++];
            while (y < hi) tmp[k++] = a[y++];
        }
        memcpy(a, tmp, sizeof(prod) * (size_t)n);
    }
}

static void esc_row(job *J, void *sv, int64_t t, int64_t i) {
    (void)sv;
    const ocsr *A = J->A, *B = J->B;
    int64_t u = 0;
    for (int64_t p = A->rp[i]; p < A->rp[i + 1]; ++p) u += B->rp[A->col[p] + 1] - B->rp[A->col[p]];
    prod *e = (prod *)malloc(sizeof(prod) * (size_t)(u ? u : 1));
    prod *tmp = (prod *)malloc(sizeof(prod) * (size_t)(u ? u : 1));
    if (!e || !tmp) { free(e); free(tmp); __atomic_store_n(&J->status, -1, __ATOMIC_SEQ_CST); return; }
    int64_t n = 0;
    for (int64_t p = A->rp[i]; p < A->rp[i + 1]; ++p)                 /* expand */
        for (int64_t q = B->rp[A->col[p]]; q < B->rp[A->col[p] + 1]; ++q) {
            e[n].j = B->col[q];
            e[n].v = A->val[p] * B->val[q];
            n++;
        }
    merge_sort_stable(e, tmp, n);                                        /* sort */
    int64_t o = J->out_rp[t], w = 0;
    for (int64_t x = 0; x < n;) {                                        /* compress */
        int32_t j = e[x].j;
        double s = e[x].v;
        int64_t y = x + 1;
        while (y < n && e[y].j == j) { s = s + e[y].v; y++; }
        if (o + w >= J->out_rp[t + 1]) { __atomic_store_n(&J->status, -2, __ATOMIC_SEQ_CST); break; }
        J->col[o + w] = j;
        J->val[o + w] = s;
        w++;
        x = y;
    }
    if (o + w != J->out_rp[t + 1]) __atomic_store_n(&J->status, -2, __ATOMIC_SEQ_CST);
    free(e);
    free(tmp);
}

int oracle_numeric_esc(const ocsr *A, const ocsr *B, const int64_t *rows, int64_t nsel, const int64_t *out_rp,
                       int32_t *col, double *val, int nthreads) {
    job J;
    memset(&J, 0, sizeof J);
    J.A = A; J.B = B; J.rows = rows; J.nsel = nsel; J.fn = esc_row;
    J.out_rp = out_rp; J.col = col; J.val = val;
    return run(&J, nthreads);
}

/* ---------------------------------------------------------------------------------------- */
/* verification of a candidate's rows against Alg. 1 (full-size parity without storing C)     */

static void vbad(vstat *v, int64_t row, int kind) {
    if (v->first_bad_row < 0 || row < v->first_bad_row) {
        v->first_bad_row = row;
        v->first_bad_kind = kind;
    }
}

static void vmerge(job *J, const vstat *x) {
    pthread_mutex_lock(&J->mu);
    vstat *o = J->vout;
    o->rows += x->rows;
    o->entries += x->entries;
    o->products += x->products;
    o->bad_rows += x->bad_rows;
    o->bad_row_ptr += x->bad_row_ptr;
    o->bad_col += x->bad_col;
    o->bad_val += x->bad_val;
    o->bad_products += x->bad_products;
    if (x->first_bad_row >= 0 && (o->first_bad_row < 0 || x->first_bad_row < o->first_bad_row)) {
        o->first_bad_row = x->first_bad_row;
        o->first_bad_kind = x->first_bad_kind;
    }
    if (x->worst_ratio > o->worst_ratio) o->worst_ratio = x->worst_ratio;
    pthread_mutex_unlock(&J->mu);
}

/* the comparison rule of the header: 1 = good; *ratio = |v - ref| / tol for finite values */
static int value_good(double v, double ref, double tol, double *ratio) {
    *ratio = 0.0;
    if (isnan(v) || isnan(ref)) return isnan(v) && isnan(ref);
    if (isinf(v) || isinf(ref)) return v == ref;
    double err = fabs(v - ref);
    if (err == 0.0) return 1;
    *ratio = tol > 0.0 ? err / tol : INFINITY;
    return err <= tol;
}

static void verify_row(job *J, void *sv, int64_t t, int64_t i_local) {
    spa *s = (spa *)sv;
    const ocsr *A = J->A, *B = J->B;
    const int64_t i = J->row0 + i_local;
    vstat *v = &s->vs;
    /* Alg. 1 lines 3-10 for row i: structure in mark[], reference sums in accL/absL */
    const int64_t g = ++s->gen;
    int64_t nset = 0, u = 0;
    for (int64_t p = A->rp[i]; p < A->rp[i + 1]; ++p) {
        int32_t k = A->col[p];
        long double a = (long double)A->val[p];
        for (int64_t q = B->rp[k]; q < B->rp[k + 1]; ++q) {
            int32_t j = B->col[q];
            long double valueL = a * (long double)B->val[q];
            if (s->mark[j] != g) {
                s->mark[j] = g;
                s->accL[j] = valueL;
                s->absL[j] = fabsl(valueL);
                nset++;
            } else {
                s->accL[j] += valueL;
                s->absL[j] += fabsl(valueL);
            }
            u++;
        }
    }
    v->rows++;
    v->products += u;
    int bad = 0;
    if (J->cprod && J->cprod[t] != u) {
        v->bad_products++;
        vbad(v, i, 4);
        bad = 1;
    }
    const int64_t o = J->crp[t] - J->crp[0], n = J->crp[t + 1] - J->crp[t];
    if (n != nset) {
        v->bad_row_ptr++;
        vbad(v, i, 1);
        v->bad_rows++;
        return;
    }
    const int64_t nc = B->ncols;
    int64_t prev = -1;
    for (int64_t e = 0; e < n; ++e) {  /* structure first: sorted, in range, in S_i */
        const int64_t j = J->ccol[o + e];
        if (j <= prev || j < 0 || j >= nc || s->mark[j] != g) {
            v->bad_col++;
            vbad(v, i, 2);
            v->bad_rows++;
            return;
        }
        prev = j;
    }
    for (int64_t e = 0; e < n; ++e) {  /* then every value against its reference sum */
        const int32_t j = J->ccol[o + e];
        double r;
        v->entries++;
        if (!value_good(J->cval[o + e], (double)s->accL[j], (double)(1e-12L * s->absL[j]), &r)) {
            v->bad_val++;
            vbad(v, i, 3);
            bad = 1;
        } else if (r > v->worst_ratio) {
            v->worst_ratio = r;
        }
    }
    if (bad) v->bad_rows++;
}

/* Check candidate rows row0 .. row0+nrows-1 of C = A x B: crp [nrows+1] offsets (any base),
 * ccol / cval the rows' entries from ccol[0] (= offset crp[0]), cprod [nrows] optional products
 * per row.  *out is overwritten.  Returns 0, or < 0 on allocation failure / bad arguments. */
/* persistent per-thread scratch for repeated oracle_verify calls over the same B (a sink checks
 * one chunk after another: allocating and stamping a dense marker array of ncols entries per
 * thread per call would cost more than the check of a small chunk) */
typedef struct {
    int64_t ncols;
    int n;
    spa **s;
} vctx;

void oracle_verify_ctx_free(void *c) {
    vctx *x = (vctx *)c;
    if (!x) return;
    for (int t = 0; t < x->n; ++t)
        if (x->s[t]) {
            spa_free_members(x->s[t]);
            free(x->s[t]);
        }
    free(x->s);
    free(x);
}

void *oracle_verify_ctx_new(int64_t ncols, int nthreads) {
    if (nthreads < 1) nthreads = 1;
    if (nthreads > 256) nthreads = 256;
    vctx *x = (vctx *)calloc(1, sizeof(vctx));
    if (!x) return NULL;
    x->ncols = ncols;
    x->n = nthreads;
    x->s = (spa **)calloc((size_t)nthreads, sizeof(spa *));
    if (!x->s) { free(x); return NULL; }
    for (int t = 0; t < nthreads; ++t)
        if (!(x->s[t] = (spa *)spa_alloc(ncols))) { oracle_verify_ctx_free(x); return NULL; }
    return x;
}

int oracle_verify(const ocsr *A, const ocsr *B, int64_t row0, int64_t nrows, const int64_t *crp,
                  const int32_t *ccol, const double *cval, const int64_t *cprod, int nthreads, vstat *out,
                  void *ctx) {
    memset(out, 0, sizeof *out);
    out->first_bad_row = -1;
    if (row0 < 0 || nrows < 0 || row0 + nrows > A->nrows) return -3;
    job J;
    memset(&J, 0, sizeof J);
    J.A = A; J.B = B; J.rows = NULL; J.nsel = nrows; J.fn = verify_row;
    J.row0 = row0; J.crp = crp; J.ccol = ccol; J.cval = cval; J.cprod = cprod; J.vout = out;
    if (ctx) {
        vctx *x = (vctx *)ctx;
        if (x->ncols != B->ncols) return -4;
        J.pool = x->s;
        J.pool_n = x->n;
        if (nthreads > x->n) nthreads = x->n;
    }
    pthread_mutex_init(&J.mu, NULL);
    int rc = run_spa(&J, nthreads);
    pthread_mutex_destroy(&J.mu);
    return rc;
}
