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

typedef struct {
    int64_t *mark;      /* mark[j] == gen  <=>  C_ij in C_i* for the row being built (Alg. 1 line 6) */
    int64_t gen;        /* one fresh stamp per row (rows may repeat in a selection) */
    double *acc;        /* fp64 accumulator, Alg. 1 order */
    long double *accL;  /* extended-precision reference sum */
    long double *absL;  /* sum of |products| for the tolerance */
    int32_t *touched;   /* columns inserted in this row (insert(), Alg. 1 line 7) */
    int64_t ntouched;
} spa;

static void *spa_new(job *J) {
    int64_t n = J->B->ncols > 0 ? J->B->ncols : 1;
    spa *s = (spa *)calloc(1, sizeof(spa));
    if (!s) return NULL;
    s->mark = (int64_t *)malloc(sizeof(int64_t) * n);
    s->acc = (double *)malloc(sizeof(double) * n);
    s->accL = (long double *)malloc(sizeof(long double) * n);
    s->absL = (long double *)malloc(sizeof(long double) * n);
    s->touched = (int32_t *)malloc(sizeof(int32_t) * n);
    if (!s->mark || !s->acc || !s->accL || !s->absL || !s->touched) return NULL;
    for (int64_t j = 0; j < n; ++j) s->mark[j] = -1;
    return s;
}

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

/* worker wrapper that frees the spa members (scratch is a struct of pointers) */
static void *worker_spa(void *arg) {
    job *J = (job *)arg;
    spa *s = (spa *)spa_new(J);
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
    spa_free_members(s);
    free(s);
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
