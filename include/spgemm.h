/*
 * include/spgemm.h -- C ABI of the B200-native out-of-core chunked SpGEMM  C = A x B  (CSR).
 *
 * Method: Xia, Jiang, Agrawal, Ramnath, "Scaling Sparse Matrix Multiplication on CPU-GPU Nodes",
 * IPDPS'21.  Row panels of A times column panels of B give independent chunks of C
 * (Alg. 3, §III-A); each chunk is computed in-core on the GPU by a two-phase hash
 * SpGEMM -- per-row product count ("row analysis", §III-B), symbolic hash pass giving nnz
 * per row (L126, §II-B), exclusive scan (L126), numeric hash accumulate + per-row sort
 * (§II-B, §III-B) -- into buffers preallocated in one device arena with no allocation
 * during compute (§IV-B), and every finished chunk streams to host memory over
 * asynchronous D2H copies overlapped with the next chunk's compute (two+ streams, two+ device
 * buffers, pinned host memory: §IV-B).
 *
 * All entry points are extern "C", take plain pointers and sizes, and return spgemm_status.
 * No PyTorch type appears here; the Python binding passes device pointers it allocated with
 * torch and a cudaStream_t as `void *`.
 *
 * Data layout (reading R3): CSR with int64 row_ptr [nrows+1] (row_ptr[0] == 0 for host
 * inputs; any base for device inputs, see spgemm_csr), int32 col_idx sorted strictly increasing in
 * every row (§II-A), fp64 values (§V-B "double").  Output C uses the same layout; its
 * rows are sorted by column (§II-B), and entries are STRUCTURAL: a sum that cancels to 0.0 is
 * stored (Alg. 1 L42-44; reading R1).  Values are the fp64 sums of the products in some order;
 * each satisfies |c - c_exact| <= 1e-12 * sum_k |a_ik * b_kj| (BASELINE.json north_star).
 *
 * Input preconditions (§II-A "column ids are sorted for each row"; reading R2):
 * every row's col_idx strictly increasing (sorted, no duplicates), 0 <= col < ncols, row_ptr
 * non-decreasing.  opts.validate = 1 checks all of it on the device and fails the plan with
 * SPGEMM_ERR_INVALID_ARGUMENT BEFORE any kernel indexes the operands with those offsets or
 * columns.  With validate = 0 the preconditions are the caller's: a column repeated inside a row
 * of B keeps the structure of C exact (the hash passes count distinct columns) but its value is
 * undefined (the warp tier adds one B row's products without atomics, relying on distinct columns
 * within a row); an unsorted row may be cut wrongly into column pieces; an out-of-range index or
 * offset is undefined behaviour (typically SPGEMM_ERR_CUDA, an illegal address).
 *
 * Errors: every call returns a status; on error a thread-local message is available from
 * spgemm_last_error(), out-parameters are left untouched (plan_out is set to NULL), and the
 * library has released whatever the failed call allocated.  No call aborts the process.
 *
 * Threading: a plan is used by one host thread at a time; distinct plans are independent.
 */
#ifndef SPGEMM_B200_H
#define SPGEMM_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SPGEMM_ABI_VERSION 3

typedef enum {
    SPGEMM_OK = 0,
    SPGEMM_ERR_INVALID_ARGUMENT = 1, /* NULL pointer, bad option, or (validate=1) malformed CSR   */
    SPGEMM_ERR_SHAPE = 2,            /* A.ncols != B.nrows, or row range outside A                 */
    SPGEMM_ERR_INDEX_OVERFLOW = 3,   /* B.ncols > INT32_MAX (col_idx is int32)                     */
    SPGEMM_ERR_BUDGET = 4,           /* device budget cannot hold B + row arrays + one C row       */
    SPGEMM_ERR_HOST_ALLOC = 5,       /* pinned host allocation failed                              */
    SPGEMM_ERR_CUDA = 6,             /* a CUDA runtime call or kernel failed                        */
    SPGEMM_ERR_STATE = 7,            /* call on a plan that failed earlier                           */
    SPGEMM_ERR_CAPACITY = 8,         /* caller's output capacity smaller than nnz(C)                 */
    SPGEMM_ERR_CALLBACK = 9          /* the chunk sink returned non-zero                             */
} spgemm_status;

typedef enum { SPGEMM_HOST = 0, SPGEMM_DEVICE = 1 } spgemm_where;

/* Input CSR matrix (borrowed: must stay valid and unmodified until spgemm_free of every plan
 * built from it).  where == SPGEMM_HOST: row_ptr[0] must be 0.  where == SPGEMM_DEVICE: pointers
 * are device pointers on opts.device (e.g. B after an NCCL broadcast); row_ptr may carry any
 * base, i.e. row r occupies col_idx[row_ptr[r]] .. col_idx[row_ptr[r+1]-1]. */
typedef struct {
    int64_t nrows, ncols, nnz;
    const int64_t *row_ptr; /* [nrows+1], non-decreasing                                         */
    const int32_t *col_idx; /* [nnz], strictly increasing in each row, 0 <= c < ncols <= INT32_MAX */
    const double *values;   /* [nnz]                                                             */
    int32_t where;          /* spgemm_where                                                       */
    int32_t reserved;
} spgemm_csr;

/* Output CSR view (plan-owned memory for spgemm_execute). */
typedef struct {
    int64_t nrows, ncols, nnz;
    int64_t *row_ptr; /* [nrows+1], row_ptr[0] == opts.row_ptr_base                               */
    int32_t *col_idx; /* [nnz]                                                                    */
    double *values;   /* [nnz]                                                                    */
} spgemm_csr_out;

typedef struct {
    int32_t device;        /* CUDA ordinal; -1 = the calling thread's current device                */
    int32_t validate;      /* 1 = check both inputs (row_ptr monotone and within the arrays, columns */
                           /*   strictly increasing and in range) before any kernel reads them     */
    int32_t ring;          /* device C chunk buffers, >= 1 (1 = synchronous ablation); default 2    */
    int32_t profile;       /* 1 = time every kernel class with CUDA events (spgemm_stats)           */
    int64_t row_begin;     /* rows [row_begin, row_end) of A are this plan's row panel (multi-GPU  */
    int64_t row_end;       /*   deal, §III-A); default 0 and -1 = all rows                     */
    void *workspace;       /* caller-owned device buffer of device_budget_bytes used as the arena   */
                           /*   (e.g. from torch's allocator); NULL = the library cudaMallocs it     */
    void *stream;          /* cudaStream_t for kernels; NULL = a library-created stream             */
    int64_t chunk_nnz;     /* > 0: cap every output chunk at this many nonzeros (test hook), else   */
                           /*   chunks are sized from the ring buffers left in the budget           */
    int64_t row_ptr_base;  /* added to every C row_ptr value delivered to the host (rank slices)    */
    int64_t min_chunks;    /* split C into at least this many chunks for D2H overlap; 0 = auto      */
    int32_t fused;         /* 0 = two-phase plan: the symbolic pass of ALL rows runs in spgemm_plan, */
                           /*   nnz(C) is known before execute (reuse, caller-sized outputs);       */
                           /* 1 = fused: spgemm_plan only counts products and cuts chunks from the  */
                           /*   row bounds min(products, ncols); each chunk's symbolic pass + scan  */
                           /*   run inside execute, overlapped with the previous chunk's D2H.       */
                           /*   C = A x A with HOST operands (A and B the same arrays) whose rows   */
                           /*   are short (longest row^2 <= 4096): the plan does not even count --  */
                           /*   chunks are cut on the host from A.row_ptr (nnz(A) x longest row),   */
                           /*   each chunk's count pass runs in execute once its operand pieces     */
                           /*   landed, and products / max_row_products are -1 until executed       */
                           /*   (env SPGEMM_NO_HOST_CUT=1 keeps the count in the plan)               */
    int32_t col_panels;    /* column panels of B (Alg. 3 line 4, §III-D):                   */
                           /*   0 = automatic: B is used whole when it fits the budget; if it does  */
                           /*       not (SPGEMM_ERR_BUDGET), the plan is retried with B cut into the */
                           /*       fewest column panels that fit ("column-panel mode", below);     */
                           /*   1 = never cut B (a B too large for the budget is SPGEMM_ERR_BUDGET); */
                           /*   >= 2 = column-panel mode with exactly this many panels.              */
                           /* Column-panel mode: A and B stream through the device (neither needs  */
                           /* to be resident), each chunk C[i][j] = A[i] x B[j] is computed by the   */
                           /* same kernels, and its row pieces are stored straight into their final */
                           /* place in host C by the GPU (zero-copy stores over the host link).     */
                           /* Plans are two-phase (fused is ignored); sink mode is not available;   */
                           /* output buffers should be page-locked (pageable ones are registered   */
                           /* for the duration of the call).                                         */
    int32_t order;         /* order in which the chunks are computed and transferred (two-phase     */
                           /*   plans; §IV-C): 0 = row order (default: consecutive chunks   */
                           /*   then share ring slots and leave in few large copies); 1 = the       */
                           /*   paper's schedule, decreasing number of flops (products) per chunk,  */
                           /*   every chunk its own copy.  Fused plans and sink mode need 0.        */
    int32_t reserved;
} spgemm_opts;

typedef struct spgemm_plan_s *spgemm_plan_t;

/* Fill *opts with defaults (device -1, validate 0, ring 2, rows all, library arena and stream). */
void spgemm_opts_default(spgemm_opts *opts);

/* Plan = steps S0-S5 + S10 of DESIGN.md: adopt or H2D-copy the inputs into the arena (one
 * allocation of device_budget_bytes; 0 = 90 % of free device memory), count products per row,
 * symbolic hash pass (nnz per row), exclusive scan to C row offsets, and cut the output into
 * chunks that fit the ring buffers left in the budget.  Synchronises the plan's stream.
 * Returns SPGEMM_ERR_BUDGET if B + the row arrays + one ring slot holding the longest C row do
 * not fit.  *plan_out receives the plan (NULL on error). */
spgemm_status spgemm_plan(const spgemm_csr *A, const spgemm_csr *B, size_t device_budget_bytes,
                          const spgemm_opts *opts, spgemm_plan_t *plan_out);

typedef struct {
    int64_t nrows, ncols;       /* shape of this plan's C slice                                   */
    int64_t nnz;                /* nnz of the slice                                               */
    int64_t products;           /* sum of intermediate products (1 multiply-add each; reading R4)  */
    int64_t max_row_nnz, max_row_products;
    int32_t num_chunks, ring;
    int64_t chunk_capacity;     /* nonzeros per ring buffer                                       */
    int64_t arena_bytes, arena_used, ring_bytes;
    int64_t rows_warp, rows_block, rows_global; /* rows per accumulator tier in the symbolic pass   */
    int32_t fused;              /* 1 if the plan is fused (nnz, max_row_nnz = -1 until executed;    */
                                /* products, max_row_products too on host-cut plans, see fused)   */
    int32_t num_copies;         /* output chunks of the last execution: runs of consecutive chunks  */
                                /* (num_chunks = symbolic/numeric units) that share one ring slot   */
                                /* and leave in one copy per array (0 before the first execution)  */
    int32_t col_panels;         /* column panels of B (1 = B used whole)                            */
    int32_t reserved;
    int64_t rows_medium;        /* rows of the medium (128-thread CTA) tier in the symbolic pass;   */
                                /* rows_block counts the large-CTA tier only                          */
} spgemm_info;

spgemm_status spgemm_plan_info(spgemm_plan_t plan, spgemm_info *info);

/* Chunk table: chunk c covers C rows [rows[c], rows[c+1]) and nonzeros [offs[c], offs[c+1])
 * (offsets relative to the slice).  Arrays of num_chunks+1 entries, caller-allocated.
 * SPGEMM_ERR_STATE for a column-panel plan (its chunks are (row unit, column panel) pairs). */
spgemm_status spgemm_plan_chunks(spgemm_plan_t plan, int64_t *rows, int64_t *offs);

/* Execute = steps S6-S8: numeric hash accumulate + sort per chunk into a ring buffer; runs of
 * consecutive chunks share a ring slot and leave as one output chunk (one D2H copy per array,
 * spgemm_info.num_copies), copied into host memory while the next is computed.  Synchronises
 * before return.
 * spgemm_execute_into writes into caller memory: row_ptr [nrows+1] (may be NULL), col_idx and
 * values [nnz]; page-locked memory (cudaHostAlloc / torch pin_memory) gives asynchronous copies,
 * pageable memory is correct but slow.  Repeatable on the same plan.  On a fused plan it needs
 * nnz(C) to be known (an earlier execution), else SPGEMM_ERR_STATE. */
spgemm_status spgemm_execute_into(spgemm_plan_t plan, int64_t *row_ptr, int32_t *col_idx, double *values);

/* Execute into caller memory with room for `capacity` nonzeros (any plan; the way to run a fused
 * plan whose nnz is not known yet).  *nnz_out receives nnz(C).  If nnz(C) > capacity nothing past
 * the capacity is written, the numeric work stops, the symbolic passes finish to report nnz(C),
 * and SPGEMM_ERR_CAPACITY is returned (the plan stays usable). */
spgemm_status spgemm_execute_capacity(spgemm_plan_t plan, int64_t *row_ptr, int32_t *col_idx, double *values,
                                      int64_t capacity, int64_t *nnz_out);

/* Same as spgemm_execute_into, into plan-owned pinned host memory allocated on the first call
 * (kept until free). */
spgemm_status spgemm_execute(spgemm_plan_t plan, spgemm_csr_out *C_out);

/* Sink mode for C larger than host memory: every output chunk (num_copies of them, consecutive
 * row ranges in order) is copied into a pinned staging ring and handed to cb (on the calling
 * thread) while the GPU computes the next chunks.  row_ptr holds
 * rows+1 offsets relative to the start of the chunk; the pointers are valid only during the call.
 * A non-zero return from cb stops execution with SPGEMM_ERR_CALLBACK. */
typedef int (*spgemm_chunk_cb)(void *user, int64_t row0, int64_t row1, const int64_t *row_ptr,
                               const int32_t *col_idx, const double *values, int64_t nnz);
spgemm_status spgemm_execute_stream(spgemm_plan_t plan, spgemm_chunk_cb cb, void *user);

/* S2 on its own ("row analysis", §III-B): u_out[i - row_begin] = the number of
 * intermediate products of row i of A x B, sum over k in A_i* of nnz(B_k*) (the trip count of
 * Alg. 1 line 4, L40), for i in [opts.row_begin, opts.row_end) -- the same k_count kernel the
 * plan runs, without the plan's clamp to min(u_i, ncols).  Reads A.row_ptr, A.col_idx and
 * B.row_ptr only; host operands are copied into a temporary device buffer (cudaMalloc, freed
 * before return; this is an analysis call, not the pipeline).  u_out: HOST memory, one int64 per
 * row; *total_out (may be NULL): the sum.  Synchronises opts.stream (NULL = legacy default).
 * Errors: as spgemm_plan for the operands; opts.validate is ignored (no check of col_idx). */
spgemm_status spgemm_row_products(const spgemm_csr *A, const spgemm_csr *B, const spgemm_opts *opts,
                                  int64_t *u_out, int64_t *total_out);

/* The plan's per-row bounds b_i = min(u_i, ncols) (S2: the count pass's output that sizes
 * the row tiers and the fused chunk cut) copied to HOST bnd_out [nrows of the plan's slice].
 * SPGEMM_ERR_STATE for column-panel plans, and for host-cut plans before their first execution
 * (their count passes run inside execute). */
spgemm_status spgemm_plan_row_bounds(spgemm_plan_t plan, int64_t *bnd_out);

/* Add `delta` to n host row_ptr entries (multi-GPU with fused plans: a rank's global base is known
 * only after every rank has counted its nnz, i.e. after execution).  Host memory, in place. */
spgemm_status spgemm_rebase_host(int64_t *row_ptr, int64_t n, int64_t delta);

/* Change the base added to C row_ptr values (multi-GPU: global offset of this rank's slice,
 * known after the ranks exchange their nnz).  Applies to the next execute. */
spgemm_status spgemm_set_row_ptr_base(spgemm_plan_t plan, int64_t base);

/* One-shot C = A x B on device-resident or host inputs into caller host buffers with capacity
 * nnz_capacity: a fused plan (opts->fused is forced to 1) + spgemm_execute_capacity + free, so the
 * per-chunk symbolic passes overlap the D2H of earlier chunks.  *nnz_out receives nnz(C) (also on
 * SPGEMM_ERR_CAPACITY). */
spgemm_status spgemm_multiply(const spgemm_csr *A, const spgemm_csr *B, size_t device_budget_bytes,
                              const spgemm_opts *opts, int64_t *row_ptr, int32_t *col_idx, double *values,
                              int64_t nnz_capacity, int64_t *nnz_out);

/* Per-kernel-class device time of the last plan/execute when opts.profile = 1 (CUDA events on
 * the launching stream).  name: "count", "symbolic", "scan", "numeric", "d2h", ... */
typedef struct {
    char name[24];
    int32_t launches;
    double ms;    /* total device ms over the launches */
    double bytes; /* algorithmic bytes moved by those launches */
} spgemm_kernel_stat;

/* Fills up to max entries; returns the number of classes in *n.  With opts.profile = 1 the times
 * of the last execution are read from its CUDA events on this call (not inside the execution, so
 * profiling adds only event records to a timed step). */
spgemm_status spgemm_stats(spgemm_plan_t plan, spgemm_kernel_stat *stats, int32_t max, int32_t *n);

/* Timeline of the last execution with opts.profile = 1: 6 doubles per chunk, milliseconds from the
 * start of the execution -- symbolic start, symbolic end (fused plans; -1 otherwise), numeric
 * start, numeric end (compute stream), copy start, copy end (copy stream; set on the last chunk
 * of each output chunk, whose copies carry all of its chunks, -1 on the others).  *n = 6 x chunks;
 * up to max values are written. */
spgemm_status spgemm_timeline(spgemm_plan_t plan, double *out, int64_t max, int64_t *n);

/* NULL-safe; frees the arena (if library-owned), streams, events and plan-owned host memory. */
void spgemm_free(spgemm_plan_t plan);

/* Process-wide number of CUDA kernels this library has launched (all plans, all devices). */
int64_t spgemm_kernel_launches(void);

/* Release the library's caches that no live plan holds: pinned staging memory, and the pooled
 * streams and events that plans take at spgemm_plan and return at spgemm_free (reused so that a
 * plan does not create or destroy CUDA objects; see api.cu "reusable CUDA objects"). */
void spgemm_release_cache(void);

const char *spgemm_status_string(spgemm_status s);
const char *spgemm_last_error(void);
int32_t spgemm_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SPGEMM_B200_H */
