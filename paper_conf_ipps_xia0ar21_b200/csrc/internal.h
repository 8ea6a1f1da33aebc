// internal.h -- launch interface between the host pipeline (api.cu) and the sm_100a kernels
// (kernels.cu).  Not part of the public ABI (include/spgemm.h).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace spg {

// Device view of a CSR operand.  rp is indexed by local row (0..nrows); its values index col/val
// directly, so a device input with an arbitrary base, or a row panel of A, needs no copy.
struct DevCSR {
    const int64_t *rp;
    const int32_t *col;
    const double *val;
    int64_t nrows, ncols;
};

// Accumulator tiers.  A row is handled by
//   W: one warp, shared-memory hash table of TW_* slots   (bound <= CAPW_*)
//   M: one 128-thread CTA, shared-memory hash table of TM_* slots (CAPW_* < bound <= CAPM_*): the
//      rows of a few hundred to two thousand nonzeros that dominate power-law inputs (R-MAT, C3-C5)
//      get up to 8-11 CTAs per SM instead of the B tier's 2 (medium tier)
//   B: one CTA,  shared-memory hash table of TB_* slots.  A row with bound <= CAPB_* is one piece;
//      a longer one (bound <= CAPS_*) is cut into column pieces [lo, hi) processed one after the
//      other in the same table, each A entry's B row resumed from a per-entry cursor -- the paper's
//      column panels with its col_offset cursors (§III-D), applied per row, so every
//      accumulation stays in shared memory.  Pieces are written in column order at a running
//      offset, so the numeric pass needs no per-piece counts from the symbolic pass.
//   G: one CTA,  dense bitmap (+ fp64 array) over all columns in arena scratch (the rest: very
//      long rows, where density makes dense accumulation the cheaper one, §III-B)
// where bound = min(products, ncols) in the symbolic pass and the exact nnz in the numeric pass.
constexpr int WARPS_W = 8;                 // warps per CTA in the W kernels
// hash tables are at most half full (CAP = T / 2; table_log2 in kernels.cu), except the W symbolic
// table whose bound (products) over-estimates nnz (C2: 729 products, 125 nnz per row)
constexpr int TW_SYM = 1024, CAPW_SYM = 768;
constexpr int TW_NUM = 512, CAPW_NUM = 256;
constexpr int THREADS_M = 128;             // medium tier: 16 KB (symbolic) / 24 KB (numeric) tables
constexpr int TM_SYM = 4096, CAPM_SYM = 2048;
constexpr int TM_NUM = 2048, CAPM_NUM = 1024;
// symbolic CTA tier: 512 threads, 16 K-slot tables, 2 CTAs per SM.  Measured on C3 (round 2): 256
// threads / 8 K slots / pieces of 4096 at 4 CTAs per SM gave the same sym_b time (383 ms) but sent
// 6x more rows to the dense tier (sym_g 30 -> 89 ms)
constexpr int THREADS_B = 512;
constexpr int TB_SYM = 16384, CAPB_SYM = 8192;
// numeric CTA tier: 512 threads, 2 CTAs per SM (96 KB table + 13 KB each).  Measured on C3
// (tools/tier_times.py): 256 threads / 4 K slots / pieces of 2048 took 1180 ms, 1024 threads /
// 16 K slots / pieces of 8192 took 1061 ms, this configuration 997 ms.
constexpr int THREADS_BN = 512, PBATCH_BN = 512;
// whole rows up to 5120 nonzeros (the ESC pass holds 6144 products; the hash fallback's 8 K table is
// then up to 5/8 full): 4096 -> 5120 took C3's num_b from 831 to 815 ms
constexpr int TB_NUM = 8192, CAPB_NUM = 5120;
// target bound / nnz per column piece, measured on C3 (profiles/r02/NOTES.md): numeric 3584 / 4096 /
// 4608 / 5120 / 5632 -> 915 / 878 / 853 / 838 / 960 ms (an ESC pass holds <= 6144 products);
// symbolic 10240 / 8192 / 6144 / 4096 -> 426 / 380 / 349 / 350 ms
constexpr int PIECE_SYM = 6144, PIECE_NUM = 5120;
constexpr int64_t CAPS_SYM = 262144, CAPS_NUM = 131072;  // longest pieced row (bound / nnz); beyond: dense tier
constexpr int CURSOR_MAX = 32768;          // longest A row a pieced row may have (cursor scratch)
constexpr int THREADS_G = 512;
// dense tier, split rows: a row is accumulated by KG_PARTS CTAs (1/KG_PARTS of its A entries each)
// into its own dense slot, then swept in KG_SWEEP column ranges by as many CTAs
constexpr int KG_PARTS = 8, KG_SWEEP = 16, THREADS_G2 = 256;
constexpr int ROW_BATCH = 16;              // rows a warp claims per atomic in the W kernels

// Per-pass control block in the arena (zeroed with cudaMemsetAsync before each pass).
struct Ctl {
    unsigned long long row_ctr;   // W kernels: next row batch                      } reset before
    unsigned int nB, nG;          // long-row list lengths                          } every pass
    unsigned long long pass_max;  // symbolic: max nnz of a row in this pass        } (CTL_RESET
    unsigned int nM, bctr;        // medium-tier list length; B-tier claim cursor   }  bytes)
    unsigned int mctr, gctr;      // M / G-tier claim cursors (rows claimed one by one) }
    unsigned int nBl, pad3;       // B tier: one-piece rows, stored from the END of listB }
    unsigned int err;             // bit 0: numeric count mismatch; bit 1: invalid input; bit 2: table overflow
    unsigned int pad;
    unsigned long long sum_u;     // count pass: sum of products
    unsigned long long max_u;     // count pass: max products in a row
    unsigned long long max_bound; // count pass: max min(products, ncols)
    unsigned long long max_nnz;   // symbolic pass: max nnz in a row
    unsigned long long rows_w, rows_b, rows_g;
    unsigned long long max_deg;   // count pass: longest row of A (cursor scratch of pieced rows)
    unsigned long long rows_m;    // rows of the medium tier (symbolic passes)
    unsigned long long pad2[2];
};
constexpr size_t CTL_RESET = 48;  // bytes of Ctl cleared before every pass (row_ctr .. pad3)

// --- launchers (all asynchronous on `s`) ---------------------------------------------------

// S2: bnd[i] = min(sum_{k in A_i} nnz(B_k), ncols) for i in [0, A.nrows) (raw: the sum itself); ctl
// gets the sum and max of products.  Reads A.rp, A.col and B.rp only.
void launch_count(const DevCSR &A, const DevCSR &B, int64_t *u, Ctl *ctl, cudaStream_t s, bool raw = false);

// Validation of a CSR operand (rows strictly increasing, 0 <= col < ncols, rp non-decreasing and
// within [*rp0, *rp0 + nnz], rp0 = device pointer to the first row_ptr entry of the whole array);
// sets ctl->err bit 1.  The caller must check it before any kernel reads the operand.
void launch_validate(const DevCSR &M, const int64_t *rp0, int64_t nnz, Ctl *ctl, cudaStream_t s);

// rp[i] -= sub for i in [0, n)
void launch_rebase(int64_t *rp, int64_t n, int64_t sub, cudaStream_t s);

struct SymArgs {
    DevCSR A, B;
    const int64_t *bnd;  // per-row bound min(products, ncols) from the count pass
    int32_t *nnz;        // out: nnz of every row in [r0, r1)
    int64_t r0, r1;      // rows of this pass
    int32_t *listB, *listG;
    int32_t *listM;      // medium tier (NULL: those rows go to the B tier)
    Ctl *ctl;
    uint32_t *gscratch;  // G tier: per-slot bitmap of ceil(ncols/32) words, zero on entry and exit
    int64_t gstride;     // words per slot
    int gblocks;         // dense slots (= CTAs of the one-CTA-per-row G kernel)
    unsigned long long *gcnt;  // G tier: per slot a counter + KG_SWEEP range counts, zero on entry and exit
    int32_t *cursor;     // B tier, pieced rows: per-CTA 2 x curstride int32 cursors (NULL: none)
    int64_t curstride;
    int bblocks;         // CTAs in the B kernel (the cursor scratch holds that many slots)
    int group;           // lanes per A entry in the W kernel (4, 8, 16, 32)
    int tiers;           // bit 0: launch the CTA tier, bit 1: the dense tier (the host knows when a
                         // pass cannot have such rows and skips launches)
    int batch;           // rows per claim in the W kernel (set by the launcher)
};

// the medium tier is on unless SPGEMM_NO_MEDIUM=1 (A/B knob): its rows then go to the B tier
bool medium_enabled();
// tier bits for a pass whose rows have bound <= maxb: 1 = B (CTA), 2 = G (dense), 4 = M (medium)
inline int sym_tiers(int64_t maxb) {
    const bool m = medium_enabled();
    return (maxb > (m ? CAPM_SYM : CAPW_SYM) ? 1 : 0) | (maxb > CAPS_SYM ? 2 : 0) | (m && maxb > CAPW_SYM ? 4 : 0);
}
inline int num_tiers(int64_t maxnnz) {
    const bool m = medium_enabled();
    return (maxnnz > (m ? CAPM_NUM : CAPW_NUM) ? 1 : 0) | (maxnnz > CAPS_NUM ? 2 : 0) | (m && maxnnz > CAPW_NUM ? 4 : 0);
}

// host2[0] = *end (a chunk's end offset), host2[1] = ctl->pass_max -- zero-copy stores into mapped
// pinned memory, so no small D2H copy queues behind the big ones on the copy engine
void launch_publish(const int64_t *end, const Ctl *ctl, int64_t *host2, cudaStream_t s);

// out[k] = largest column index in A's rows [rows[k], rows[k+1]) (-1 if none)
void launch_seg_max_col(const DevCSR &A, const int64_t *rows, int64_t nseg, int64_t *out, cudaStream_t s);

// out[k] = max(x[rows[k] .. rows[k+1]-1]) for k < nseg (0 for empty segments)
void launch_seg_max(const int64_t *x, const int64_t *rows, int64_t nseg, int64_t *out, cudaStream_t s);
// out[k] = sum(x[rows[k] .. rows[k+1]-1])
void launch_seg_sum(const int64_t *x, const int64_t *rows, int64_t nseg, int64_t *out, cudaStream_t s);
// S3+S4: symbolic pass over all rows (tiering + the four tiers).  ev: NULL or 5 events recorded
// before W, between W/M, M/B, B/G and after G (per-kernel timing on the launching stream).
void launch_symbolic(const SymArgs &a, int num_sms, cudaStream_t s, cudaEvent_t *ev);

// S5: y[1 + t] = y[0] + x[0] + ... + x[t] for t < n, y[0] (the base) read on the device.
// tmp: >= ceil(n / SCAN_TILE) int64 of scratch.
constexpr int SCAN_TILE = 4096;
void launch_scan(const int32_t *x, int64_t n, int64_t *y, int64_t *tmp, cudaStream_t s);
void launch_scan64(const int64_t *x, int64_t n, int64_t *y, int64_t *tmp, cudaStream_t s);

// chunk ids: bounds[c] = first row whose offset - crp[0] >= c * cap_prime (empty ids repeat);
// bounds has nids+1 entries with bounds[nids] = n.
void launch_cut(const int64_t *crp, int64_t n, int64_t cap_prime, int64_t *bounds, int64_t nids, cudaStream_t s);

// crp[i] += delta for i in [0, n]
void launch_add(int64_t *crp, int64_t n, int64_t delta, cudaStream_t s);

struct NumArgs {
    DevCSR A, B;
    const int64_t *crp;  // scanned offsets (any base)
    int64_t r0, r1;      // chunk rows
    int32_t *out_col;    // ring slot: nnz of the chunk
    double *out_val;
    int32_t *listB, *listG;
    int32_t *listM;      // as in SymArgs
    Ctl *ctl;
    uint32_t *gbits;     // G tier scratch: per slot gstride_bits words of bitmap ...
    double *gvals;       // ... and gstride_vals doubles, all zero on entry and exit
    int64_t gstride_bits, gstride_vals;
    int gblocks;
    unsigned long long *gcnt;  // as in SymArgs
    int32_t *cursor;     // as in SymArgs (a separate scratch: both passes may run concurrently)
    int64_t curstride;
    int bblocks;
    int group;
    int tiers;           // as in SymArgs
    int batch;
    int tload;           // W tier table sizing: 0 -> >= 2n slots, 1 -> >= 3n, 2 -> >= 4n (capped at TW_NUM)
};
// S6+S7: numeric pass over chunk rows [r0, r1); ev as in launch_symbolic
void launch_numeric(const NumArgs &a, int num_sms, cudaStream_t s, cudaEvent_t *ev);

// out[i] = crp[idx[i]]
void launch_gather(const int64_t *crp, const int64_t *idx, int64_t n, int64_t *out, cudaStream_t s);

// lanes per A entry for the W kernels from B's average row length
int choose_group(const DevCSR &B, int64_t nnzB);

// occupancy-derived grid sizes (queried once per device)
struct Grids {
    int count_blocks, symw_blocks, numw_blocks, symb_blocks, numb_blocks, symm_blocks, numm_blocks;
};
const Grids &grids(int device, int num_sms);

// process-wide count of kernels launched by the library
long long kernel_launches();

size_t symw_smem();
size_t numw_smem(bool wide);
size_t symb_smem();
size_t numb_smem();
size_t symm_smem();
size_t numm_smem();

// --- column panels of B (NEXT-1; kernels.cu "column panels") ---------------------------------
// hist[col >> shift] += 1 over n column ids (nbins <= 4096)
void launch_col_hist(const int32_t *col, int64_t n, int shift, int nbins, unsigned long long *hist, cudaStream_t s);
// len[k] = entries of piece row k with lo <= col < hi
void launch_panel_len(const DevCSR &Bp, int32_t lo, int32_t hi, int32_t *len, cudaStream_t s);
// copy those entries to col/val at rp[k] (rp: the panel's offsets of the piece's rows)
void launch_panel_fill(const DevCSR &Bp, int32_t lo, const int64_t *rp, int32_t *col, double *val, cudaStream_t s);
// y[r] += x[r] for r < n; atomicMax(mx, max_r y[r]) (mx may be NULL)
void launch_acc_i32(const int32_t *x, int32_t *y, int64_t n, unsigned long long *mx, cudaStream_t s);
// rows [0, n) of chunk C[i][j] from a ring slot to mapped host memory at crpt[r] + pre[r] (k_scatter)
void launch_scatter(const int32_t *scol, const double *sval, const int64_t *crpj, const int32_t *pre,
                    const int64_t *crpt, int64_t n, int32_t *hcol, double *hval, int num_sms, cudaStream_t s);

}  // namespace spg
