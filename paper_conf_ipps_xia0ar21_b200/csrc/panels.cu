// panels.cu -- column-panel mode of the planner and pipeline (B larger than the device budget).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <string>
#include <vector>

#include "host.h"

// ================================================================ column panels of B (NEXT-1)
//
// Mode for a B that does not fit the device budget (the paper's reason for partitioning B at
// all: "to handle cases where either matrix of them is too large to reside in device memory",
// §III-A).  B is cut into P column panels B[j] (Alg. 3 line 4; §III-D) and every
// chunk of C is C[i][j] = A[i] x B[j] (Alg. 3 lines 5-10), computed by the same count / symbolic /
// scan / numeric kernels as the in-core path.  Nothing of A or B needs to be resident: both stream
// through two staging slots on an H2D stream (B rows to build one panel at a time on the device,
// A rows per unit), overlapping the kernels.  Loop order: panels outer, row units inner, so each
// panel is built once per phase.
//   plan     histogram of B's column ids -> balanced panel boundaries; for every panel: build
//            B[j], count + symbolic of every row unit -> nnz of every (row, panel) piece;
//            then C row offsets from the row totals, and per panel the numeric units cut from
//            the exact piece sizes.
//   execute  for every panel: build B[j]; numeric of every unit into a ring slot; a scatter
//            kernel stores each row piece straight into its final place in host C (zero-copy over
//            the host link: a row's pieces from different panels are not contiguous in host C,
//            so one copy-engine transfer per chunk cannot place them).
struct Panels {
    int P = 0;
    std::vector<int32_t> lo;    // P+1 column boundaries
    std::vector<int64_t> pnnz;  // entries of B in each panel
    spgemm_csr A{}, B{};        // borrowed descriptors
    std::vector<int64_t> arp_copy, brp_copy;  // host copies of device operands' row_ptr
    const int64_t *arp = nullptr, *brp = nullptr;  // host row_ptr of A (all rows) and B
    int64_t rb = 0;              // first row of A in this plan
    int32_t *npj = nullptr;      // [R] nnz of the current panel's row pieces
    int32_t *pre = nullptr;      // [R] execute: nnz of each row's pieces in earlier panels
    int32_t *hnp = nullptr;      // pinned host [P][R]: nnz of every (panel, row) piece
    int32_t *tot = nullptr;      // [R] row totals
    int64_t *crpt = nullptr;     // [R+1] C row offsets (slice-relative)
    int64_t *crpj = nullptr;     // [R+1] offsets of the current panel's pieces
    int64_t *bj_rp = nullptr;    // the current panel B[j]
    int32_t *bj_col = nullptr;
    double *bj_val = nullptr;
    int64_t bj_cap = 0;
    char *stage[2] = {nullptr, nullptr};
    size_t stage_bytes = 0;
    cudaEvent_t ev_staged[2] = {}, ev_used[2] = {}, ev_scat_all = nullptr;
    bool used_pending[2] = {false, false};
    int next_slot = 0, cur_slot = 0;
    int64_t *ubnd = nullptr;     // [U] per-unit row bounds
    int32_t *plen = nullptr;     // [max piece rows] panel row lengths
    int64_t unit_rows = 0;
    std::vector<int64_t> bpieces;                 // B row boundaries of the streaming pieces
    std::vector<int64_t> sym_units;               // row boundaries of the symbolic units
    std::vector<std::vector<int64_t>> num_units;  // per panel: row boundaries of the numeric units
    std::vector<int> group;                       // W-kernel lanes per A entry, per panel
    cudaStream_t h = nullptr, z = nullptr;
    int64_t max_piece_nnz = 0;                    // largest (row, panel) piece
    bool validate = false;
    // built panels parked in pinned host memory by the plan (execute then uploads each panel
    // instead of rebuilding it from all of B); NULL if that memory could not be had
    char *hpan = nullptr;
    std::vector<size_t> hoff;                     // per panel: byte offset of rp | col | val
    cudaEvent_t ev_saved = nullptr;
    bool saved_pending = false;
};

void delete_panels(Panels *p) {
    if (p) {
        pin_release(p->hnp);
        pin_release(p->hpan);
    }
    delete p;
}

namespace {

size_t al256(size_t x) { return (x + 255) & ~size_t(255); }

// Rows [r0, r1) of operand M (rp: its host row_ptr) as a device CSR view: device operands are
// viewed in place; host operands are copied into the next staging slot on the H2D stream, after
// the slot's previous user finished on the compute stream, and rebased to 0 there.
DevCSR stage_rows(spgemm_plan_s *P, Panels &Q, const spgemm_csr &M, const int64_t *rp, int64_t r0, int64_t r1,
                  bool vals, const int32_t **col0) {
    const int64_t n = r1 - r0, p0 = rp[r0], p1 = rp[r1];
    if (M.where == SPGEMM_DEVICE) {
        if (col0) *col0 = M.col_idx + p0;
        Q.cur_slot = -1;
        return DevCSR{M.row_ptr + r0, M.col_idx, M.values, n, M.ncols};
    }
    const int sl = Q.next_slot;
    Q.next_slot ^= 1;
    Q.cur_slot = sl;
    char *b = Q.stage[sl];
    const size_t o1 = al256(size_t(n + 1) * 8), o2 = o1 + al256(size_t(p1 - p0) * 4);
    if (o2 + (vals ? size_t(p1 - p0) * 8 : 0) > Q.stage_bytes)
        fail(SPGEMM_ERR_STATE, "internal: staged rows exceed the staging slot");
    int64_t *drp = reinterpret_cast<int64_t *>(b);
    int32_t *dcol = reinterpret_cast<int32_t *>(b + o1);
    double *dval = reinterpret_cast<double *>(b + o2);
    if (Q.used_pending[sl]) CK(cudaStreamWaitEvent(Q.h, Q.ev_used[sl], 0));
    CK(cudaMemcpyAsync(drp, M.row_ptr + r0, size_t(n + 1) * 8, cudaMemcpyHostToDevice, Q.h));
    if (p1 > p0) {
        CK(cudaMemcpyAsync(dcol, M.col_idx + p0, size_t(p1 - p0) * 4, cudaMemcpyHostToDevice, Q.h));
        if (vals) CK(cudaMemcpyAsync(dval, M.values + p0, size_t(p1 - p0) * 8, cudaMemcpyHostToDevice, Q.h));
    }
    CK(cudaEventRecord(Q.ev_staged[sl], Q.h));
    CK(cudaStreamWaitEvent(P->stream, Q.ev_staged[sl], 0));
    launch_rebase(drp, n + 1, p0, P->stream);
    CKL("rebase staged rows");
    if (col0) *col0 = dcol;
    return DevCSR{drp, dcol, dval, n, M.ncols};
}

// the kernels reading the current staging slot have been enqueued on the compute stream
void stage_done(spgemm_plan_s *P, Panels &Q) {
    if (Q.cur_slot < 0) return;
    CK(cudaEventRecord(Q.ev_used[Q.cur_slot], P->stream));
    Q.used_pending[Q.cur_slot] = true;
}

// bytes a staging slot needs for rows [r0, r1)
size_t stage_need(const int64_t *rp, int64_t r0, int64_t r1, bool vals) {
    const int64_t e = rp[r1] - rp[r0];
    return al256(size_t(r1 - r0 + 1) * 8) + al256(size_t(e) * 4) + (vals ? size_t(e) * 8 : 0);
}

// row boundaries [0 = b0 < b1 < ... = n) of consecutive row ranges, each as long as possible
// subject to ok(r0, r1) (monotone in r1; a single row must satisfy it)
template <typename OK>
std::vector<int64_t> cut_rows(int64_t n, OK ok) {
    std::vector<int64_t> b{0};
    int64_t r0 = 0;
    while (r0 < n) {
        int64_t lo = r0 + 1, hi = n;  // largest r1 in [lo, hi] with ok(r0, r1)
        if (!ok(r0, lo)) fail(SPGEMM_ERR_BUDGET, "budget too small for one row in column-panel mode");
        while (lo < hi) {
            const int64_t m = lo + (hi - lo + 1) / 2;
            if (ok(r0, m)) lo = m;
            else hi = m - 1;
        }
        b.push_back(lo);
        r0 = lo;
    }
    return b;
}

// B[j] on the device: B streams through the staging slots; per piece, panel row lengths, the
// chained scan (y[0] of a piece is the last offset of the previous one) and the fill
DevCSR build_panel(spgemm_plan_s *P, Panels &Q, int j) {
    cudaStream_t s = P->stream;
    CK(cudaMemsetAsync(Q.bj_rp, 0, sizeof(int64_t), s));
    for (size_t q = 0; q + 1 < Q.bpieces.size(); ++q) {
        const int64_t k0 = Q.bpieces[q], k1 = Q.bpieces[q + 1];
        DevCSR v = stage_rows(P, Q, Q.B, Q.brp, k0, k1, true, nullptr);
        launch_panel_len(v, Q.lo[j], Q.lo[j + 1], Q.plen, s);
        launch_scan(Q.plen, k1 - k0, Q.bj_rp + k0, P->tmp, s);
        launch_panel_fill(v, Q.lo[j], Q.bj_rp + k0, Q.bj_col, Q.bj_val, s);
        CKL("panel build");
        stage_done(P, Q);
    }
    return DevCSR{Q.bj_rp, Q.bj_col, Q.bj_val, Q.B.nrows, Q.B.ncols};
}

void panel_plan(const spgemm_csr *Ah, const spgemm_csr *Bh, size_t budget, const spgemm_opts *o,
                spgemm_plan_s *P) {
    NvtxRange nv("spgemm_plan (column panels)");
    check_csr(Ah, "A");
    check_csr(Bh, "B");
    if (Ah->ncols != Bh->nrows)
        fail(SPGEMM_ERR_SHAPE, "A.ncols (" + std::to_string(Ah->ncols) + ") != B.nrows (" + std::to_string(Bh->nrows) + ")");
    if (Bh->ncols > INT32_MAX) fail(SPGEMM_ERR_INDEX_OVERFLOW, "B.ncols exceeds INT32_MAX (col_idx is int32)");
    spgemm_opts opts;
    spgemm_opts_default(&opts);
    if (o) opts = *o;
    const int64_t rb = opts.row_begin, re = opts.row_end < 0 ? Ah->nrows : opts.row_end;
    if (rb < 0 || re < rb || re > Ah->nrows) fail(SPGEMM_ERR_SHAPE, "row range outside A");
    if (re - rb > INT32_MAX) fail(SPGEMM_ERR_INDEX_OVERFLOW, "more than INT32_MAX rows in one plan");
    if (opts.ring < 1 || opts.ring > 64) fail(SPGEMM_ERR_INVALID_ARGUMENT, "ring must be in [1, 64]");
    if (opts.device >= 0) {
        CK(cudaSetDevice(opts.device));
        P->device = opts.device;
    } else {
        CK(cudaGetDevice(&P->device));
    }
    CK(cudaDeviceGetAttribute(&P->num_sms, cudaDevAttrMultiProcessorCount, P->device));
    P->fused = false;
    P->ring = opts.ring;
    P->row_begin = rb;
    P->R = re - rb;
    P->ncols = Bh->ncols;
    P->nnzB = Bh->nnz;
    P->base_wanted = opts.row_ptr_base;
    P->pan = new Panels();
    Panels &Q = *P->pan;
    Q.A = *Ah;
    Q.B = *Bh;
    Q.rb = rb;
    Q.validate = opts.validate != 0;
    if (Q.validate) {  // host row_ptr monotone before any staging copy is sized from it
        check_rows_host(Ah, "A");
        check_rows_host(Bh, "B");
    }
    P->res = res_acquire(P->device);
    Res *rs = P->res;
    P->stream = opts.stream ? (cudaStream_t)opts.stream : rs->stream(rs->own);
    P->copy = rs->stream(rs->copy);  // the scatter stream
    Q.h = rs->stream(rs->hstream);
    Q.z = P->copy;
    P->ev_num = rs->events(Res::PLAIN, 0, P->ring);
    P->ev_d2h = rs->events(Res::PLAIN, P->ring, P->ring);
    P->ev_ready = rs->events(Res::PLAIN, 2 * P->ring, 1)[0];
    {
        auto e = rs->events(Res::PLAIN, 2 * size_t(P->ring) + 1, 6);
        Q.ev_staged[0] = e[0];
        Q.ev_staged[1] = e[1];
        Q.ev_used[0] = e[2];
        Q.ev_used[1] = e[3];
        Q.ev_scat_all = e[4];
        Q.ev_saved = e[5];
    }
    cudaStream_t s = P->stream;
    const int64_t R = P->R, K = Bh->nrows;

    // host views of the row pointers (device operands: one D2H each)
    if (Ah->where == SPGEMM_DEVICE) {
        Q.arp_copy.resize(Ah->nrows + 1);
        CK(cudaMemcpy(Q.arp_copy.data(), Ah->row_ptr, sizeof(int64_t) * (Ah->nrows + 1), cudaMemcpyDeviceToHost));
        Q.arp = Q.arp_copy.data();
    } else {
        Q.arp = Ah->row_ptr;
    }
    if (Bh->where == SPGEMM_DEVICE) {
        Q.brp_copy.resize(K + 1);
        CK(cudaMemcpy(Q.brp_copy.data(), Bh->row_ptr, sizeof(int64_t) * (K + 1), cudaMemcpyDeviceToHost));
        Q.brp = Q.brp_copy.data();
    } else {
        Q.brp = Bh->row_ptr;
    }
    if (Q.validate && (Ah->where == SPGEMM_DEVICE || Bh->where == SPGEMM_DEVICE)) {  // the host views too
        spgemm_csr av = *Ah, bv = *Bh;
        av.where = bv.where = SPGEMM_HOST;
        av.row_ptr = Q.arp;
        bv.row_ptr = Q.brp;
        check_rows_host(&av, "A");
        check_rows_host(&bv, "B");
    }
    const int64_t *arp = Q.arp + rb;  // plan rows
    int64_t max_deg = 0, max_brow = 0;
    for (int64_t r = 0; r < R; ++r) max_deg = std::max<int64_t>(max_deg, arp[r + 1] - arp[r]);
    for (int64_t k = 0; k < K; ++k) max_brow = std::max<int64_t>(max_brow, Q.brp[k + 1] - Q.brp[k]);
    P->nnzA = arp[R] - arp[0];

    // S9 arena
    if (opts.workspace) {
        if (budget == 0) fail(SPGEMM_ERR_INVALID_ARGUMENT, "workspace given with a zero budget");
        P->arena = (char *)opts.workspace;
        P->arena_bytes = budget;
    } else {
        if (budget == 0) {
            size_t fr = 0, tot = 0;
            CK(cudaMemGetInfo(&fr, &tot));
            budget = size_t(double(fr) * 0.9);
        }
        if (cudaMalloc(&P->arena, budget) != cudaSuccess) {
            cudaGetLastError();
            fail(SPGEMM_ERR_BUDGET, "cudaMalloc of the " + std::to_string(budget) + "-byte arena failed");
        }
        P->arena_bytes = budget;
        P->own_arena = true;
    }

    // staging slots: >= the largest single row of A or B (structure + values)
    const size_t row_need = std::max(al256(16) + al256(size_t(max_deg) * 4) + size_t(max_deg) * 8,
                                     al256(16) + al256(size_t(max_brow) * 4) + size_t(max_brow) * 8);
    Q.stage_bytes = al256(std::max<size_t>(row_need, std::min<size_t>(std::max<size_t>(budget / 32, 256 << 10), 64 << 20)));
    Q.unit_rows = std::max<int64_t>(1, std::min<int64_t>(std::max<int64_t>(R, 1), int64_t(1) << 20));
    Q.unit_rows = std::min<int64_t>(Q.unit_rows, std::max<int64_t>(4096, int64_t(budget / 64 / 40)));
    Q.bpieces = cut_rows(K, [&](int64_t a, int64_t b) { return stage_need(Q.brp, a, b, true) <= Q.stage_bytes; });
    int64_t max_piece_rows = 1;
    for (size_t q = 0; q + 1 < Q.bpieces.size(); ++q)
        max_piece_rows = std::max<int64_t>(max_piece_rows, Q.bpieces[q + 1] - Q.bpieces[q]);

    // fixed arena part
    P->ctl = P->alloc<Ctl>(2, "ctl");
    P->tmp = P->alloc<int64_t>((std::max<int64_t>(std::max(R, K), Q.unit_rows) + SCAN_TILE - 1) / SCAN_TILE + 64,
                               "scan scratch");
    Q.tot = P->alloc<int32_t>(R, "row totals");
    Q.npj = P->alloc<int32_t>(R, "panel piece counts");
    Q.pre = P->alloc<int32_t>(R, "earlier-panel piece counts");
    Q.crpt = P->alloc<int64_t>(R + 1, "C.row_ptr");
    Q.crpj = P->alloc<int64_t>(R + 1, "panel offsets");
    Q.bj_rp = P->alloc<int64_t>(K + 1, "B[j].row_ptr");
    Q.stage[0] = P->alloc<char>(int64_t(Q.stage_bytes), "staging slot 0");
    Q.stage[1] = P->alloc<char>(int64_t(Q.stage_bytes), "staging slot 1");
    Q.ubnd = P->alloc<int64_t>(Q.unit_rows, "unit bounds");
    Q.plen = P->alloc<int32_t>(max_piece_rows, "panel lengths");
    P->listB = P->alloc<int32_t>(Q.unit_rows, "listB");
    P->listG = P->alloc<int32_t>(Q.unit_rows, "listG");
    P->listBn = P->alloc<int32_t>(Q.unit_rows, "numeric listB");
    P->listM = P->alloc<int32_t>(Q.unit_rows, "listM");
    P->listMn = P->alloc<int32_t>(Q.unit_rows, "numeric listM");
    P->listGn = P->alloc<int32_t>(Q.unit_rows, "numeric listG");
    const int nbins_max = 4096;
    unsigned long long *dhist = P->alloc<unsigned long long>(nbins_max, "column histogram");
    CK(cudaMemsetAsync(P->ctl, 0, 2 * sizeof(Ctl), s));
    // long-row scratch: cursors of the pieced CTA tier and one dense-tier CTA slot per pass
    {
        const Grids &gr = grids(P->device, P->num_sms);
        P->curstride = (std::min<int64_t>(std::max<int64_t>(max_deg, 1), CURSOR_MAX) + 31) & ~int64_t(31);
        P->bblocks_sym = gr.symb_blocks;
        P->bblocks_num = gr.numb_blocks;
        P->cur_sym = P->alloc<int32_t>(int64_t(P->bblocks_sym) * 2 * P->curstride, "CTA-tier cursors (symbolic)");
        P->cur_num = P->alloc<int32_t>(int64_t(P->bblocks_num) * 2 * P->curstride, "CTA-tier cursors (numeric)");
        const int64_t nwords = (P->ncols + 31) / 32;
        P->gstride_bits = (nwords + 63) & ~int64_t(63);
        P->gstride_vals = (P->ncols + 31) & ~int64_t(31);
        P->gblocks = 1;
        P->gbits = P->alloc<uint32_t>(P->gstride_bits, "dense-tier bitmap (numeric)");
        P->gbits_sym = P->alloc<uint32_t>(P->gstride_bits, "dense-tier bitmap (symbolic)");
        P->gvals = P->alloc<double>(P->gstride_vals, "dense-tier values");
        P->gcnt = P->alloc<unsigned long long>(2 * (KG_SWEEP + 1), "dense-tier counters");
        CK(cudaMemsetAsync(P->gcnt, 0, sizeof(unsigned long long) * 2 * (KG_SWEEP + 1), s));
        CK(cudaMemsetAsync(P->gbits, 0, size_t(P->gstride_bits) * 4, s));
        CK(cudaMemsetAsync(P->gbits_sym, 0, size_t(P->gstride_bits) * 4, s));
        CK(cudaMemsetAsync(P->gvals, 0, size_t(P->gstride_vals) * 8, s));
    }

    // histogram of B's column ids (and validation of B) over the streamed pieces
    int shift = 0;
    while (P->ncols > 0 && ((P->ncols - 1) >> shift) >= nbins_max) ++shift;
    const int nbins = P->ncols > 0 ? int(((P->ncols - 1) >> shift) + 1) : 1;
    CK(cudaMemsetAsync(dhist, 0, sizeof(unsigned long long) * nbins, s));
    for (size_t q = 0; q + 1 < Q.bpieces.size(); ++q) {
        const int64_t k0 = Q.bpieces[q], k1 = Q.bpieces[q + 1];
        const int32_t *c0 = nullptr;
        DevCSR v = stage_rows(P, Q, Q.B, Q.brp, k0, k1, false, &c0);
        if (Q.validate)  // (k_col_hist skips out-of-range ids; the plan fails below if any)
            launch_validate(v, Bh->where == SPGEMM_DEVICE ? Bh->row_ptr : v.rp,
                            Bh->where == SPGEMM_DEVICE ? Bh->nnz : Q.brp[k1] - Q.brp[k0], P->ctl, s);
        launch_col_hist(c0, Q.brp[k1] - Q.brp[k0], shift, nbins, dhist, s);
        CKL("column histogram");
        stage_done(P, Q);
    }
    std::vector<unsigned long long> hist(nbins);
    CK(cudaMemcpyAsync(hist.data(), dhist, sizeof(unsigned long long) * nbins, cudaMemcpyDeviceToHost, s));
    Ctl hc;
    CK(cudaMemcpyAsync(&hc, P->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (hc.err & 2u) fail(SPGEMM_ERR_INVALID_ARGUMENT, "input validation failed (B)");
    if (Q.validate && Ah->where == SPGEMM_HOST) {
        // A streams through the staging slots as well
        auto ab = cut_rows(R, [&](int64_t a, int64_t b) { return stage_need(arp, a, b, false) <= Q.stage_bytes; });
        for (size_t q = 0; q + 1 < ab.size(); ++q) {
            DevCSR v = stage_rows(P, Q, Q.A, Q.arp, rb + ab[q], rb + ab[q + 1], false, nullptr);
            launch_validate(v, v.rp, Q.arp[rb + ab[q + 1]] - Q.arp[rb + ab[q]], P->ctl, s);
            stage_done(P, Q);
        }
    } else if (Q.validate) {
        launch_validate(DevCSR{Ah->row_ptr + rb, Ah->col_idx, Ah->values, R, Ah->ncols}, Ah->row_ptr, Ah->nnz, P->ctl, s);
    }
    if (Q.validate) {  // A checked before any kernel reads it
        Ctl hv;
        CK(cudaMemcpyAsync(&hv, P->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (hv.err & 2u) fail(SPGEMM_ERR_INVALID_ARGUMENT, "input validation failed (A)");
    }

    // panel count and boundaries: the fewest panels whose largest one fits, with at least ~20% of
    // the budget left for the ring (the piece counts of every (panel, row) wait in pinned host
    // memory, 4 B each)
    auto bounds_for = [&](int np, std::vector<int32_t> &lo, std::vector<int64_t> &pn) {
        lo.assign(np + 1, 0);
        pn.assign(np, 0);
        const double tgt = double(Bh->nnz) / np;
        unsigned long long cum = 0;
        int j = 0;
        for (int b = 0; b < nbins; ++b) {
            cum += hist[b];
            pn[j] += (int64_t)hist[b];
            if (j + 1 < np && double(cum) >= tgt * (j + 1)) lo[++j] = (int32_t)std::min<int64_t>(int64_t(b + 1) << shift, P->ncols);
        }
        for (int q = j + 1; q <= np; ++q) lo[q] = (int32_t)P->ncols;
        lo[np] = (int32_t)P->ncols;
        int64_t mx = 0;
        for (auto x : pn) mx = std::max(mx, x);
        return mx;
    };
    const size_t fixed = P->used;
    int np = opts.col_panels >= 2 ? opts.col_panels : 0;
    if (np == 0) {
        for (int t = 2; t <= 256 && np == 0; ++t) {
            std::vector<int32_t> lo;
            std::vector<int64_t> pn;
            const int64_t mx = bounds_for(t, lo, pn);
            const size_t need = fixed + al256(size_t(std::max<int64_t>(mx, 1)) * 4) +
                                size_t(std::max<int64_t>(mx, 1)) * 8 + 512;
            if (double(need) <= 0.8 * double(P->arena_bytes)) np = t;
        }
        if (np == 0) fail(SPGEMM_ERR_BUDGET, "budget cannot hold one column panel of B (tried up to 256 panels)");
    }
    Q.P = np;
    P->col_panels = np;
    const int64_t mxp = bounds_for(np, Q.lo, Q.pnnz);
    Q.hnp = (int32_t *)pin_acquire(sizeof(int32_t) * size_t(np) * size_t(std::max<int64_t>(R, 1)));
    Q.bj_cap = std::max<int64_t>(mxp, 1);
    Q.bj_col = P->alloc<int32_t>(Q.bj_cap, "B[j].col_idx");
    Q.bj_val = P->alloc<double>(Q.bj_cap, "B[j].values");
    Q.group.assign(np, 32);
    {
        size_t off = 0;
        Q.hoff.assign(size_t(np) * 3, 0);
        // every parked array starts on a host page (copies to or from an offset within a page
        // ran up to 6 % slower on some boxes, tools/d2h_offsets.py)
        auto al4k = [](size_t x) { return (x + 4095) & ~size_t(4095); };
        for (int j = 0; j < np; ++j) {
            Q.hoff[3 * j] = off;
            off += al4k(size_t(K + 1) * 8);
            Q.hoff[3 * j + 1] = off;
            off += al4k(size_t(Q.pnnz[j]) * 4);
            Q.hoff[3 * j + 2] = off;
            off += al4k(size_t(Q.pnnz[j]) * 8);
        }
        try {
            Q.hpan = (char *)pin_acquire(off);
        } catch (const Err &) {
            Q.hpan = nullptr;  // execute rebuilds every panel from B instead
            cudaGetLastError();
        }
    }

    // symbolic phase: per panel, build B[j] then count + symbolic of every row unit
    Q.sym_units = cut_rows(R, [&](int64_t a, int64_t b) {
        return b - a <= Q.unit_rows && stage_need(arp, a, b, false) <= Q.stage_bytes;
    });
    CK(cudaMemsetAsync(Q.tot, 0, sizeof(int32_t) * R, s));
    for (int j = 0; j < np; ++j) {
        if (Q.saved_pending) CK(cudaStreamWaitEvent(s, Q.ev_saved, 0));  // B[j-1] parked on the host
        DevCSR Bj = build_panel(P, Q, j);
        if (Q.hpan) {  // park B[j] in pinned host memory on the copy stream, under the symbolic units
            CK(cudaEventRecord(P->ev_ready, s));
            CK(cudaStreamWaitEvent(Q.z, P->ev_ready, 0));
            CK(cudaMemcpyAsync(Q.hpan + Q.hoff[3 * j], Q.bj_rp, size_t(K + 1) * 8, cudaMemcpyDeviceToHost, Q.z));
            CK(cudaMemcpyAsync(Q.hpan + Q.hoff[3 * j + 1], Q.bj_col, size_t(Q.pnnz[j]) * 4, cudaMemcpyDeviceToHost, Q.z));
            CK(cudaMemcpyAsync(Q.hpan + Q.hoff[3 * j + 2], Q.bj_val, size_t(Q.pnnz[j]) * 8, cudaMemcpyDeviceToHost, Q.z));
            CK(cudaEventRecord(Q.ev_saved, Q.z));
            Q.saved_pending = true;
        }
        DevCSR Bc = Bj;  // the count's bound uses the panel width
        Bc.ncols = std::max<int64_t>(1, int64_t(Q.lo[j + 1]) - Q.lo[j]);
        Q.group[j] = choose_group(Bj, Q.pnnz[j]);
        for (size_t u = 0; u + 1 < Q.sym_units.size(); ++u) {
            const int64_t r0 = Q.sym_units[u], r1 = Q.sym_units[u + 1];
            DevCSR v = stage_rows(P, Q, Q.A, Q.arp, rb + r0, rb + r1, false, nullptr);
            launch_count(v, Bc, Q.ubnd, P->ctl, s);
            CKL("count");
            SymArgs sa{};
            sa.A = v;
            sa.B = Bj;
            sa.bnd = Q.ubnd;
            sa.nnz = Q.npj + r0;
            sa.r0 = 0;
            sa.r1 = r1 - r0;
            sa.listB = P->listB;
            sa.listM = P->listM;
            sa.listG = P->listG;
            sa.ctl = P->ctl;
            sa.gscratch = P->gbits_sym;
            sa.gcnt = P->gcnt;
    sa.gcnt = P->gcnt;
            sa.gstride = P->gstride_bits;
            sa.gblocks = P->gblocks;
            sa.cursor = P->cur_sym;
            sa.curstride = P->curstride;
            sa.bblocks = P->bblocks_sym;
            sa.group = Q.group[j];
            sa.tiers = 3 | (medium_enabled() ? 4 : 0);
            launch_symbolic(sa, P->num_sms, s, nullptr);
            CKL("symbolic");
            stage_done(P, Q);
        }
        // row totals; the panel's piece counts go to pinned host memory
        launch_acc_i32(Q.npj, Q.tot, R, j + 1 == np ? &P->ctl[1].max_nnz : nullptr, s);
        CKL("row totals");
        if (R > 0) CK(cudaMemcpyAsync(Q.hnp + size_t(j) * R, Q.npj, sizeof(int32_t) * R, cudaMemcpyDeviceToHost, s));
    }
    // C row offsets from the row totals
    CK(cudaMemsetAsync(Q.crpt, 0, sizeof(int64_t), s));
    launch_scan(Q.tot, R, Q.crpt, P->tmp, s);
    CKL("row totals");
    int64_t total = 0;
    CK(cudaMemcpyAsync(&total, Q.crpt + R, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    Ctl hc2[2];
    CK(cudaMemcpyAsync(hc2, P->ctl, 2 * sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (hc2[0].err & 2u) fail(SPGEMM_ERR_INVALID_ARGUMENT, "input validation failed (A)");
    P->nnz = total;
    P->products = (int64_t)hc2[0].sum_u;
    P->max_u = (int64_t)hc2[0].max_u;
    P->max_nnz = (int64_t)hc2[1].max_nnz;
    Q.max_piece_nnz = (int64_t)hc2[0].max_nnz;
    P->rows_w = (int64_t)hc2[0].rows_w;
    P->rows_b = (int64_t)hc2[0].rows_b;
    P->rows_g = (int64_t)hc2[0].rows_g;
    P->rows_m = (int64_t)hc2[0].rows_m;
    CK(cudaMemsetAsync(&P->ctl[1], 0, sizeof(Ctl), s));

    // ring from what is left; numeric units per panel from the exact piece sizes
    {
        const size_t freeb = P->arena_bytes > P->used + 4096 ? P->arena_bytes - P->used - 4096 : 0;
        int64_t cap = int64_t(((freeb / P->ring) & ~size_t(255)) / 12) & ~int64_t(63);
        if (opts.chunk_nnz > 0) cap = std::min<int64_t>(cap, std::max<int64_t>(opts.chunk_nnz, Q.max_piece_nnz));
        if (cap < std::max<int64_t>(Q.max_piece_nnz, 1))
            fail(SPGEMM_ERR_BUDGET, "ring buffer of " + std::to_string(cap) +
                                        " nonzeros cannot hold the longest row piece (" + std::to_string(Q.max_piece_nnz) + ")");
        P->cap = cap;
    }
    int64_t *hcrp = (int64_t *)pin_acquire(sizeof(int64_t) * (R + 1));
    struct Rel {
        void *p;
        ~Rel() { pin_release(p); }
    } rel{hcrp};
    Q.num_units.assign(np, {});
    int64_t nunits = 0;
    for (int j = 0; j < np; ++j) {
        if (R > 0) CK(cudaMemcpyAsync(Q.npj, Q.hnp + size_t(j) * R, sizeof(int32_t) * R, cudaMemcpyHostToDevice, s));
        CK(cudaMemsetAsync(Q.crpj, 0, sizeof(int64_t), s));
        launch_scan(Q.npj, R, Q.crpj, P->tmp, s);
        CKL("panel scan");
        CK(cudaMemcpyAsync(hcrp, Q.crpj, sizeof(int64_t) * (R + 1), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        Q.num_units[j] = cut_rows(R, [&](int64_t a, int64_t b) {
            return b - a <= Q.unit_rows && hcrp[b] - hcrp[a] <= P->cap && stage_need(arp, a, b, true) <= Q.stage_bytes;
        });
        nunits += int64_t(Q.num_units[j].size()) - 1;
    }
    P->ring_col.assign(P->ring, nullptr);
    P->ring_val.assign(P->ring, nullptr);
    for (int r = 0; r < P->ring; ++r) {
        P->ring_val[r] = P->alloc<double>(P->cap, "ring values");
        P->ring_col[r] = P->alloc<int32_t>(P->cap, "ring col_idx");
    }
    P->ring_bytes = size_t(P->ring) * size_t(P->cap) * 12;
    P->num_groups = 0;
    P->chunk_offs.clear();
    P->chunk_rows.clear();
    P->panel_units = nunits;
    if (Q.saved_pending) CK(cudaStreamWaitEvent(s, Q.ev_saved, 0));
    CK(cudaStreamSynchronize(s));
}

// device-accessible view of caller host memory for the scatter kernel (zero-copy): page-locked
// memory is used as is; pageable memory is registered for the call
struct HostMap {
    std::vector<void *> reg;
    void *map(void *p, size_t bytes) {
        if (!p || bytes == 0) return p;
        void *d = nullptr;
        if (cudaHostGetDevicePointer(&d, p, 0) == cudaSuccess && d) return d;
        cudaGetLastError();
        CK(cudaHostRegister(p, bytes, cudaHostRegisterMapped));
        reg.push_back(p);
        CK(cudaHostGetDevicePointer(&d, p, 0));
        return d;
    }
    ~HostMap() {
        for (auto p : reg) cudaHostUnregister(p);
    }
};

int64_t panel_run(spgemm_plan_s *P, int64_t *rp_out, int32_t *col_out, double *val_out, int64_t capacity,
                  const Sink *sink, bool *overflow) {
    NvtxRange nv("spgemm_execute (column panels)");
    if (P->failed) fail(SPGEMM_ERR_STATE, "plan is in a failed state");
    if (sink) fail(SPGEMM_ERR_INVALID_ARGUMENT, "sink mode is not available with column panels of B (a row of C is "
                                                "complete only after the last panel)");
    DeviceGuard g(P->device);
    Panels &Q = *P->pan;
    cudaStream_t s = P->stream, z = Q.z;
    const int64_t R = P->R, total = P->nnz;
    *overflow = total > capacity;
    if (*overflow || (!col_out && total > 0)) return total;
    HostMap hm;
    int32_t *hcol = (int32_t *)hm.map(col_out, sizeof(int32_t) * size_t(total));
    double *hval = (double *)hm.map(val_out, sizeof(double) * size_t(total));
    CK(cudaEventRecord(P->ev_ready, s));
    CK(cudaStreamWaitEvent(z, P->ev_ready, 0));
    CK(cudaStreamWaitEvent(Q.h, P->ev_ready, 0));
    std::vector<bool> slot_used(P->ring, false);
    int64_t unit = 0;
    CK(cudaMemsetAsync(Q.pre, 0, sizeof(int32_t) * R, s));
    for (int j = 0; j < Q.P; ++j) {
        DevCSR Bj{Q.bj_rp, Q.bj_col, Q.bj_val, Q.B.nrows, Q.B.ncols};
        if (Q.hpan) {  // upload the panel parked by the plan (after panel j-1's numeric passes, in order on s)
            const int64_t K = Q.B.nrows;
            CK(cudaMemcpyAsync(Q.bj_rp, Q.hpan + Q.hoff[3 * j], size_t(K + 1) * 8, cudaMemcpyHostToDevice, s));
            CK(cudaMemcpyAsync(Q.bj_col, Q.hpan + Q.hoff[3 * j + 1], size_t(Q.pnnz[j]) * 4, cudaMemcpyHostToDevice, s));
            CK(cudaMemcpyAsync(Q.bj_val, Q.hpan + Q.hoff[3 * j + 2], size_t(Q.pnnz[j]) * 8, cudaMemcpyHostToDevice, s));
        } else {
            Bj = build_panel(P, Q, j);
        }
        if (j > 0) {  // panel j-1's scatters still read crpj, npj and pre
            CK(cudaStreamWaitEvent(s, Q.ev_scat_all, 0));
            launch_acc_i32(Q.npj, Q.pre, R, nullptr, s);
            CKL("earlier pieces");
        }
        if (R > 0) CK(cudaMemcpyAsync(Q.npj, Q.hnp + size_t(j) * R, sizeof(int32_t) * R, cudaMemcpyHostToDevice, s));
        CK(cudaMemsetAsync(Q.crpj, 0, sizeof(int64_t), s));
        launch_scan(Q.npj, R, Q.crpj, P->tmp, s);
        CKL("panel scan");
        const auto &U = Q.num_units[j];
        for (size_t u = 0; u + 1 < U.size(); ++u, ++unit) {
            const int64_t r0 = U[u], r1 = U[u + 1];
            const int b = int(unit % P->ring);
            if (slot_used[b]) CK(cudaStreamWaitEvent(s, P->ev_d2h[b], 0));
            DevCSR v = stage_rows(P, Q, Q.A, Q.arp, Q.rb + r0, Q.rb + r1, true, nullptr);
            NumArgs na{};
            na.A = v;
            na.B = Bj;
            na.crp = Q.crpj + r0;
            na.r0 = 0;
            na.r1 = r1 - r0;
            na.out_col = P->ring_col[b];
            na.out_val = P->ring_val[b];
            na.listB = P->listBn;
            na.listM = P->listMn;
            na.listG = P->listGn;
            na.ctl = P->ctl + 1;
            na.gbits = P->gbits;
            na.gvals = P->gvals;
            na.gcnt = P->gcnt ? P->gcnt + size_t(P->gblocks) * (KG_SWEEP + 1) : nullptr;
    na.gcnt = P->gcnt ? P->gcnt + size_t(P->gblocks) * (KG_SWEEP + 1) : nullptr;
            na.gstride_bits = P->gstride_bits;
            na.gstride_vals = P->gstride_vals;
            na.gblocks = P->gblocks;
            na.cursor = P->cur_num;
            na.curstride = P->curstride;
            na.bblocks = P->bblocks_num;
            na.group = Q.group[j];
            na.tiers = num_tiers(Q.max_piece_nnz);
            launch_numeric(na, P->num_sms, s, nullptr);
            CKL("numeric");
            stage_done(P, Q);
            CK(cudaEventRecord(P->ev_num[b], s));
            CK(cudaStreamWaitEvent(z, P->ev_num[b], 0));
            launch_scatter(P->ring_col[b], P->ring_val[b], Q.crpj + r0, Q.pre + r0, Q.crpt + r0, r1 - r0, hcol, hval,
                           P->num_sms, z);
            CKL("scatter");
            CK(cudaEventRecord(P->ev_d2h[b], z));
            slot_used[b] = true;
        }
        CK(cudaEventRecord(Q.ev_scat_all, z));
    }
    CK(cudaStreamWaitEvent(s, Q.ev_scat_all, 0));
    if (rp_out) {  // C.row_ptr + base (crpj is free now)
        CK(cudaMemcpyAsync(Q.crpj, Q.crpt, sizeof(int64_t) * (R + 1), cudaMemcpyDeviceToDevice, s));
        launch_add(Q.crpj, R, P->base_wanted, s);
        CK(cudaMemcpyAsync(rp_out, Q.crpj, sizeof(int64_t) * (R + 1), cudaMemcpyDeviceToHost, s));
    }
    CK(cudaStreamSynchronize(s));
    CK(cudaStreamSynchronize(z));
    CK(cudaStreamSynchronize(Q.h));
    unsigned err = 0;
    CK(cudaMemcpy(&err, &P->ctl[1].err, sizeof(unsigned), cudaMemcpyDeviceToHost));
    if (err) fail(SPGEMM_ERR_STATE, "internal: numeric pass produced a row whose nnz differs from the symbolic pass");
    P->num_groups = unit;
    return total;
}

}  // namespace

namespace spgh {
void do_panel_plan(const spgemm_csr *Ah, const spgemm_csr *Bh, size_t budget, const spgemm_opts *o, spgemm_plan_s *P) {
    panel_plan(Ah, Bh, budget, o, P);
}
int64_t run_panels(spgemm_plan_s *P, int64_t *rp_out, int32_t *col_out, double *val_out, int64_t capacity,
                   const Sink *sink, bool *overflow) {
    return panel_run(P, rp_out, col_out, val_out, capacity, sink, overflow);
}
}  // namespace spgh