// api.cu -- C ABI (include/spgemm.h), arena, planner and the chunk pipeline.
//
// Host side of the hot path (DESIGN.md §2 rows):
//   S0 residency   inputs adopted in place (device) or H2D-copied once into the arena (host);
//                  A == B is kept once (C = A x A, §V-B).
//   S1 panels      rows [row_begin, row_end) of A are this plan's row panel (§III-A, §III-D
//                  L169); B is used whole (one column panel: B fits every configured budget).
//   S9 arena       ONE device allocation (or caller workspace) sub-allocated by offsets; nothing
//                  is allocated between spgemm_plan returning and spgemm_free (§IV-B).
//   S10 planner    two-phase plans cut chunks from the exact symbolic nnz; fused plans cut them
//                  from the per-row bound min(products, ncols) (§IV-B: the flop bound is loose,
//                  so it sizes only chunk boundaries, never the output buffers).
//   S8 pipeline    compute stream + copy stream, R ring buffers, CUDA events.  In a fused plan the
//                  symbolic pass + scan of chunk j+1 run while chunk j is being copied out (the
//                  paper's Fig. 6 overlap, without its PCIe transfer splitting: the only
//                  small transfer is one 8-byte chunk total read through pinned memory).
#include <cuda_runtime.h>

#include <algorithm>
#include <condition_variable>
#include <thread>
#include <cstdio>
#include <cstdlib>
#include <cstddef>
#include <cstring>
#include <functional>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "../../include/spgemm.h"
#include "internal.h"

using namespace spg;

#include "host.h"

namespace spgh {
thread_local std::string g_err;
// ---------------------------------------------------------------- pinned host staging cache
struct PinnedBlock {
    void *p;
    size_t n;
    bool used;
};
std::mutex g_pin_mu;
std::vector<PinnedBlock> g_pins;

void *pin_acquire(size_t n) {
    std::lock_guard<std::mutex> lk(g_pin_mu);
    int best = -1;
    for (size_t i = 0; i < g_pins.size(); ++i)
        if (!g_pins[i].used && g_pins[i].n >= n && (best < 0 || g_pins[i].n < g_pins[best].n)) best = (int)i;
    if (best >= 0) {
        g_pins[best].used = true;
        return g_pins[best].p;
    }
    void *p = nullptr;
    if (cudaHostAlloc(&p, n ? n : 1, cudaHostAllocPortable) != cudaSuccess) {
        cudaGetLastError();
        fail(SPGEMM_ERR_HOST_ALLOC, "cudaHostAlloc of " + std::to_string(n) + " bytes failed");
    }
    g_pins.push_back({p, n ? n : 1, true});
    return p;
}

void pin_release(void *p) {
    if (!p) return;
    std::lock_guard<std::mutex> lk(g_pin_mu);
    for (auto &b : g_pins)
        if (b.p == p) b.used = false;
}

double elapsed(cudaEvent_t a, cudaEvent_t b) {
    float ms = 0;
    if (cudaEventElapsedTime(&ms, a, b) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    return ms;
}

std::mutex g_res_mu;
std::vector<Res *> g_res;

Res *res_acquire(int device) {
    std::lock_guard<std::mutex> lk(g_res_mu);
    for (auto r : g_res)
        if (!r->used && r->device == device) {
            r->used = true;
            return r;
        }
    Res *r = new Res();
    r->device = device;
    r->used = true;
    g_res.push_back(r);
    return r;
}

void res_release(Res *r) {
    if (!r) return;
    std::lock_guard<std::mutex> lk(g_res_mu);
    r->used = false;
}
}  // namespace spgh

void spgh::check_csr(const spgemm_csr *M, const char *name) {
    if (!M) fail(SPGEMM_ERR_INVALID_ARGUMENT, std::string(name) + " is NULL");
    if (M->nrows < 0 || M->ncols < 0 || M->nnz < 0)
        fail(SPGEMM_ERR_INVALID_ARGUMENT, std::string(name) + " has a negative dimension");
    if (!M->row_ptr) fail(SPGEMM_ERR_INVALID_ARGUMENT, std::string(name) + ".row_ptr is NULL");
    if (M->nnz > 0 && (!M->col_idx || !M->values))
        fail(SPGEMM_ERR_INVALID_ARGUMENT, std::string(name) + ".col_idx/values is NULL");
    if (M->where != SPGEMM_HOST && M->where != SPGEMM_DEVICE)
        fail(SPGEMM_ERR_INVALID_ARGUMENT, std::string(name) + ".where is invalid");
    if (M->where == SPGEMM_HOST) {
        if (M->row_ptr[0] != 0) fail(SPGEMM_ERR_INVALID_ARGUMENT, std::string(name) + ".row_ptr[0] != 0");
        if (M->row_ptr[M->nrows] != M->nnz)
            fail(SPGEMM_ERR_INVALID_ARGUMENT, std::string(name) + ".row_ptr[nrows] != nnz");
    }
}

// validate = 1, host operand: row_ptr non-decreasing (O(nrows) on the host, before any copy is
// sized from it); the columns are checked on the device by k_validate
void spgh::check_rows_host(const spgemm_csr *M, const char *name) {
    if (M->where != SPGEMM_HOST) return;
    for (int64_t r = 0; r < M->nrows; ++r)
        if (M->row_ptr[r + 1] < M->row_ptr[r])
            fail(SPGEMM_ERR_INVALID_ARGUMENT, std::string(name) + ".row_ptr decreases at row " + std::to_string(r));
}

namespace {

// chunk boundaries from a scanned prefix `pre` (pre[0] = 0, pre[R] = total): every chunk's span
// of `pre` is < capp + (largest single-row increment); empty ids are dropped.  The first chunks
// ramp up (1/4, 3/8, 1/2, 3/4 of capp, then capp) so that the first D2H starts
// early and each later chunk is computed while the previous one is being copied.
void cut_chunks(spgemm_plan_s *P, const int64_t *pre, int64_t total, int64_t capp, int64_t limit,
                std::vector<int64_t> *offs_out, std::vector<int64_t> *maxb_out = nullptr,
                std::vector<int64_t> *maxcol_out = nullptr) {
    // maxb_out / maxcol_out: per chunk, the largest row bound and the largest column its rows
    // read -- reduced on the device over the fine ids and returned in the same round trip
    const int64_t R = P->R;
    cudaStream_t s = P->stream;
    P->chunk_rows.clear();
    if (offs_out) offs_out->clear();
    if (maxb_out) maxb_out->clear();
    if (maxcol_out) maxcol_out->clear();
    if (total <= 0) return;
    constexpr int F = 8;
    const bool ramp = capp >= F && total / capp >= 4;
    if (ramp) capp /= F;
    const int64_t nids = total / capp + 1;
    const size_t save = P->used;  // temporary arrays at the start of the (not yet used) ring region
    int64_t *bounds = P->alloc<int64_t>(nids + 1, "chunk bounds");
    int64_t *offs = P->alloc<int64_t>(nids + 1, "chunk offsets");
    int64_t *fmax = maxb_out ? P->alloc<int64_t>(nids, "fine max bound") : nullptr;
    int64_t *fcol = maxcol_out ? P->alloc<int64_t>(nids, "fine max column") : nullptr;
    launch_cut(pre, R, capp, bounds, nids, s);
    launch_gather(pre, bounds, nids + 1, offs, s);
    if (fmax) launch_seg_max(P->bnd, bounds, nids, fmax, s);
    if (fcol) launch_seg_max_col(P->A, bounds, nids, fcol, s);
    CKL("cut");
    std::vector<int64_t> hb(nids + 1), ho(nids + 1), hm(fmax ? nids : 0), hc(fcol ? nids : 0);
    CK(cudaMemcpyAsync(hb.data(), bounds, sizeof(int64_t) * (nids + 1), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(ho.data(), offs, sizeof(int64_t) * (nids + 1), cudaMemcpyDeviceToHost, s));
    if (fmax) CK(cudaMemcpyAsync(hm.data(), fmax, sizeof(int64_t) * nids, cudaMemcpyDeviceToHost, s));
    if (fcol) CK(cudaMemcpyAsync(hc.data(), fcol, sizeof(int64_t) * nids, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    P->used = save;
    P->chunk_rows.push_back(hb[0]);
    if (offs_out) offs_out->push_back(ho[0]);
    int64_t last_off = ho[0];
    // ids (fine units when ramping) that close a chunk
    std::vector<int64_t> ends;
    {
        static const int units[] = {2, 3, 4, 6};
        int64_t id = 0;
        for (int k = 0; id < nids; ++k) {
            id += ramp ? (k < 4 ? units[k] : F) : 1;
            ends.push_back(std::min(id, nids));
        }
    }
    int64_t id0 = 0, mb = 0, mc = -1;  // fine ids not yet in an emitted chunk, and their maxima
    for (int64_t c : ends) {
        for (; id0 < c; ++id0) {
            if (fmax) mb = std::max(mb, hm[id0]);
            if (fcol) mc = std::max(mc, hc[id0]);
        }
        if (hb[c] == P->chunk_rows.back()) continue;
        if (ho[c] - last_off > limit) fail(SPGEMM_ERR_STATE, "internal: chunk exceeds the ring capacity");
        P->chunk_rows.push_back(hb[c]);
        if (offs_out) offs_out->push_back(ho[c]);
        if (maxb_out) maxb_out->push_back(mb);
        if (maxcol_out) maxcol_out->push_back(mc);
        mb = 0;
        mc = -1;
        last_off = ho[c];
    }
    if (P->chunk_rows.front() != 0 || P->chunk_rows.back() != R)
        fail(SPGEMM_ERR_STATE, "internal: chunk bounds do not cover the rows");
}

SymArgs sym_args(spgemm_plan_s *P, int64_t r0, int64_t r1, int tiers) {
    SymArgs sa{};
    sa.A = P->A;
    sa.B = P->B;
    sa.bnd = P->bnd;
    sa.nnz = P->nnzr;
    sa.r0 = r0;
    sa.r1 = r1;
    sa.listB = P->listB;
    sa.listM = P->listM;
    sa.listG = P->listG;
    sa.ctl = P->ctl;
    sa.gscratch = P->gbits_sym;
    sa.gcnt = P->gcnt;
    sa.gstride = P->gstride_bits;
    sa.gblocks = P->gblocks;
    sa.cursor = P->cur_sym;
    sa.curstride = P->curstride;
    sa.bblocks = P->bblocks_sym;
    sa.group = P->group;
    sa.tiers = tiers;
    return sa;
}

void do_plan(const spgemm_csr *Ah, const spgemm_csr *Bh, size_t budget, const spgemm_opts *o, spgemm_plan_s *P) {
    NvtxRange nv("spgemm_plan");
    check_csr(Ah, "A");
    check_csr(Bh, "B");
    if (Ah->ncols != Bh->nrows)
        fail(SPGEMM_ERR_SHAPE, "A.ncols (" + std::to_string(Ah->ncols) + ") != B.nrows (" + std::to_string(Bh->nrows) + ")");
    if (Bh->ncols > INT32_MAX) fail(SPGEMM_ERR_INDEX_OVERFLOW, "B.ncols exceeds INT32_MAX (col_idx is int32)");
    spgemm_opts opts;
    spgemm_opts_default(&opts);
    if (o) opts = *o;
    if (opts.validate) {
        check_rows_host(Ah, "A");
        check_rows_host(Bh, "B");
    }
    const int64_t rb = opts.row_begin, re = opts.row_end < 0 ? Ah->nrows : opts.row_end;
    if (rb < 0 || re < rb || re > Ah->nrows) fail(SPGEMM_ERR_SHAPE, "row range outside A");
    if (re - rb > INT32_MAX) fail(SPGEMM_ERR_INDEX_OVERFLOW, "more than INT32_MAX rows in one plan");
    if (opts.ring < 1 || opts.ring > 64) fail(SPGEMM_ERR_INVALID_ARGUMENT, "ring must be in [1, 64]");
    if (opts.order < 0 || opts.order > 1) fail(SPGEMM_ERR_INVALID_ARGUMENT, "order must be 0 or 1");
    if (opts.order && opts.fused)
        fail(SPGEMM_ERR_INVALID_ARGUMENT, "order = 1 needs a two-phase plan (a fused plan learns a chunk's host offset "
                                          "only after the chunks before it)");

    if (opts.device >= 0) {
        CK(cudaSetDevice(opts.device));
        P->device = opts.device;
    } else {
        CK(cudaGetDevice(&P->device));
    }
    CK(cudaDeviceGetAttribute(&P->num_sms, cudaDevAttrMultiProcessorCount, P->device));
    P->profile = opts.profile != 0;
    P->fused = opts.fused != 0;
    P->ring = opts.ring;
    P->row_begin = rb;
    P->R = re - rb;
    P->ncols = Bh->ncols;
    P->nnzB = Bh->nnz;
    P->base_wanted = opts.row_ptr_base;

    // streams and events: taken from the device's pool at plan time (nothing is created inside
    // execute; plans after the first reuse the previous plans' objects)
    P->res = res_acquire(P->device);
    Res *rs = P->res;
    P->stream = opts.stream ? (cudaStream_t)opts.stream : rs->stream(rs->own);
    P->copy = rs->stream(rs->copy);
    // plain-event layout in the pool: [0, ring) numeric done, [ring, 2 ring) copy done, 2 ring
    // ready, then per-chunk totals, then value pieces
    P->ev_num = rs->events(Res::PLAIN, 0, P->ring);
    P->ev_d2h = rs->events(Res::PLAIN, P->ring, P->ring);
    P->ev_ready = rs->events(Res::PLAIN, 2 * P->ring, 1)[0];
    const size_t ev_base = 2 * size_t(P->ring) + 1;
    cudaStream_t s = P->stream;

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

    EvSet pe(P->profile, rs, 0, 12);
    pe.rec(0, s);

    // S0 residency: B.  Host operands: row_ptr and col_idx now (the count and symbolic passes need
    // only the structure); the values follow in row pieces on the H2D stream, overlapping the
    // planning and the first chunks (the numeric pass of a chunk waits for the pieces it reads).
    std::vector<std::pair<size_t, size_t>> bval_pieces;  // (element offset, count)
    double *bval_dev = nullptr;
    // C = A x A with host operands (A aliases B): the structure goes up in the same row pieces as
    // the values, on the H2D stream, and the count pass of each piece's rows runs as soon as the
    // piece has landed (it needs B.row_ptr, uploaded first, and the piece's columns), overlapping
    // the rest of the upload
    const bool host_alias = Bh->where == SPGEMM_HOST && Ah->where == SPGEMM_HOST && Ah->row_ptr == Bh->row_ptr &&
                            Ah->col_idx == Bh->col_idx && Ah->values == Bh->values && Ah->nrows == Bh->nrows &&
                            Ah->ncols == Bh->ncols;
    const bool pieced_count = host_alias && !opts.validate && Bh->nnz > 0;
    // Host cut: with short rows the plan needs no count pass at all.  Every row bound
    // min(products, ncols) is at most ub = min(ncols, maxlen^2) (maxlen = longest row of B = A),
    // so when ub <= CAPB_NUM (no long-row scratch) chunks are cut on the host from A.row_ptr by
    // nnz(A) x maxlen, and each chunk's count pass runs in execute, right before its symbolic pass,
    // once the pieces it reads have landed -- the first chunk starts ~1 ms into the upload instead
    // of after the whole structure.  SPGEMM_NO_HOST_CUT=1 disables it (ablation).
    int64_t hc_maxlen = -1;
    if (pieced_count && P->fused) {
        const char *no = getenv("SPGEMM_NO_HOST_CUT");
        if (!(no && no[0] == '1')) {
            const int64_t lim = Bh->ncols <= CAPB_NUM ? INT64_MAX : 64;  // maxlen^2 <= CAPB_NUM
            // longest row: one pass over row_ptr, split over host threads (C2: 2 M rows, ~1.7 ms
            // on one core, on the critical path of the step), each stopping once past `lim`
            const int64_t *brp = Bh->row_ptr;
            const int64_t n = Bh->nrows;
            const int nt = n < (1 << 18) ? 1 : int(std::min<unsigned>(8, std::max(1u, std::thread::hardware_concurrency())));
            std::vector<int64_t> part(nt, 0);
            auto scan = [&](int t) {
                const int64_t a = n * t / nt, b = n * (t + 1) / nt;
                int64_t ml = 0;
                for (int64_t r = a; r < b && ml <= lim; r += 4096) {
                    const int64_t e = std::min<int64_t>(r + 4096, b);
                    int64_t m = 0;
                    for (int64_t q = r; q < e; ++q) m = std::max<int64_t>(m, brp[q + 1] - brp[q]);
                    ml = std::max(ml, m);
                }
                part[t] = ml;
            };
            std::vector<std::thread> th;
            for (int t = 1; t < nt; ++t) th.emplace_back(scan, t);
            scan(0);
            for (auto &x : th) x.join();
            const int64_t ml = *std::max_element(part.begin(), part.end());
            // (ml * ml only when ml <= 2^31: a longer row means invalid input or ncols <= CAPB_NUM)
            const int64_t ub = ml > (int64_t(1) << 31) ? Bh->ncols : std::min<int64_t>(Bh->ncols, ml * ml);
            if (ml <= lim && ub <= CAPB_NUM) hc_maxlen = ml;
        }
    }
    P->host_cut = hc_maxlen >= 0;
    std::vector<cudaEvent_t> ev_col;
    if (Bh->where == SPGEMM_DEVICE) {
        P->B = DevCSR{Bh->row_ptr, Bh->col_idx, Bh->values, Bh->nrows, Bh->ncols};
    } else {
        int64_t *rp = P->alloc<int64_t>(Bh->nrows + 1, "B.row_ptr");
        int32_t *c = P->alloc<int32_t>(Bh->nnz, "B.col_idx");
        double *v = P->alloc<double>(Bh->nnz, "B.values");
        if (!P->host_cut)
            CK(cudaMemcpyAsync(rp, Bh->row_ptr, sizeof(int64_t) * (Bh->nrows + 1), cudaMemcpyHostToDevice, s));
        if (Bh->nnz && !pieced_count)
            CK(cudaMemcpyAsync(c, Bh->col_idx, sizeof(int32_t) * Bh->nnz, cudaMemcpyHostToDevice, s));
        // pieces of ~32 MB of values, cut at row boundaries; the first ones smaller (1/8, 1/4,
        // 1/2) so that the first chunk's rows land early
        int64_t target = std::max<int64_t>(1, (32ll << 20) / 8);
        if (const char *pn = getenv("SPGEMM_PIECE_NNZ")) target = std::max<int64_t>(1, atoll(pn));  // test hook
        P->bpiece_rows.push_back(0);
        int64_t r = 0;
        while (r < Bh->nrows) {
            const size_t k = bval_pieces.size();
            const int64_t want = Bh->row_ptr[r] + (k < 3 ? std::max<int64_t>(1, target >> (3 - k)) : target);
            int64_t e = std::upper_bound(Bh->row_ptr + r + 1, Bh->row_ptr + Bh->nrows + 1, want) - Bh->row_ptr - 1;
            e = std::max<int64_t>(e, r + 1);
            bval_pieces.push_back({size_t(Bh->row_ptr[r]), size_t(Bh->row_ptr[e] - Bh->row_ptr[r])});
            P->bpiece_rows.push_back(e);
            r = e;
        }
        bval_dev = v;
        P->B = DevCSR{rp, c, v, Bh->nrows, Bh->ncols};
        if (P->host_cut) {
            // piece k = row_ptr (b_k, b_k+1] (+ entry 0 with the first) , col_idx, values of its
            // rows, in that order on the H2D stream; ev_col[k] / ev_piece[k] after its structure /
            // values.  A chunk waits for the piece holding the largest row it reads (its own last
            // row, or the largest column of its rows), which covers every earlier piece.
            const size_t np = bval_pieces.size();
            P->hstream = rs->stream(rs->hstream);
            P->ev_col = rs->events(Res::PIECE, np, np);
            P->ev_piece = rs->events(Res::PIECE, 0, np);
            cudaEvent_t alloc_ready = rs->events(Res::PIECE, 2 * np, 1)[0];
            CK(cudaEventRecord(alloc_ready, s));  // allocation order: after everything queued so far
            CK(cudaStreamWaitEvent(P->hstream, alloc_ready, 0));
            for (size_t k = 0; k < np; ++k) {
                const int64_t b0 = P->bpiece_rows[k], b1 = P->bpiece_rows[k + 1];
                const int64_t q0 = k == 0 ? 0 : b0 + 1;
                CK(cudaMemcpyAsync(rp + q0, Bh->row_ptr + q0, sizeof(int64_t) * (b1 + 1 - q0), cudaMemcpyHostToDevice,
                                   P->hstream));
                const auto &pc = bval_pieces[k];
                if (pc.second)
                    CK(cudaMemcpyAsync(c + pc.first, Bh->col_idx + pc.first, sizeof(int32_t) * pc.second,
                                       cudaMemcpyHostToDevice, P->hstream));
                CK(cudaEventRecord(P->ev_col[k], P->hstream));
                if (pc.second)
                    CK(cudaMemcpyAsync(v + pc.first, Bh->values + pc.first, sizeof(double) * pc.second,
                                       cudaMemcpyHostToDevice, P->hstream));
                CK(cudaEventRecord(P->ev_piece[k], P->hstream));
            }
            bval_pieces.clear();  // queued
        } else if (pieced_count) {
            const size_t np = bval_pieces.size();
            P->hstream = rs->stream(rs->hstream);
            ev_col = rs->events(Res::PIECE, np, np);
            cudaEvent_t rp_ready = rs->events(Res::PIECE, 2 * np, 1)[0];
            CK(cudaEventRecord(rp_ready, s));  // allocation order + B.row_ptr queued first
            CK(cudaStreamWaitEvent(P->hstream, rp_ready, 0));
            for (size_t k = 0; k < np; ++k) {
                const auto &pc = bval_pieces[k];
                if (pc.second)
                    CK(cudaMemcpyAsync(c + pc.first, Bh->col_idx + pc.first, sizeof(int32_t) * pc.second,
                                       cudaMemcpyHostToDevice, P->hstream));
                CK(cudaEventRecord(ev_col[k], P->hstream));
            }
        }
    }
    // S0 residency + S1 row panel: A
    if (Ah->where == SPGEMM_DEVICE) {
        P->A = DevCSR{Ah->row_ptr + rb, Ah->col_idx, Ah->values, P->R, Ah->ncols};
        P->nnzA = -1;  // unknown without a read; statistics only
    } else {
        const bool alias = Bh->where == SPGEMM_HOST && Ah->row_ptr == Bh->row_ptr && Ah->col_idx == Bh->col_idx &&
                           Ah->values == Bh->values && Ah->nrows == Bh->nrows && Ah->ncols == Bh->ncols;
        const int64_t p0 = Ah->row_ptr[rb], p1 = Ah->row_ptr[re];
        P->nnzA = p1 - p0;
        if (alias) {
            P->A = DevCSR{P->B.rp + rb, P->B.col, P->B.val, P->R, Ah->ncols};
            P->a_alias = true;
            if (P->host_cut) {
                P->hA_rp = Ah->row_ptr + rb;
                P->hA_col = Ah->col_idx;
            }
        } else {
            int64_t *rp = P->alloc<int64_t>(P->R + 1, "A.row_ptr");
            int32_t *c = P->alloc<int32_t>(p1 - p0, "A.col_idx");
            double *v = P->alloc<double>(p1 - p0, "A.values");
            CK(cudaMemcpyAsync(rp, Ah->row_ptr + rb, sizeof(int64_t) * (P->R + 1), cudaMemcpyHostToDevice, s));
            if (p1 > p0) {
                CK(cudaMemcpyAsync(c, Ah->col_idx + p0, sizeof(int32_t) * (p1 - p0), cudaMemcpyHostToDevice, s));
                CK(cudaMemcpyAsync(v, Ah->values + p0, sizeof(double) * (p1 - p0), cudaMemcpyHostToDevice, s));
            }
            launch_rebase(rp, P->R + 1, p0, s);
            CKL("rebase");
            P->A = DevCSR{rp, c, v, P->R, Ah->ncols};
        }
    }
    // start the B value pieces (host operands) on their own stream, one event per piece
    if (!bval_pieces.empty()) {
        P->hstream = rs->stream(rs->hstream);
        CK(cudaEventRecord(P->ev_ready, s));  // allocation order: after everything queued so far
        CK(cudaStreamWaitEvent(P->hstream, P->ev_ready, 0));
        P->ev_piece = rs->events(Res::PIECE, 0, bval_pieces.size());
        for (size_t k = 0; k < bval_pieces.size(); ++k) {
            const auto &pc = bval_pieces[k];
            if (pc.second)
                CK(cudaMemcpyAsync(bval_dev + pc.first, Bh->values + pc.first, sizeof(double) * pc.second,
                                   cudaMemcpyHostToDevice, P->hstream));
            CK(cudaEventRecord(P->ev_piece[k], P->hstream));
        }
    }
    P->group = choose_group(P->B, P->nnzB);

    // per-row arrays (28 B/row) and control blocks
    const int64_t R = P->R;
    P->bnd = P->alloc<int64_t>(R, "row bounds");
    P->crp = P->alloc<int64_t>(R + 1, "C.row_ptr");
    P->nnzr = P->alloc<int32_t>(R, "row nnz");
    P->listB = P->alloc<int32_t>(R, "listB");
    P->listG = P->alloc<int32_t>(R, "listG");
    P->listBn = P->alloc<int32_t>(R, "numeric listB");
    P->listM = P->alloc<int32_t>(R, "listM");
    P->listMn = P->alloc<int32_t>(R, "numeric listM");
    P->listGn = P->alloc<int32_t>(R, "numeric listG");
    P->ctl = P->alloc<Ctl>(2, "ctl");
    P->tmp = P->alloc<int64_t>((R + SCAN_TILE - 1) / SCAN_TILE + 64, "scan scratch");
    CK(cudaMemsetAsync(P->ctl, 0, 2 * sizeof(Ctl), s));
    CK(cudaMemsetAsync(P->crp, 0, sizeof(int64_t), s));

    if (opts.validate) {
        // every offset checked against the caller's whole array (device: its own first entry;
        // host: the arena copy), and the result read back BEFORE any kernel indexes the operands
        // with these offsets or columns
        const int64_t *a0 = Ah->where == SPGEMM_DEVICE ? Ah->row_ptr : P->a_alias ? P->B.rp : P->A.rp;
        const int64_t an = Ah->where == SPGEMM_DEVICE ? Ah->nnz : P->a_alias ? Bh->nnz : P->nnzA;
        launch_validate(P->A, a0, an, P->ctl, s);
        launch_validate(P->B, Bh->where == SPGEMM_DEVICE ? Bh->row_ptr : P->B.rp, Bh->nnz, P->ctl, s);
        CKL("validate");
        unsigned verr = 0;
        CK(cudaMemcpyAsync(&verr, &P->ctl[0].err, sizeof(unsigned), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (verr & 2u)
            fail(SPGEMM_ERR_INVALID_ARGUMENT, "input validation failed (unsorted/duplicate/out-of-range col_idx or bad row_ptr)");
    }

    // S2 count (host cut: per chunk, inside execute)
    pe.rec(1, s);
    if (P->host_cut) {
        P->products = -1;  // known after the first execution
        P->max_u = -1;
        P->max_bound = hc_maxlen > (int64_t(1) << 31) ? P->ncols
                                                      : std::min<int64_t>(P->ncols, hc_maxlen * hc_maxlen);  // upper bound
        P->max_deg = hc_maxlen;
    } else if (pieced_count) {
        for (size_t k = 0; k + 1 < P->bpiece_rows.size(); ++k) {
            const int64_t g0 = std::max<int64_t>(P->bpiece_rows[k], rb), g1 = std::min<int64_t>(P->bpiece_rows[k + 1], re);
            CK(cudaStreamWaitEvent(s, ev_col[k], 0));
            if (g1 <= g0) continue;
            DevCSR Ak = P->A;
            Ak.rp = P->A.rp + (g0 - rb);
            Ak.nrows = g1 - g0;
            launch_count(Ak, P->B, P->bnd + (g0 - rb), P->ctl, s);
        }
    } else {
        launch_count(P->A, P->B, P->bnd, P->ctl, s);
    }
    CKL("count");
    pe.rec(2, s);
    // fused plans: the prefix of the row bounds (chunk boundaries) is scanned before the first
    // host round trip, which then reads both the count totals and the prefix total
    int64_t total_b = 0;
    if (P->fused && !P->host_cut) {
        launch_scan64(P->bnd, P->R, P->crp, P->tmp, s);
        CKL("bound scan");
        CK(cudaMemcpyAsync(&total_b, P->crp + P->R, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    }
    Ctl hc;
    if (!P->host_cut) {
        CK(cudaMemcpyAsync(&hc, P->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (hc.err & 2u)
            fail(SPGEMM_ERR_INVALID_ARGUMENT, "input validation failed (unsorted/duplicate/out-of-range col_idx or bad row_ptr)");
        P->products = (int64_t)hc.sum_u;
        P->max_u = (int64_t)hc.max_u;
        P->max_bound = (int64_t)hc.max_bound;
        P->max_deg = (int64_t)hc.max_deg;
    }

    // arena-resident accumulator scratch, sized only if a row can exceed one CTA-tier piece:
    //   cursors of the pieced CTA tier (per CTA: 2 x curstride int32 for each pass -- separate,
    //   so both passes may run concurrently on two streams) and
    //   G (dense, per CTA: a bitmap for each pass + fp64 [ncols] for the numeric pass).
    //   The dense scratch takes at most 1/4 of what is left after the smallest ring.
    if (P->max_bound > CAPB_NUM) {
        const Grids &gr = grids(P->device, P->num_sms);
        P->curstride = (std::min<int64_t>(std::max<int64_t>(P->max_deg, 1), CURSOR_MAX) + 31) & ~int64_t(31);
        P->bblocks_sym = gr.symb_blocks;
        P->bblocks_num = gr.numb_blocks;
        P->cur_sym = P->alloc<int32_t>(int64_t(P->bblocks_sym) * 2 * P->curstride, "CTA-tier cursors (symbolic)");
        P->cur_num = P->alloc<int32_t>(int64_t(P->bblocks_num) * 2 * P->curstride, "CTA-tier cursors (numeric)");
        const int64_t nwords = (P->ncols + 31) / 32;
        const size_t ring_min = size_t(P->ring) * size_t(P->max_bound) * 12 + 4096;
        const size_t freeb = P->arena_bytes > P->used ? P->arena_bytes - P->used : 0;
        const size_t avail = freeb > ring_min ? (freeb - ring_min) / 4 : 0;
        P->gstride_bits = (nwords + 63) & ~int64_t(63);
        P->gstride_vals = (P->ncols + 31) & ~int64_t(31);
        const size_t gper = size_t(P->gstride_bits) * 8 + size_t(P->gstride_vals) * 8;
        // up to 4 dense-tier CTAs per SM (the kernels are latency-bound on their L2 atomics and
        // fit 4 x 512 threads per SM; C3's 9 K hub rows: 1 CTA per SM left 3/4 of the warps idle)
        const int64_t gwant = (P->max_bound > CAPS_NUM || P->max_deg > CURSOR_MAX) ? 4 * int64_t(P->num_sms) : 8;
        int64_t ng = std::min<int64_t>(gwant, int64_t(avail / gper));
        if (const char *mg = getenv("SPGEMM_MAX_GSLOTS"))  // test hook: few slots, so that dense rows
            ng = std::min<int64_t>(ng, std::max(1, atoi(mg)));  // overflow to the one-CTA kernels
        if (ng < 1) {
            const size_t fb = P->arena_bytes > P->used + ring_min ? P->arena_bytes - P->used - ring_min : 0;
            ng = fb >= gper ? 1 : 0;
        }
        if (ng < 1) fail(SPGEMM_ERR_BUDGET, "budget cannot hold one dense accumulator for the longest row");
        P->gblocks = (int)ng;
        P->gbits = P->alloc<uint32_t>(P->gstride_bits * ng, "dense-tier bitmap (numeric)");
        P->gbits_sym = P->alloc<uint32_t>(P->gstride_bits * ng, "dense-tier bitmap (symbolic)");
        P->gvals = P->alloc<double>(P->gstride_vals * ng, "dense-tier values");
        // split dense rows: per slot a fresh-column counter (symbolic) / KG_SWEEP range counts (numeric)
        P->gcnt = P->alloc<unsigned long long>(2 * ng * (KG_SWEEP + 1), "dense-tier counters");
        CK(cudaMemsetAsync(P->gcnt, 0, sizeof(unsigned long long) * 2 * ng * (KG_SWEEP + 1), s));
        CK(cudaMemsetAsync(P->gbits, 0, size_t(P->gstride_bits) * ng * 4, s));
        CK(cudaMemsetAsync(P->gbits_sym, 0, size_t(P->gstride_bits) * ng * 4, s));
        CK(cudaMemsetAsync(P->gvals, 0, size_t(P->gstride_vals) * ng * 8, s));
    }

    // ring capacity from what is left: each slot holds `cap` nonzeros (val fp64 + col int32)
    auto ring_cap = [&](int64_t need_row) {
        const size_t freeb = P->arena_bytes > P->used + 4096 ? P->arena_bytes - P->used - 4096 : 0;
        const size_t slot = (freeb / P->ring) & ~size_t(255);
        // RING_PAD elements per slot stay free for the alignment pad of run_pipeline's groups
        int64_t cap = (int64_t(slot / 12) & ~int64_t(63)) - 2 * RING_PAD;
        if (opts.chunk_nnz > 0) cap = std::min<int64_t>(cap, std::max<int64_t>(opts.chunk_nnz, need_row));
        if (cap < std::max<int64_t>(need_row, 1))
            fail(SPGEMM_ERR_BUDGET, "ring buffer of " + std::to_string(cap) +
                                        " nonzeros cannot hold the longest C row (bound " + std::to_string(need_row) + ")");
        return cap;
    };

    std::vector<int64_t> chunk_maxcol;  // host operands: largest column each chunk reads
    if (!P->fused) {
        // S3+S4 symbolic and S5 scan over all rows, then cut by exact nnz
        SymArgs sa = sym_args(P, 0, R, sym_tiers(P->max_bound));
        pe.rec(3, s);
        launch_symbolic(sa, P->num_sms, s, pe.at(4));
        CKL("symbolic");
        launch_scan(P->nnzr, R, P->crp, P->tmp, s);
        CKL("scan");
        pe.rec(9, s);
        int64_t total = 0;
        CK(cudaMemcpyAsync(&hc, P->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(&total, P->crp + R, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        P->nnz = total;
        P->max_nnz = (int64_t)hc.max_nnz;
        P->rows_w = (int64_t)hc.rows_w;
        P->rows_b = (int64_t)hc.rows_b;
        P->rows_g = (int64_t)hc.rows_g;
        P->rows_m = (int64_t)hc.rows_m;
        int64_t cap = ring_cap(P->max_nnz);
        cap = std::max<int64_t>(std::min<int64_t>(cap, std::max<int64_t>(total, 1)), std::max<int64_t>(P->max_nnz, 1));
        P->cap = cap;
        int64_t capp = std::max<int64_t>(1, cap - P->max_nnz);
        int64_t minc = opts.min_chunks;
        if (minc <= 0) minc = std::min<int64_t>(64, std::max<int64_t>(1, total * 12 / (128ll << 20)));
        if (minc > 1) capp = std::min<int64_t>(capp, std::max<int64_t>(1, (total + minc - 1) / minc));
        if (opts.chunk_nnz > 0) capp = std::min<int64_t>(capp, std::max<int64_t>(1, opts.chunk_nnz - P->max_nnz));
        cut_chunks(P, P->crp, total, std::max<int64_t>(capp, 1), cap, &P->chunk_offs);
        // §IV-C: process the chunks in decreasing order of their flops, so that a
        // chunk's computation tends to hide under the transfer of the (larger) one before it
        const int64_t nch = P->num_chunks();
        if (opts.order == 1 && nch > 1) {
            const size_t save = P->used;
            int64_t *drows = P->alloc<int64_t>(nch + 1, "chunk rows");
            int64_t *dfl = P->alloc<int64_t>(nch, "chunk flops");
            std::vector<int64_t> fl(nch);
            CK(cudaMemcpyAsync(drows, P->chunk_rows.data(), sizeof(int64_t) * (nch + 1), cudaMemcpyHostToDevice, s));
            launch_seg_sum(P->bnd, drows, nch, dfl, s);  // bound = min(products, ncols) per row
            CKL("chunk flops");
            CK(cudaMemcpyAsync(fl.data(), dfl, sizeof(int64_t) * nch, cudaMemcpyDeviceToHost, s));
            CK(cudaStreamSynchronize(s));
            P->used = save;
            P->unit_order.resize(nch);
            for (int64_t j = 0; j < nch; ++j) P->unit_order[j] = j;
            std::stable_sort(P->unit_order.begin(), P->unit_order.end(),
                             [&](int64_t a, int64_t b) { return fl[a] > fl[b]; });
        }
    } else if (P->host_cut) {
        // host cut: a chunk of rows [r0, r1) has sum of row bounds <= (A.row_ptr[r1] - A.row_ptr[r0]) x
        // maxlen, so chunks are cut by nnz(A) with that product <= capp (one row alone if longer); the
        // products are estimated as nnz(A) x mean row length of B for the chunk count only
        const int64_t ml = std::max<int64_t>(hc_maxlen, 1);
        const int64_t *hrp = P->hA_rp;
        const int64_t nnzA = hrp[R] - hrp[0];
        const int64_t est = Bh->nrows ? int64_t(double(nnzA) * (double(Bh->nnz) / double(Bh->nrows))) : 0;
        P->sum_bound = -1;
        int64_t cap = ring_cap(P->max_bound);
        cap = std::max<int64_t>(std::min<int64_t>(cap, std::max<int64_t>(nnzA * ml, 1)), std::max<int64_t>(P->max_bound, 1));
        P->cap = cap;
        int64_t capp = std::max<int64_t>(1, cap - P->max_bound);
        int64_t minc = opts.min_chunks;
        if (minc <= 0) minc = std::min<int64_t>(64, std::max<int64_t>(1, est * 12 / (512ll << 20)));
        if (minc > 1) capp = std::min<int64_t>(capp, std::max<int64_t>(1, (est + minc - 1) / minc));
        if (opts.chunk_nnz > 0) capp = std::min<int64_t>(capp, std::max<int64_t>(1, opts.chunk_nnz - P->max_bound));
        // ramp as in cut_chunks: 2/8, 3/8, 4/8, 6/8 of capp, then capp
        const bool ramp = capp >= 8 && est / capp >= 4;
        P->chunk_rows.assign(1, 0);
        int64_t r = 0;
        for (int k = 0; r < R; ++k) {
            static const int units[] = {2, 3, 4, 6};
            const int64_t sz = ramp && k < 4 ? std::max<int64_t>(1, capp / 8 * units[k]) : capp;
            const int64_t want = hrp[r] + std::max<int64_t>(sz / ml, 1);
            int64_t e = std::upper_bound(hrp + r + 1, hrp + R + 1, want) - hrp - 1;
            e = std::max<int64_t>(e, r + 1);
            P->chunk_rows.push_back(e);
            r = e;
        }
        if (nnzA == 0) P->chunk_rows.clear();  // every row is empty: no chunk (as cut_chunks)
        P->chunk_maxb.assign(P->num_chunks(), P->max_bound);
        const int64_t nch = P->num_chunks();
        P->ev_tot = rs->events(Res::PLAIN, ev_base, nch);
        P->astream = rs->stream(rs->astream);
    } else {
        // fused: boundaries from the prefix of the row bounds; the symbolic pass runs per chunk
        // inside execute.  crp temporarily holds that prefix.
        P->sum_bound = total_b;
        int64_t cap = ring_cap(P->max_bound);
        cap = std::max<int64_t>(std::min<int64_t>(cap, std::max<int64_t>(total_b, 1)), std::max<int64_t>(P->max_bound, 1));
        P->cap = cap;
        int64_t capp = std::max<int64_t>(1, cap - P->max_bound);
        int64_t minc = opts.min_chunks;
        if (minc <= 0) minc = std::min<int64_t>(64, std::max<int64_t>(1, total_b * 12 / (512ll << 20)));
        if (minc > 1) capp = std::min<int64_t>(capp, std::max<int64_t>(1, (total_b + minc - 1) / minc));
        if (opts.chunk_nnz > 0) capp = std::min<int64_t>(capp, std::max<int64_t>(1, opts.chunk_nnz - P->max_bound));
        // with the cut: per chunk the max row bound (which symbolic tiers a chunk needs) and, for
        // host operands, the largest column it reads (which value pieces its numeric pass waits for)
        // -- one round trip, no H2D (a small H2D would queue behind the value pieces on the copy engine)
        cut_chunks(P, P->crp, total_b, std::max<int64_t>(capp, 1), cap, nullptr, &P->chunk_maxb,
                   P->ev_piece.empty() ? nullptr : &chunk_maxcol);
        CK(cudaMemsetAsync(P->crp, 0, sizeof(int64_t), s));
        const int64_t nch = P->num_chunks();
        P->ev_tot = rs->events(Res::PLAIN, ev_base, nch);
        // The symbolic passes run on the compute stream, two units ahead of the numeric passes
        // (run_pipeline), so the GPU never waits for the host between units.  With
        // SPGEMM_CONCURRENT_ANALYSIS=1 they get their own stream and overlap the numeric passes
        // instead: no faster on the configured workloads (the step is host-link-bound: C3 5.72 s
        // both ways, C2 55.5 / 55.7 ms), and the kernels' event times then include each other's
        // contention, which makes per-kernel rates meaningless (profiles/r02/serial_analysis.md).
        const char *conc = getenv("SPGEMM_CONCURRENT_ANALYSIS");
        P->astream = (conc && conc[0] == '1') ? rs->stream(rs->astream) : P->stream;
    }
    // host operands: the last value piece each chunk's numeric pass reads (largest B row touched;
    // with A aliasing B also the chunk's own rows)
    {
        const int64_t nch = P->num_chunks();
        P->chunk_wait.assign(nch, -1);  // host cut: set per chunk in execute (enqueue_analysis)
        if (!P->ev_piece.empty() && nch > 0 && !P->host_cut) {
            std::vector<int64_t> &hmax = chunk_maxcol;
            if ((int64_t)hmax.size() != nch) {  // two-phase plans: one more round trip
                hmax.resize(nch);
                const size_t save = P->used;
                int64_t *drows = P->alloc<int64_t>(nch + 1, "chunk rows");
                int64_t *dmax = P->alloc<int64_t>(nch, "chunk max column");
                CK(cudaMemcpyAsync(drows, P->chunk_rows.data(), sizeof(int64_t) * (nch + 1), cudaMemcpyHostToDevice, s));
                launch_seg_max_col(P->A, drows, nch, dmax, s);
                CKL("chunk max column");
                CK(cudaMemcpyAsync(hmax.data(), dmax, sizeof(int64_t) * nch, cudaMemcpyDeviceToHost, s));
                CK(cudaStreamSynchronize(s));
                P->used = save;
            }
            for (int64_t j = 0; j < nch; ++j) {
                int64_t need = hmax[j];
                if (P->a_alias) need = std::max<int64_t>(need, rb + P->chunk_rows[j + 1] - 1);
                if (need < 0) continue;
                const auto it = std::upper_bound(P->bpiece_rows.begin(), P->bpiece_rows.end(), need);
                P->chunk_wait[j] = int(it - P->bpiece_rows.begin()) - 1;
            }
        }
    }
    P->h_small = (int64_t *)pin_acquire(sizeof(int64_t) * (2 * P->num_chunks() + 2));
    CK(cudaHostGetDevicePointer((void **)&P->d_small, P->h_small, 0));

    // ring buffers
    P->ring_col.assign(P->ring, nullptr);
    P->ring_val.assign(P->ring, nullptr);
    if (P->num_chunks() > 0) {
        for (int r = 0; r < P->ring; ++r) {
            P->ring_val[r] = P->alloc<double>(P->cap + RING_PAD, "ring values");
            P->ring_col[r] = P->alloc<int32_t>(P->cap + RING_PAD, "ring col_idx");
        }
        P->ring_bytes = size_t(P->ring) * size_t(P->cap) * 12;
    }
    pe.rec(10, s);
    CK(cudaStreamSynchronize(s));
    if (P->profile) {
        P->stats.clear();
        P->add_stat("plan_device_span", elapsed(pe.ev[0], pe.ev[10]), 0);
        P->add_stat("plan_upload", elapsed(pe.ev[0], pe.ev[1]), 0);  // operand H2D (host operands) + setup
        P->add_stat("count", elapsed(pe.ev[1], pe.ev[2]), 0);
        P->add_stat("plan_cut", elapsed(pe.ev[2], pe.ev[10]), 0);    // scans, cuts, round trips, ring
        if (!P->fused) {
            P->add_stat("sym_w", elapsed(pe.ev[4], pe.ev[5]), 0);
            P->add_stat("sym_m", elapsed(pe.ev[5], pe.ev[6]), 0);
            P->add_stat("sym_b", elapsed(pe.ev[6], pe.ev[7]), 0);
            P->add_stat("sym_g", elapsed(pe.ev[7], pe.ev[8]), 0);
            P->add_stat("scan", elapsed(pe.ev[8], pe.ev[9]), 0);
        }
    }
}

void enqueue_numeric(spgemm_plan_s *P, int64_t c, int b, int64_t slot_off, int64_t max_row_nnz, cudaEvent_t *ev) {
    NvtxRange nv("enqueue numeric");
    NumArgs na{};
    na.A = P->A;
    na.B = P->B;
    na.crp = P->crp;
    na.r0 = P->chunk_rows[c];
    na.r1 = P->chunk_rows[c + 1];
    na.out_col = P->ring_col[b] + slot_off;
    na.out_val = P->ring_val[b] + slot_off;
    na.listB = P->listBn;
    na.listM = P->listMn;
    na.listG = P->listGn;
    na.ctl = P->ctl + 1;
    na.gbits = P->gbits;
    na.gvals = P->gvals;
    na.gcnt = P->gcnt ? P->gcnt + size_t(P->gblocks) * (KG_SWEEP + 1) : nullptr;
    na.gstride_bits = P->gstride_bits;
    na.gstride_vals = P->gstride_vals;
    na.gblocks = P->gblocks;
    na.cursor = P->cur_num;
    na.curstride = P->curstride;
    na.bblocks = P->bblocks_num;
    na.group = P->group;
    na.tiers = num_tiers(max_row_nnz);
    if (P->profile && c < int64_t(P->tiers_num.size())) P->tiers_num[c] = na.tiers;
    launch_numeric(na, P->num_sms, P->stream, ev);
    CKL("numeric");
}

// fused plans: symbolic + scan of chunk j; its end offset and max row nnz land in
// h_small[1 + 2j], h_small[2 + 2j] through zero-copy stores (no D2H on the copy engine)
void enqueue_analysis(spgemm_plan_s *P, int64_t j, cudaEvent_t *ev) {
    NvtxRange nv("enqueue symbolic + scan");
    const int64_t r0 = P->chunk_rows[j], r1 = P->chunk_rows[j + 1];
    cudaStream_t as = P->astream;
    if (P->host_cut) {
        // the piece holding the largest row chunk j reads: its own last row or the largest column
        // of its rows (each row's last entry, rows sorted); the count and symbolic passes wait for
        // its structure, the numeric pass (chunk_wait) for its values
        int64_t need = P->row_begin + r1 - 1;
        const int64_t *hrp = P->hA_rp;
        for (int64_t r = r0; r < r1; ++r)
            if (hrp[r + 1] > hrp[r]) need = std::max<int64_t>(need, P->hA_col[hrp[r + 1] - 1]);
        const auto it = std::upper_bound(P->bpiece_rows.begin(), P->bpiece_rows.end(), need);
        const int w = int(it - P->bpiece_rows.begin()) - 1;
        P->chunk_wait[j] = w;
        CK(cudaStreamWaitEvent(as, P->ev_col[w], 0));
        DevCSR Ak = P->A;
        Ak.rp = P->A.rp + r0;
        Ak.nrows = r1 - r0;
        launch_count(Ak, P->B, P->bnd + r0, P->ctl, as);
        CKL("count");
    }
    SymArgs sa = sym_args(P, r0, r1, sym_tiers(P->chunk_maxb[j]));
    if (P->profile && j < int64_t(P->tiers_sym.size())) P->tiers_sym[j] = sa.tiers;
    launch_symbolic(sa, P->num_sms, as, ev);
    CKL("symbolic");
    launch_scan(P->nnzr + r0, r1 - r0, P->crp + r0, P->tmp, as);
    CKL("scan");
    if (ev) CK(cudaEventRecord(ev[5], as));
    launch_publish(P->crp + r1, P->ctl, P->d_small + 1 + 2 * j, as);
    CKL("publish");
    CK(cudaEventRecord(P->ev_tot[j], as));
}

// Per-kernel statistics and the timeline of the last execution, from its timing events.  Done
// on demand (spgemm_stats / spgemm_timeline, or before the next execution reuses the events):
// ~500 cudaEventElapsedTime calls cost ~2 ms of host time, which must not sit inside a timed step.
void finalize_profile(spgemm_plan_s *P) {
    if (!P->pend.active) return;
    P->pend.active = false;
    std::vector<cudaEvent_t> &ev = P->pend.ev;
    auto ev_at = [&](size_t k) { return ev.data() + k; };
    const int64_t nch = P->pend.nch;
    const size_t per = P->pend.per;
    const bool overflow = P->pend.overflow;
    const int64_t total = P->pend.total;
    P->clear_stats({"num_w", "num_m", "num_b", "num_g", "d2h_span", "execute_total"});
    if (P->fused) P->clear_stats({"sym_w", "sym_m", "sym_b", "sym_g", "scan"});
    // per unit: e[0..4] symbolic tier boundaries, e[5] after the scan, e[6] numeric placement,
    // e[7..11] numeric tier boundaries, e[12..13] copy start / end (last unit of an output chunk)
    for (int64_t c = 0; c < nch; ++c) {
        cudaEvent_t *e = ev_at(size_t(c) * per);
        // a tier's time counts only for the units that launched it
        const int ts = c < int64_t(P->tiers_sym.size()) ? P->tiers_sym[c] : 7;
        const int tn = c < int64_t(P->tiers_num.size()) ? P->tiers_num[c] : 7;
        const bool g_ok = P->gblocks > 0;
        if (P->fused) {
            P->add_stat("sym_w", elapsed(e[0], e[1]), 0);
            if (ts & 4) P->add_stat("sym_m", elapsed(e[1], e[2]), 0);
            if (ts & 1) P->add_stat("sym_b", elapsed(e[2], e[3]), 0);
            if ((ts & 3) && g_ok) P->add_stat("sym_g", elapsed(e[3], e[4]), 0);
            P->add_stat("scan", elapsed(e[4], e[5]), 0);
        }
        if (!overflow) {
            P->add_stat("num_w", elapsed(e[7], e[8]), 0);
            if (tn & 4) P->add_stat("num_m", elapsed(e[8], e[9]), 0);
            if (tn & 1) P->add_stat("num_b", elapsed(e[9], e[10]), 0);
            if ((tn & 3) && g_ok) P->add_stat("num_g", elapsed(e[10], e[11]), 0);
        }
    }
    const std::vector<int64_t> &gl = P->pend.group_last;
    for (size_t g = 0; g < gl.size() && !overflow; ++g) {
        const int64_t c = gl[g];
        cudaEvent_t end = g + 1 < gl.size() ? ev[size_t(gl[g + 1]) * per + 12] : ev[size_t(nch) * per + 1];
        P->add_stat("d2h_span", elapsed(ev[size_t(c) * per + 12], end), double(P->pend.group_nnz[g]) * 12);
    }
    P->add_stat("execute_total", elapsed(ev[size_t(nch) * per], ev[size_t(nch) * per + 1]),
                double(total) * 12 + 8.0 * (P->R + 1));
    // timeline: per chunk [analysis start, end, numeric start, end, copy start, end] in ms
    P->timeline.assign(size_t(nch) * 6, -1.0);
    cudaEvent_t t0 = ev[size_t(nch) * per];
    for (int64_t c = 0; c < nch; ++c) {
        cudaEvent_t *e = ev_at(size_t(c) * per);
        double *t = &P->timeline[size_t(c) * 6];
        if (P->fused) {
            t[0] = elapsed(t0, e[0]);
            t[1] = elapsed(t0, e[5]);
        }
        if (!overflow) {
            t[2] = elapsed(t0, e[7]);
            t[3] = elapsed(t0, e[11]);
        }
    }
    for (size_t g = 0; g < gl.size() && !overflow; ++g) {  // copies: on each output chunk's last unit
        const size_t c = size_t(gl[g]);
        P->timeline[c * 6 + 4] = elapsed(t0, ev[c * per + 12]);
        P->timeline[c * 6 + 5] = elapsed(t0, ev[c * per + 13]);
    }
}

// The pipeline.  Direct mode writes into (rp_out, col_out, val_out) with room for `capacity`
// nonzeros; sink mode copies every chunk into a pinned staging slot and calls sink->cb.
// Returns nnz of the slice (also when the capacity was too small, in which case nothing past the
// capacity is written and *overflow is set).
int64_t run_pipeline(spgemm_plan_s *P, int64_t *rp_out, int32_t *col_out, double *val_out, int64_t capacity,
                     const Sink *sink, bool *overflow);

int64_t run_pipeline(spgemm_plan_s *P, int64_t *rp_out, int32_t *col_out, double *val_out, int64_t capacity,
                     const Sink *sink, bool *overflow) {
    NvtxRange nv("spgemm_execute");
    if (P->pan) return run_panels(P, rp_out, col_out, val_out, capacity, sink, overflow);
    if (P->failed) fail(SPGEMM_ERR_STATE, "plan is in a failed state");
    DeviceGuard g(P->device);
    finalize_profile(P);  // the previous execution's events are about to be reused
    cudaStream_t s = P->stream, cp = P->copy;
    const int64_t nch = P->num_chunks();
    const int ring = P->ring;
    *overflow = false;

    // row_ptr base
    int64_t base;
    if (P->fused) {
        base = P->base_wanted;
        P->h_small[0] = base;
        // the analysis stream starts after everything already queued on the compute stream
        CK(cudaEventRecord(P->ev_ready, s));
        CK(cudaStreamWaitEvent(P->astream, P->ev_ready, 0));
        // crp[0] = base without an H2D (a small copy would queue behind the operand pieces)
        CK(cudaMemsetAsync(P->crp, 0, sizeof(int64_t), P->astream));
        launch_add(P->crp, 0, base, P->astream);
        CKL("row_ptr base");
        if (P->host_cut)  // the count passes of this execution accumulate sum_u / max_u / max_bound
            CK(cudaMemsetAsync(&P->ctl[0].sum_u, 0, 3 * sizeof(unsigned long long), P->astream));
        // the symbolic passes of this execution accumulate max_nnz and the per-tier row counts
        static_assert(offsetof(Ctl, rows_g) == offsetof(Ctl, max_nnz) + 3 * sizeof(unsigned long long), "Ctl layout");
        CK(cudaMemsetAsync(&P->ctl[0].max_nnz, 0, 4 * sizeof(unsigned long long), P->astream));
        CK(cudaMemsetAsync(&P->ctl[0].rows_m, 0, sizeof(unsigned long long), P->astream));
        P->base_applied = base;
    } else {
        if (P->base_wanted != P->base_applied) {
            launch_add(P->crp, P->R, P->base_wanted - P->base_applied, s);
            CKL("row_ptr base");
            P->base_applied = P->base_wanted;
        }
        base = P->base_applied;
    }
    const int64_t off0 = P->fused ? 0 : P->chunk_offs.empty() ? 0 : P->chunk_offs[0];

    // sink staging
    std::vector<void *> stage(sink ? ring : 0, nullptr);
    struct Release {
        std::vector<void *> &v;
        ~Release() {
            for (auto p : v) pin_release(p);
        }
    } rel{stage};
    int64_t maxn = 0, maxr = 0;
    maxr = P->R;  // an output chunk (group of units) may span any number of rows
    maxn = P->cap;
    if (sink)
        for (int r = 0; r < ring; ++r) stage[r] = pin_acquire(size_t(maxn) * 12 + size_t(maxr + 1) * 8 + 64);
    auto st_val = [&](int b) { return reinterpret_cast<double *>(stage[b]); };
    auto st_col = [&](int b) { return reinterpret_cast<int32_t *>((char *)stage[b] + size_t(maxn) * 8); };
    auto st_rp = [&](int b) {
        return reinterpret_cast<int64_t *>((char *)stage[b] + ((size_t(maxn) * 12 + 7) & ~size_t(7)));
    };

    const int per = 14;
    EvSet pe(P->profile, P->res, 12, size_t(nch) * per + 4);
    if (P->profile) {
        P->tiers_sym.assign(size_t(nch), 0);
        P->tiers_num.assign(size_t(nch), 0);
    }
    CK(cudaEventRecord(P->ev_ready, s));
    CK(cudaStreamWaitEvent(cp, P->ev_ready, 0));
    pe.rec(size_t(nch) * per, s);
    if (rp_out && !sink) {
        if (P->fused) {
            rp_out[0] = base;
            if (nch == 0)  // every row is empty: no chunk will deliver offsets
                for (int64_t r = 1; r <= P->R; ++r) rp_out[r] = base;
        } else {
            CK(cudaMemcpyAsync(rp_out, P->crp, sizeof(int64_t) * (P->R + 1), cudaMemcpyDeviceToHost, cp));
        }
    }
    // fused plans: the symbolic pass + scan of unit j + 2 is enqueued while unit j's numeric pass is
    // (the host waits for unit j + 1's total in between, so the stream always holds queued work)
    constexpr int64_t LOOKAHEAD = 2;
    if (P->fused)
        for (int64_t j = 0; j < std::min<int64_t>(LOOKAHEAD, nch); ++j) enqueue_analysis(P, j, pe.at(size_t(j) * per));

    std::vector<int64_t> offs(nch + 1, 0);  // chunk offsets relative to the slice
    if (!P->fused && nch > 0)
        for (int64_t c = 0; c <= nch; ++c) offs[c] = P->chunk_offs[c] - off0;
    // Output chunks ("groups") are runs of consecutive analysis units sharing one ring slot: the
    // copy engine moves few large pieces (a 60 MB copy runs ~8% slower than a 1 GB one on the
    // host link) while the units stay small for a quick pipeline start.  A group closes when the
    // next unit would not fit the slot, when it reaches its target (the first group: one unit;
    // each later target: twice the previous group), or when the previous group's copy has
    // finished (so the copy engine never waits for a large group to fill).
    static const bool no_pad = [] {  // ablation knob: ring data at the start of the slot
        const char *v = getenv("SPGEMM_NO_ALIGN_PAD");
        return v && v[0] == '1';
    }();
    // A group's data starts `pad` elements into its ring slot, chosen so that the slot addresses
    // and the host destinations agree modulo 256 bytes; its copy is split into a head up to the
    // next 8 KB boundary of the host values and a bulk that starts page-aligned on the host and
    // 256-byte aligned on the device.  On some boxes copy-engine D2H copies whose host destination
    // does not start on a page ran 6 % slower (tools/d2h_offsets.py: C2's output in 9 copies at
    // 53.7 GB/s with 128-byte-aligned starts, 56.7 with 4 KB-aligned ones, 57.1 as one copy).
    struct Group {
        int b;
        int64_t u0, u1, r0, r1, off, nnz, pad;
    };
    std::vector<Group> groups;
    // Sink mode: a consumer thread hands every output chunk to the callback as soon as its copy has
    // landed in the staging slot, while this thread keeps enqueueing later units; a staging slot is
    // reused only after the callback of the chunk in it returned (back-pressure), so a slow sink
    // delays the pipeline only when it is `ring` chunks behind.
    struct Consumer {
        std::mutex mu;
        std::condition_variable cv;
        std::vector<Group> q;  // closed groups, in order
        int64_t done = 0;      // callbacks completed
        bool stop = false;
        int rc = 0;            // first non-zero callback return
        std::string cuda_err;
        std::thread th;
        ~Consumer() {
            {
                std::lock_guard<std::mutex> lk(mu);
                stop = true;
            }
            cv.notify_all();
            if (th.joinable()) th.join();
        }
    } cons;
    if (sink) {
        cons.th = std::thread([&, dev = P->device] {
            cudaSetDevice(dev);
            for (int64_t g = 0;; ++g) {
                Group G;
                {
                    std::unique_lock<std::mutex> lk(cons.mu);
                    cons.cv.wait(lk, [&] { return int64_t(cons.q.size()) > g || cons.stop; });
                    if (int64_t(cons.q.size()) <= g) return;
                    G = cons.q[g];
                }
                const cudaError_t e = cudaEventSynchronize(P->ev_d2h[G.b]);
                int rc = 0;
                if (e != cudaSuccess) {
                    std::lock_guard<std::mutex> lk(cons.mu);
                    cons.cuda_err = cudaGetErrorString(e);
                    rc = -1;
                } else {
                    int64_t *rp = st_rp(G.b);
                    const int64_t first = rp[0];
                    for (int64_t k = 0; k <= G.r1 - G.r0; ++k) rp[k] -= first;
                    NvtxRange cbr("sink callback");
                    rc = sink->cb(sink->user, P->row_begin + G.r0, P->row_begin + G.r1, rp, st_col(G.b), st_val(G.b),
                                  rp[G.r1 - G.r0]);
                }
                {
                    std::lock_guard<std::mutex> lk(cons.mu);
                    if (rc != 0 && cons.rc == 0) cons.rc = rc;
                    if (rc == 0) cons.done = g + 1;
                }
                cons.cv.notify_all();
                if (rc != 0) return;
            }
        });
    }
    auto sink_failed = [&]() {  // after a callback failure: drain the GPU and report
        CK(cudaStreamSynchronize(cp));
        CK(cudaStreamSynchronize(s));
        if (P->astream && P->astream != s) CK(cudaStreamSynchronize(P->astream));
        if (!cons.cuda_err.empty()) fail(SPGEMM_ERR_CUDA, "chunk copy: " + cons.cuda_err);
        fail(SPGEMM_ERR_CALLBACK, "chunk sink returned " + std::to_string(cons.rc));
    };
    auto wait_consumed = [&](int64_t upto) {  // sink: callbacks of groups < upto have returned
        std::unique_lock<std::mutex> lk(cons.mu);
        cons.cv.wait(lk, [&] { return cons.done >= upto || cons.rc != 0; });
        if (cons.rc != 0) {
            lk.unlock();
            sink_failed();
        }
    };
    auto push_group = [&](const Group &G) {
        groups.push_back(G);
        if (sink) {
            {
                std::lock_guard<std::mutex> lk(cons.mu);
                cons.q.push_back(G);
            }
            cons.cv.notify_all();
        }
    };
    auto close_group = [&](Group &G) {  // enqueue the group's copies after its numeric passes
        CK(cudaEventRecord(P->ev_num[G.b], s));
        CK(cudaStreamWaitEvent(cp, P->ev_num[G.b], 0));
        pe.rec(size_t(G.u1 - 1) * per + 12, cp);
        int32_t *dcol = sink ? st_col(G.b) : col_out + G.off;
        double *dval = sink ? st_val(G.b) : val_out + G.off;
        if (G.nnz > 0) {
            // a head of < 32 elements up to the first 256-byte boundary of the host values, then
            // the bulk with source and destination both aligned
            // head: up to the next 8 KB boundary of the host values (then, with page-aligned host
            // arrays, the columns start on a 4 KB boundary too)
            int64_t h = 0;
            if (!no_pad) h = std::min<int64_t>(G.nnz, int64_t(((8192u - (reinterpret_cast<uintptr_t>(dval) & 8191u)) & 8191u) / 8u));
            const int32_t *scol = P->ring_col[G.b] + G.pad;
            const double *sval = P->ring_val[G.b] + G.pad;
            if (h > 0) {
                CK(cudaMemcpyAsync(dcol, scol, sizeof(int32_t) * h, cudaMemcpyDeviceToHost, cp));
                CK(cudaMemcpyAsync(dval, sval, sizeof(double) * h, cudaMemcpyDeviceToHost, cp));
            }
            if (G.nnz > h) {
                CK(cudaMemcpyAsync(dcol + h, scol + h, sizeof(int32_t) * (G.nnz - h), cudaMemcpyDeviceToHost, cp));
                CK(cudaMemcpyAsync(dval + h, sval + h, sizeof(double) * (G.nnz - h), cudaMemcpyDeviceToHost, cp));
            }
        }
        if (sink) {
            CK(cudaMemcpyAsync(st_rp(G.b), P->crp + G.r0, sizeof(int64_t) * (G.r1 - G.r0 + 1), cudaMemcpyDeviceToHost, cp));
        } else if (rp_out && P->fused && G.r1 > G.r0) {
            int64_t *drp = rp_out + G.r0 + 1;
            const int64_t n = G.r1 - G.r0;
            int64_t h = 0;  // head up to the next 4 KB boundary of the host destination
            if (!no_pad) h = std::min<int64_t>(n, int64_t(((4096u - (reinterpret_cast<uintptr_t>(drp) & 4095u)) & 4095u) / 8u));
            if (h > 0) CK(cudaMemcpyAsync(drp, P->crp + G.r0 + 1, sizeof(int64_t) * h, cudaMemcpyDeviceToHost, cp));
            if (n > h)
                CK(cudaMemcpyAsync(drp + h, P->crp + G.r0 + 1 + h, sizeof(int64_t) * (n - h), cudaMemcpyDeviceToHost, cp));
        }
        pe.rec(size_t(G.u1 - 1) * per + 13, cp);
        CK(cudaEventRecord(P->ev_d2h[G.b], cp));
    };

    Group cur{-1, 0, 0, 0, 0, 0, 0, 0};
    int64_t target = 0;
    static const bool no_groups = [] {  // ablation knob: one output chunk per unit
        const char *v = getenv("SPGEMM_NO_GROUPS");
        return v && v[0] == '1';
    }();
    // reordered chunks are not contiguous in host C: each leaves as its own copy
    const bool reorder = !P->unit_order.empty();
    if (reorder && sink) fail(SPGEMM_ERR_INVALID_ARGUMENT, "sink mode delivers rows in order: needs order = 0");
    const bool one_per_unit = no_groups || reorder;
    for (int64_t t = 0; t < nch; ++t) {
        const int64_t j = reorder ? P->unit_order[t] : t;
        const int64_t r0 = P->chunk_rows[j], r1 = P->chunk_rows[j + 1];
        int64_t mx = P->max_nnz;
        if (P->fused) {
            // unit j's symbolic pass was enqueued LOOKAHEAD iterations ago; its total decides where the
            // unit lands on the host and its max row nnz which numeric tiers to launch
            {
                NvtxRange w("wait unit total");
                CK(cudaEventSynchronize(P->ev_tot[j]));
            }
            offs[j + 1] = P->h_small[1 + 2 * j] - base;
            mx = P->h_small[2 + 2 * j];
        }
        const int64_t o = offs[j], n = offs[j + 1] - offs[j];
        if (!sink && o + n > capacity) *overflow = true;
        if (*overflow) {
            if (P->fused && j + LOOKAHEAD < nch) enqueue_analysis(P, j + LOOKAHEAD, pe.at(size_t(j + LOOKAHEAD) * per));
            continue;
        }
        if (cur.b >= 0) {
            bool close = one_per_unit || cur.nnz + n > P->cap || cur.nnz >= target;
            if (!close && !groups.empty()) close = cudaEventQuery(P->ev_d2h[groups.back().b]) == cudaSuccess;
            if (close) {
                close_group(cur);
                push_group(cur);
                target = std::min<int64_t>(P->cap, 2 * cur.nnz);
                cur.b = -1;
            }
        }
        if (cur.b < 0) {  // open a group in the next ring slot
            const int64_t g = int64_t(groups.size());
            cur = Group{int(g % ring), j, j, r0, r0, o, 0, 0};
            if (!sink && val_out && !no_pad) {
                const uintptr_t hv = reinterpret_cast<uintptr_t>(val_out + o);
                const uintptr_t rv = reinterpret_cast<uintptr_t>(P->ring_val[cur.b]);
                cur.pad = int64_t(((hv - rv) & 255u) / 8u);  // < RING_PAD
            }
            if (g >= ring) {
                CK(cudaStreamWaitEvent(s, P->ev_d2h[cur.b], 0));
                if (sink) wait_consumed(g - ring + 1);  // staging slot cur.b is free again
            }
        }
        if (P->fused) CK(cudaStreamWaitEvent(s, P->ev_tot[j], 0));  // (already complete: host waited)
        if (!P->chunk_wait.empty() && P->chunk_wait[j] >= 0)       // host operands: value pieces
            CK(cudaStreamWaitEvent(s, P->ev_piece[P->chunk_wait[j]], 0));
        pe.rec(size_t(j) * per + 6, s);
        enqueue_numeric(P, j, cur.b, cur.pad + cur.nnz, mx, pe.at(size_t(j) * per + 7));
        cur.nnz += n;
        cur.u1 = j + 1;
        cur.r1 = r1;
        if (one_per_unit || (cur.nnz >= target && cur.nnz > 0)) {
            // the group reached its target: its copy goes now, not one analysis pass later when
            // the next unit's total is known (the first group is one unit: the first copy starts
            // right after the first numeric pass)
            close_group(cur);
            push_group(cur);
            target = std::min<int64_t>(P->cap, 2 * cur.nnz);
            cur.b = -1;
        }
        if (P->fused && j + LOOKAHEAD < nch) enqueue_analysis(P, j + LOOKAHEAD, pe.at(size_t(j + LOOKAHEAD) * per));
    }
    if (cur.b >= 0) {
        close_group(cur);
        push_group(cur);
    }
    if (sink) wait_consumed(int64_t(groups.size()));
    P->num_groups = int64_t(groups.size());
    pe.rec(size_t(nch) * per + 1, cp);
    CK(cudaStreamSynchronize(cp));
    CK(cudaStreamSynchronize(s));
    if (P->astream && P->astream != s) CK(cudaStreamSynchronize(P->astream));
    unsigned err[2] = {0, 0};
    CK(cudaMemcpy(&err[0], &P->ctl[1].err, sizeof(unsigned), cudaMemcpyDeviceToHost));
    if (err[0]) fail(SPGEMM_ERR_STATE, "internal: numeric pass produced a row whose nnz differs from the symbolic pass");
    const int64_t total = offs[nch];
    if (P->fused) {
        P->nnz = total;
        P->chunk_offs = offs;
        Ctl hc;
        CK(cudaMemcpy(&hc, P->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost));
        P->max_nnz = (int64_t)hc.max_nnz;
        P->rows_w = (int64_t)hc.rows_w;
        P->rows_b = (int64_t)hc.rows_b;
        P->rows_g = (int64_t)hc.rows_g;
        P->rows_m = (int64_t)hc.rows_m;
        if (P->host_cut) {
            P->products = (int64_t)hc.sum_u;
            P->max_u = (int64_t)hc.max_u;
        }
    }
    if (P->profile) {  // per-kernel times are read from the events lazily (finalize_profile)
        P->pend.active = true;
        P->pend.ev = pe.ev;
        P->pend.nch = nch;
        P->pend.per = per;
        P->pend.overflow = *overflow;
        P->pend.offs = offs;
        P->pend.total = total;
        P->pend.group_last.clear();
        P->pend.group_nnz.clear();
        for (const auto &G : groups) {
            P->pend.group_last.push_back(G.u1 - 1);
            P->pend.group_nnz.push_back(G.nnz);
        }
    }
    return total;
}

}  // namespace

namespace {
spgemm_status guarded(const std::function<void()> &f) {
    try {
        f();
        return SPGEMM_OK;
    } catch (const Err &e) {
        g_err = e.msg;
        return e.st;
    } catch (const std::bad_alloc &) {
        g_err = "host out of memory";
        return SPGEMM_ERR_HOST_ALLOC;
    } catch (...) {
        g_err = "unknown internal error";
        return SPGEMM_ERR_STATE;
    }
}

void mark_failed(spgemm_plan_s *P, spgemm_status st) {
    if (st == SPGEMM_ERR_CUDA || st == SPGEMM_ERR_STATE) P->failed = true;
}

}  // namespace

extern "C" {

void spgemm_opts_default(spgemm_opts *o) {
    if (!o) return;
    std::memset(o, 0, sizeof(*o));
    o->device = -1;
    o->ring = 2;
    o->row_begin = 0;
    o->row_end = -1;
}

spgemm_status spgemm_plan(const spgemm_csr *A, const spgemm_csr *B, size_t budget, const spgemm_opts *opts,
                          spgemm_plan_t *plan_out) {
    if (!plan_out) {
        g_err = "plan_out is NULL";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    *plan_out = nullptr;
    spgemm_plan_s *P = nullptr;
    int prev = -1;
    cudaGetDevice(&prev);
    const int cp = opts ? opts->col_panels : 0;
    spgemm_status st = guarded([&] {
        P = new spgemm_plan_s();
        if (cp >= 2) do_panel_plan(A, B, budget, opts, P);
        else do_plan(A, B, budget, opts, P);
    });
    if (st == SPGEMM_ERR_BUDGET && cp == 0 && A && B && (B->where == SPGEMM_HOST || A->where == SPGEMM_HOST)) {
        // B (or A) does not fit the budget: retry with B cut into column panels (§III-A)
        const std::string first = g_err;
        delete P;
        P = nullptr;
        st = guarded([&] {
            P = new spgemm_plan_s();
            do_panel_plan(A, B, budget, opts, P);
        });
        if (st != SPGEMM_OK) g_err = first + "; column-panel mode: " + g_err;
    }
    if (st != SPGEMM_OK) {
        delete P;
        if (prev >= 0) cudaSetDevice(prev);
        return st;
    }
    if (prev >= 0) cudaSetDevice(prev);
    *plan_out = P;
    return SPGEMM_OK;
}

spgemm_status spgemm_plan_info(spgemm_plan_t P, spgemm_info *info) {
    if (!P || !info) {
        g_err = "NULL argument";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    std::memset(info, 0, sizeof(*info));
    info->nrows = P->R;
    info->ncols = P->ncols;
    info->nnz = P->nnz;
    info->products = P->products;
    info->max_row_nnz = P->nnz >= 0 ? P->max_nnz : -1;
    info->max_row_products = P->max_u;
    info->num_chunks = (int32_t)P->num_chunks();
    info->ring = P->ring;
    info->chunk_capacity = P->cap;
    info->arena_bytes = (int64_t)P->arena_bytes;
    info->arena_used = (int64_t)P->used;
    info->ring_bytes = (int64_t)P->ring_bytes;
    info->rows_warp = P->rows_w;
    info->rows_block = P->rows_b;
    info->rows_global = P->rows_g;
    info->rows_medium = P->rows_m;
    info->fused = P->fused ? 1 : 0;
    info->num_copies = (int32_t)P->num_groups;
    info->col_panels = P->col_panels;
    if (P->pan) info->num_chunks = (int32_t)P->panel_units;
    return SPGEMM_OK;
}

spgemm_status spgemm_plan_chunks(spgemm_plan_t P, int64_t *rows, int64_t *offs) {
    if (!P || !rows) {
        g_err = "NULL argument";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    if (P->pan) {
        g_err = "column-panel plan: chunks are (row unit, column panel) pairs";
        return SPGEMM_ERR_STATE;
    }
    const int64_t n = P->num_chunks();
    if (n == 0) {
        rows[0] = 0;
        if (offs) offs[0] = 0;
        return SPGEMM_OK;
    }
    const bool known = (int64_t)P->chunk_offs.size() == n + 1;
    const int64_t base0 = known ? P->chunk_offs[0] : 0;
    for (int64_t k = 0; k <= n; ++k) {
        rows[k] = P->chunk_rows[k];
        if (offs) offs[k] = known ? P->chunk_offs[k] - base0 : -1;
    }
    return SPGEMM_OK;
}

spgemm_status spgemm_execute_into(spgemm_plan_t P, int64_t *row_ptr, int32_t *col_idx, double *values) {
    if (!P) {
        g_err = "plan is NULL";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    spgemm_status st = guarded([&] {
        if (P->nnz < 0)
            fail(SPGEMM_ERR_STATE, "fused plan: nnz(C) is not known yet (use spgemm_multiply, spgemm_execute_stream "
                                   "or spgemm_execute_capacity)");
        if (P->nnz > 0 && (!col_idx || !values)) fail(SPGEMM_ERR_INVALID_ARGUMENT, "col_idx/values output is NULL");
        bool ovf = false;
        run_pipeline(P, row_ptr, col_idx, values, P->nnz, nullptr, &ovf);
        if (ovf) fail(SPGEMM_ERR_STATE, "internal: nnz changed between executions");
    });
    mark_failed(P, st);
    return st;
}

spgemm_status spgemm_execute_capacity(spgemm_plan_t P, int64_t *row_ptr, int32_t *col_idx, double *values,
                                      int64_t capacity, int64_t *nnz_out) {
    if (!P) {
        g_err = "plan is NULL";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    int64_t total = -1;
    bool ovf = false;
    spgemm_status st = guarded([&] {
        if (capacity > 0 && (!col_idx || !values)) fail(SPGEMM_ERR_INVALID_ARGUMENT, "col_idx/values output is NULL");
        total = run_pipeline(P, row_ptr, col_idx, values, capacity, nullptr, &ovf);
    });
    if (nnz_out && total >= 0) *nnz_out = total;
    if (st == SPGEMM_OK && ovf) {
        g_err = "output capacity " + std::to_string(capacity) + " < nnz(C) = " + std::to_string(total);
        return SPGEMM_ERR_CAPACITY;
    }
    mark_failed(P, st);
    return st;
}

spgemm_status spgemm_execute(spgemm_plan_t P, spgemm_csr_out *C) {
    if (!P || !C) {
        g_err = "NULL argument";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    spgemm_status st = guarded([&] {
        DeviceGuard g(P->device);
        if (P->nnz < 0) {  // fused: learn nnz with a sink-less counting run is not possible; run once into nothing
            bool ovf = false;
            run_pipeline(P, nullptr, nullptr, nullptr, 0, nullptr, &ovf);
        }
        if (!P->h_rp) {
            if (cudaHostAlloc(&P->h_rp, sizeof(int64_t) * (P->R + 1), 0) != cudaSuccess ||
                cudaHostAlloc(&P->h_col, sizeof(int32_t) * std::max<int64_t>(P->nnz, 1), 0) != cudaSuccess ||
                cudaHostAlloc(&P->h_val, sizeof(double) * std::max<int64_t>(P->nnz, 1), 0) != cudaSuccess) {
                cudaGetLastError();
                fail(SPGEMM_ERR_HOST_ALLOC, "pinned allocation of the output failed");
            }
        }
        bool ovf = false;
        run_pipeline(P, P->h_rp, P->h_col, P->h_val, P->nnz, nullptr, &ovf);
        C->nrows = P->R;
        C->ncols = P->ncols;
        C->nnz = P->nnz;
        C->row_ptr = P->h_rp;
        C->col_idx = P->h_col;
        C->values = P->h_val;
    });
    mark_failed(P, st);
    return st;
}

spgemm_status spgemm_execute_stream(spgemm_plan_t P, spgemm_chunk_cb cb, void *user) {
    if (!P) {
        g_err = "plan is NULL";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    spgemm_status st = guarded([&] {
        if (!cb) fail(SPGEMM_ERR_INVALID_ARGUMENT, "callback is NULL");
        Sink sk;
        sk.cb = cb;
        sk.user = user;
        bool ovf = false;
        run_pipeline(P, nullptr, nullptr, nullptr, INT64_MAX, &sk, &ovf);
    });
    mark_failed(P, st);
    return st;
}

spgemm_status spgemm_row_products(const spgemm_csr *A, const spgemm_csr *B, const spgemm_opts *o, int64_t *u_out,
                                  int64_t *total_out) {
    return guarded([&] {
        check_csr(A, "A");
        check_csr(B, "B");
        if (!u_out) fail(SPGEMM_ERR_INVALID_ARGUMENT, "u_out is NULL");
        if (A->ncols != B->nrows) fail(SPGEMM_ERR_SHAPE, "A.ncols != B.nrows");
        spgemm_opts opts;
        spgemm_opts_default(&opts);
        if (o) opts = *o;
        const int64_t rb = opts.row_begin, re = opts.row_end < 0 ? A->nrows : opts.row_end;
        if (rb < 0 || re < rb || re > A->nrows) fail(SPGEMM_ERR_SHAPE, "row range outside A");
        int dev = opts.device;
        if (dev < 0) CK(cudaGetDevice(&dev));
        DeviceGuard g(dev);
        cudaStream_t s = (cudaStream_t)opts.stream;
        const int64_t R = re - rb;
        // the count reads A.rp, A.col and B.rp: host operands go up into one temporary buffer
        // (this call is analysis, not the pipeline: no arena)
        const int64_t p0 = A->where == SPGEMM_HOST ? A->row_ptr[rb] : 0;
        const int64_t p1 = A->where == SPGEMM_HOST ? A->row_ptr[re] : 0;
        size_t bytes = 256 + size_t(R) * 8 + sizeof(Ctl) + 256;
        if (A->where == SPGEMM_HOST) bytes += size_t(R + 1) * 8 + size_t(p1 - p0) * 4 + 512;
        if (B->where == SPGEMM_HOST) bytes += size_t(B->nrows + 1) * 8 + 256;
        char *buf = nullptr;
        CK(cudaMalloc(&buf, bytes));
        struct Free {
            char *p;
            ~Free() { cudaFree(p); }
        } fr{buf};
        size_t off = 0;
        auto take = [&](size_t n) {
            char *q = buf + off;
            off = (off + n + 255) & ~size_t(255);
            return q;
        };
        int64_t *du = reinterpret_cast<int64_t *>(take(size_t(std::max<int64_t>(R, 1)) * 8));
        Ctl *ctl = reinterpret_cast<Ctl *>(take(sizeof(Ctl)));
        CK(cudaMemsetAsync(ctl, 0, sizeof(Ctl), s));
        DevCSR dA{}, dB{};
        if (A->where == SPGEMM_DEVICE) {
            dA = DevCSR{A->row_ptr + rb, A->col_idx, A->values, R, A->ncols};
        } else {
            int64_t *rp = reinterpret_cast<int64_t *>(take(size_t(R + 1) * 8));
            int32_t *c = reinterpret_cast<int32_t *>(take(size_t(std::max<int64_t>(p1 - p0, 1)) * 4));
            CK(cudaMemcpyAsync(rp, A->row_ptr + rb, size_t(R + 1) * 8, cudaMemcpyHostToDevice, s));
            if (p1 > p0) CK(cudaMemcpyAsync(c, A->col_idx + p0, size_t(p1 - p0) * 4, cudaMemcpyHostToDevice, s));
            launch_rebase(rp, R + 1, p0, s);
            CKL("rebase");
            dA = DevCSR{rp, c, nullptr, R, A->ncols};
        }
        if (B->where == SPGEMM_DEVICE) {
            dB = DevCSR{B->row_ptr, B->col_idx, B->values, B->nrows, B->ncols};
        } else {
            int64_t *rp = reinterpret_cast<int64_t *>(take(size_t(B->nrows + 1) * 8));
            CK(cudaMemcpyAsync(rp, B->row_ptr, size_t(B->nrows + 1) * 8, cudaMemcpyHostToDevice, s));
            dB = DevCSR{rp, nullptr, nullptr, B->nrows, B->ncols};
        }
        launch_count(dA, dB, du, ctl, s, true);
        CKL("count");
        Ctl hc;
        if (R > 0) CK(cudaMemcpyAsync(u_out, du, size_t(R) * 8, cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(&hc, ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        if (total_out) *total_out = (int64_t)hc.sum_u;
    });
}

spgemm_status spgemm_plan_row_bounds(spgemm_plan_t P, int64_t *bnd_out) {
    return guarded([&] {
        if (!P || !bnd_out) fail(SPGEMM_ERR_INVALID_ARGUMENT, "NULL argument");
        if (P->pan) fail(SPGEMM_ERR_STATE, "column-panel plans keep no row bounds (one per panel and unit)");
        if (P->host_cut && P->products < 0) fail(SPGEMM_ERR_STATE, "host-cut plan: bounds are counted in execute");
        DeviceGuard g(P->device);
        if (P->R > 0) CK(cudaMemcpyAsync(bnd_out, P->bnd, size_t(P->R) * 8, cudaMemcpyDeviceToHost, P->stream));
        CK(cudaStreamSynchronize(P->stream));
    });
}

spgemm_status spgemm_rebase_host(int64_t *row_ptr, int64_t n, int64_t delta) {
    if (n > 0 && !row_ptr) {
        g_err = "row_ptr is NULL";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    if (delta == 0) return SPGEMM_OK;
    for (int64_t i = 0; i < n; ++i) row_ptr[i] += delta;
    return SPGEMM_OK;
}

spgemm_status spgemm_set_row_ptr_base(spgemm_plan_t P, int64_t base) {
    if (!P) {
        g_err = "plan is NULL";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    P->base_wanted = base;
    return SPGEMM_OK;
}

spgemm_status spgemm_multiply(const spgemm_csr *A, const spgemm_csr *B, size_t budget, const spgemm_opts *opts,
                              int64_t *row_ptr, int32_t *col_idx, double *values, int64_t cap, int64_t *nnz_out) {
    spgemm_opts o;
    spgemm_opts_default(&o);
    if (opts) o = *opts;
    o.fused = 1;
    spgemm_plan_t P = nullptr;
    spgemm_status st = spgemm_plan(A, B, budget, &o, &P);
    if (st != SPGEMM_OK) return st;
    st = spgemm_execute_capacity(P, row_ptr, col_idx, values, cap, nnz_out);
    spgemm_free(P);
    return st;
}

spgemm_status spgemm_stats(spgemm_plan_t P, spgemm_kernel_stat *out, int32_t max, int32_t *n) {
    if (!P || !n) {
        g_err = "NULL argument";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    {
        DeviceGuard g(P->device);
        finalize_profile(P);
    }
    *n = (int32_t)P->stats.size();
    for (int32_t k = 0; k < max && k < *n && out; ++k) {
        std::memset(&out[k], 0, sizeof(out[k]));
        std::strncpy(out[k].name, P->stats[k].name.c_str(), sizeof(out[k].name) - 1);
        out[k].launches = P->stats[k].launches;
        out[k].ms = P->stats[k].ms;
        out[k].bytes = P->stats[k].bytes;
    }
    return SPGEMM_OK;
}

spgemm_status spgemm_timeline(spgemm_plan_t P, double *out, int64_t max, int64_t *n) {
    if (!P || !n) {
        g_err = "NULL argument";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    {
        DeviceGuard g(P->device);
        finalize_profile(P);
    }
    *n = (int64_t)P->timeline.size();
    for (int64_t k = 0; k < max && k < *n && out; ++k) out[k] = P->timeline[k];
    return SPGEMM_OK;
}

void spgemm_free(spgemm_plan_t P) {
    if (!P) return;
    int prev = -1;
    cudaGetDevice(&prev);
    cudaSetDevice(P->device);
    delete P;
    if (prev >= 0) cudaSetDevice(prev);
}

void spgemm_release_cache(void) {
    {
        std::lock_guard<std::mutex> lk(g_pin_mu);
        std::vector<PinnedBlock> keep;
        for (auto &b : g_pins) {
            if (b.used) keep.push_back(b);
            else cudaFreeHost(b.p);
        }
        g_pins.swap(keep);
    }
    std::lock_guard<std::mutex> lk(g_res_mu);
    std::vector<Res *> keep;
    int prev = -1;
    cudaGetDevice(&prev);
    for (auto r : g_res) {
        if (r->used) {
            keep.push_back(r);
            continue;
        }
        cudaSetDevice(r->device);
        r->destroy();
        delete r;
    }
    if (prev >= 0) cudaSetDevice(prev);
    g_res.swap(keep);
}

const char *spgemm_status_string(spgemm_status s) {
    switch (s) {
        case SPGEMM_OK: return "SPGEMM_OK";
        case SPGEMM_ERR_INVALID_ARGUMENT: return "SPGEMM_ERR_INVALID_ARGUMENT";
        case SPGEMM_ERR_SHAPE: return "SPGEMM_ERR_SHAPE";
        case SPGEMM_ERR_INDEX_OVERFLOW: return "SPGEMM_ERR_INDEX_OVERFLOW";
        case SPGEMM_ERR_BUDGET: return "SPGEMM_ERR_BUDGET";
        case SPGEMM_ERR_HOST_ALLOC: return "SPGEMM_ERR_HOST_ALLOC";
        case SPGEMM_ERR_CUDA: return "SPGEMM_ERR_CUDA";
        case SPGEMM_ERR_STATE: return "SPGEMM_ERR_STATE";
        case SPGEMM_ERR_CAPACITY: return "SPGEMM_ERR_CAPACITY";
        case SPGEMM_ERR_CALLBACK: return "SPGEMM_ERR_CALLBACK";
    }
    return "SPGEMM_ERR_UNKNOWN";
}

const char *spgemm_last_error(void) { return g_err.c_str(); }

int32_t spgemm_abi_version(void) { return SPGEMM_ABI_VERSION; }

int64_t spgemm_kernel_launches(void) { return (int64_t)kernel_launches(); }

}  // extern "C"
