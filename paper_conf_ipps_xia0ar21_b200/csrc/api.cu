// api.cu -- C ABI (include/spgemm.h), arena, planner and the chunk pipeline.
//
// Host side of the hot path (DESIGN.md §8 rows):
//   S0 residency   inputs adopted in place (device) or H2D-copied once into the arena (host);
//                  A == B is kept once (C = A x A, §V-B).
//   S1 panels      rows [row_begin, row_end) of A are this plan's row panel (§III-A, §III-D
//                  L169); B is used whole (one column panel, B fits the budget).
//   S9 arena       ONE device allocation (or caller workspace) sub-allocated by offsets; nothing
//                  is allocated between spgemm_plan returning and spgemm_free (§IV-B).
//   S10 planner    output chunks cut from the exact symbolic nnz so that each fits a ring buffer
//                  (the paper's upper-bound sizing is loose, §IV-B).
//   S8 pipeline    compute stream + copy stream, R ring buffers, CUDA events only -- the host
//                  never blocks inside spgemm_execute_into until the last copy (§IV-B).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <functional>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "../../include/spgemm.h"
#include "internal.h"

using namespace spg;

namespace {

thread_local std::string g_err;

struct Err {
    spgemm_status st;
    std::string msg;
};

[[noreturn]] void fail(spgemm_status st, const std::string &msg) { throw Err{st, msg}; }

void ck(cudaError_t e, const char *what) {
    if (e != cudaSuccess) fail(SPGEMM_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}
#define CK(x) ck((x), #x)
#define CKL(what) ck(cudaGetLastError(), what)

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        if (dev >= 0) {
            CK(cudaGetDevice(&prev));
            if (prev != dev) CK(cudaSetDevice(dev));
            else prev = -1;
        }
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

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

struct Stat {
    std::string name;
    int launches = 0;
    double ms = 0, bytes = 0;
};

}  // namespace

struct spgemm_plan_s {
    int device = 0, num_sms = 148;
    cudaStream_t stream = nullptr, copy = nullptr;
    bool own_stream = false;
    std::vector<cudaEvent_t> ev_num, ev_d2h;
    cudaEvent_t ev_ready = nullptr;

    char *arena = nullptr;
    size_t arena_bytes = 0, used = 0;
    bool own_arena = false;

    DevCSR A{}, B{};
    int64_t R = 0, ncols = 0, nnzA = 0, nnzB = 0, row_begin = 0;
    int group = 32;

    int64_t *u = nullptr, *crp = nullptr, *tmp = nullptr;
    int32_t *listB = nullptr, *listG = nullptr;
    Ctl *ctl = nullptr;  // [0] plan passes, [1] numeric passes

    uint32_t *gbits = nullptr;
    double *gvals = nullptr;
    int64_t gstride_bits = 0, gstride_vals = 0;
    int gblocks = 0;

    int ring = 2;
    int64_t cap = 0;
    size_t ring_bytes = 0;
    std::vector<int32_t *> ring_col;
    std::vector<double *> ring_val;

    std::vector<int64_t> chunk_rows, chunk_offs;  // num_chunks + 1 each; offs relative to slice
    int64_t nnz = 0, products = 0, max_nnz = 0, max_u = 0, max_bound = 0;
    int64_t rows_w = 0, rows_b = 0, rows_g = 0;
    int64_t base_applied = 0, base_wanted = 0;

    int64_t *h_rp = nullptr;
    int32_t *h_col = nullptr;
    double *h_val = nullptr;

    bool profile = false;
    std::vector<Stat> stats;
    bool failed = false;

    size_t take(size_t bytes, const char *what) {
        size_t off = (used + 255) & ~size_t(255);
        if (off + bytes > arena_bytes)
            fail(SPGEMM_ERR_BUDGET, std::string("device budget exhausted placing ") + what + " (" +
                                        std::to_string(bytes) + " B, used " + std::to_string(off) + " of " +
                                        std::to_string(arena_bytes) + ")");
        used = off + bytes;
        return off;
    }
    template <typename T>
    T *alloc(int64_t n, const char *what) {
        return reinterpret_cast<T *>(arena + take(size_t(n > 0 ? n : 1) * sizeof(T), what));
    }
    void add_stat(const std::string &name, double ms, double bytes) {
        for (auto &s : stats)
            if (s.name == name) {
                s.launches++;
                s.ms += ms;
                s.bytes += bytes;
                return;
            }
        Stat s;
        s.name = name;
        s.launches = 1;
        s.ms = ms;
        s.bytes = bytes;
        stats.push_back(s);
    }
    ~spgemm_plan_s() {
        DeviceGuard g(-1);
        if (stream) cudaStreamSynchronize(stream);
        if (copy) cudaStreamSynchronize(copy);
        for (auto e : ev_num) cudaEventDestroy(e);
        for (auto e : ev_d2h) cudaEventDestroy(e);
        if (ev_ready) cudaEventDestroy(ev_ready);
        if (copy) cudaStreamDestroy(copy);
        if (own_stream && stream) cudaStreamDestroy(stream);
        if (own_arena && arena) cudaFree(arena);
        if (h_rp) cudaFreeHost(h_rp);
        if (h_col) cudaFreeHost(h_col);
        if (h_val) cudaFreeHost(h_val);
    }
};

namespace {

spgemm_status guarded(const std::function<void()> &f);

void check_csr(const spgemm_csr *M, const char *name) {
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

double elapsed(cudaEvent_t a, cudaEvent_t b) {
    float ms = 0;
    if (cudaEventElapsedTime(&ms, a, b) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    return ms;
}

struct EvSet {  // events for profiling one launch group
    std::vector<cudaEvent_t> ev;
    explicit EvSet(bool on, int n) {
        if (!on) return;
        ev.resize(n);
        for (auto &e : ev) CK(cudaEventCreate(&e));
    }
    ~EvSet() {
        for (auto e : ev) cudaEventDestroy(e);
    }
    cudaEvent_t *ptr() { return ev.empty() ? nullptr : ev.data(); }
};

void do_plan(const spgemm_csr *Ah, const spgemm_csr *Bh, size_t budget, const spgemm_opts *o, spgemm_plan_s *P) {
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
    P->profile = opts.profile != 0;
    P->ring = opts.ring;
    P->row_begin = rb;
    P->R = re - rb;
    P->ncols = Bh->ncols;
    P->nnzB = Bh->nnz;
    P->base_wanted = opts.row_ptr_base;

    // streams and events (created at plan time: no creation inside execute)
    if (opts.stream) {
        P->stream = (cudaStream_t)opts.stream;
    } else {
        CK(cudaStreamCreateWithFlags(&P->stream, cudaStreamNonBlocking));
        P->own_stream = true;
    }
    CK(cudaStreamCreateWithFlags(&P->copy, cudaStreamNonBlocking));
    P->ev_num.resize(P->ring);
    P->ev_d2h.resize(P->ring);
    for (int r = 0; r < P->ring; ++r) {
        CK(cudaEventCreateWithFlags(&P->ev_num[r], cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&P->ev_d2h[r], cudaEventDisableTiming));
    }
    CK(cudaEventCreateWithFlags(&P->ev_ready, cudaEventDisableTiming));
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

    EvSet pe(P->profile, 16);
    if (P->profile) CK(cudaEventRecord(pe.ev[0], s));

    // S0 residency: B
    if (Bh->where == SPGEMM_DEVICE) {
        P->B = DevCSR{Bh->row_ptr, Bh->col_idx, Bh->values, Bh->nrows, Bh->ncols};
    } else {
        int64_t *rp = P->alloc<int64_t>(Bh->nrows + 1, "B.row_ptr");
        int32_t *c = P->alloc<int32_t>(Bh->nnz, "B.col_idx");
        double *v = P->alloc<double>(Bh->nnz, "B.values");
        CK(cudaMemcpyAsync(rp, Bh->row_ptr, sizeof(int64_t) * (Bh->nrows + 1), cudaMemcpyHostToDevice, s));
        if (Bh->nnz) {
            CK(cudaMemcpyAsync(c, Bh->col_idx, sizeof(int32_t) * Bh->nnz, cudaMemcpyHostToDevice, s));
            CK(cudaMemcpyAsync(v, Bh->values, sizeof(double) * Bh->nnz, cudaMemcpyHostToDevice, s));
        }
        P->B = DevCSR{rp, c, v, Bh->nrows, Bh->ncols};
    }
    // S0 residency + S1 row panel: A
    if (Ah->where == SPGEMM_DEVICE) {
        P->A = DevCSR{Ah->row_ptr + rb, Ah->col_idx, Ah->values, P->R, Ah->ncols};
        P->nnzA = -1;  // unknown without a read; only used for statistics
    } else {
        const bool alias = Bh->where == SPGEMM_HOST && Ah->row_ptr == Bh->row_ptr && Ah->col_idx == Bh->col_idx &&
                           Ah->values == Bh->values && Ah->nrows == Bh->nrows && Ah->ncols == Bh->ncols;
        const int64_t p0 = Ah->row_ptr[rb], p1 = Ah->row_ptr[re];
        P->nnzA = p1 - p0;
        if (alias) {
            P->A = DevCSR{P->B.rp + rb, P->B.col, P->B.val, P->R, Ah->ncols};
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
    P->group = choose_group(P->B, P->nnzB);

    // per-row arrays (24 B/row + 8) and control blocks
    const int64_t R = P->R;
    P->u = P->alloc<int64_t>(R, "u");
    P->crp = P->alloc<int64_t>(R + 1, "C.row_ptr");
    P->listB = P->alloc<int32_t>(R, "listB");
    P->listG = P->alloc<int32_t>(R, "listG");
    P->ctl = P->alloc<Ctl>(2, "ctl");
    P->tmp = P->alloc<int64_t>(2 * ((R + 1 + SCAN_TILE - 1) / SCAN_TILE) + 64, "scan scratch");
    CK(cudaMemsetAsync(P->ctl, 0, 2 * sizeof(Ctl), s));

    if (opts.validate) {
        launch_validate(P->A, P->ctl, s);
        launch_validate(P->B, P->ctl, s);
        CKL("validate");
    }

    // S2 count
    if (P->profile) CK(cudaEventRecord(pe.ev[1], s));
    launch_count(P->A, P->B, P->u, P->ctl, s);
    CKL("count");
    if (P->profile) CK(cudaEventRecord(pe.ev[2], s));
    Ctl hc;
    CK(cudaMemcpyAsync(&hc, P->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (hc.err & 2u) fail(SPGEMM_ERR_INVALID_ARGUMENT, "input validation failed (unsorted/duplicate/out-of-range col_idx or bad row_ptr)");
    P->products = (int64_t)hc.sum_u;
    P->max_u = (int64_t)hc.max_u;
    P->max_bound = (int64_t)hc.max_bound;

    // G-tier scratch, sized only if a row can exceed the CTA tier
    const int64_t nwords = (P->ncols + 31) / 32;
    if (P->max_bound > CAPB_NUM) {
        const bool num = true;  // numeric may need it: nnz_i <= min(u_i, ncols)
        P->gstride_bits = (nwords + 63) & ~int64_t(63);
        P->gstride_vals = num ? ((P->ncols + 31) & ~int64_t(31)) : 0;
        const size_t per = size_t(P->gstride_bits) * 4 + size_t(P->gstride_vals) * 8;
        const size_t ring_min = size_t(P->ring) * size_t(std::min<int64_t>(P->max_bound, P->products)) * 12 + 4096;
        size_t freeb = P->arena_bytes > P->used ? P->arena_bytes - P->used : 0;
        size_t avail = freeb > ring_min ? freeb - ring_min : 0;
        int64_t nb = std::min<int64_t>(P->num_sms, int64_t((avail / 4) / (per ? per : 1)));
        if (nb < 1) nb = int64_t(avail / (per ? per : 1)) >= 1 ? 1 : 0;
        if (nb < 1) fail(SPGEMM_ERR_BUDGET, "budget cannot hold one dense accumulator for the longest row");
        P->gblocks = (int)nb;
        P->gbits = P->alloc<uint32_t>(P->gstride_bits * nb, "G bitmap");
        P->gvals = P->alloc<double>(std::max<int64_t>(P->gstride_vals * nb, 1), "G values");
        CK(cudaMemsetAsync(P->gbits, 0, size_t(P->gstride_bits) * nb * 4, s));
        CK(cudaMemsetAsync(P->gvals, 0, size_t(P->gstride_vals) * nb * 8, s));
    }

    // S3+S4 symbolic, S5 scan
    CK(cudaMemsetAsync(P->crp + R, 0, sizeof(int64_t), s));
    SymArgs sa{P->A, P->B, P->u, P->crp, P->listB, P->listG, P->ctl, P->gbits, P->gstride_bits, P->gblocks, P->group};
    if (P->profile) CK(cudaEventRecord(pe.ev[3], s));
    launch_symbolic(sa, P->num_sms, s, P->profile ? pe.ptr() + 4 : nullptr);
    CKL("symbolic");
    if (P->profile) CK(cudaEventRecord(pe.ev[8], s));
    launch_scan(P->crp, R, 0, P->tmp, s);
    CKL("scan");
    if (P->profile) CK(cudaEventRecord(pe.ev[9], s));
    int64_t total = 0;
    CK(cudaMemcpyAsync(&hc, P->ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(&total, P->crp + R, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    P->nnz = total;
    P->max_nnz = (int64_t)hc.max_nnz;
    P->rows_w = (int64_t)hc.rows_w;
    P->rows_b = (int64_t)hc.rows_b;
    P->rows_g = (int64_t)hc.rows_g;

    // S10 ring + chunk cut.  Each ring slot holds `cap` nonzeros (val fp64 + col int32).
    const size_t freeb = P->arena_bytes > P->used + 4096 ? P->arena_bytes - P->used - 4096 : 0;
    size_t slot = (freeb / P->ring) & ~size_t(255);
    int64_t cap = int64_t(slot / 12) & ~int64_t(63);
    if (opts.chunk_nnz > 0) cap = std::min<int64_t>(cap, std::max<int64_t>(opts.chunk_nnz, P->max_nnz));
    if (total > 0 && cap < std::max<int64_t>(P->max_nnz, 1))
        fail(SPGEMM_ERR_BUDGET, "ring buffer of " + std::to_string(cap) + " nonzeros cannot hold the longest C row (" +
                                    std::to_string(P->max_nnz) + ")");
    cap = std::max<int64_t>(std::min<int64_t>(cap, std::max<int64_t>(total, 1)), std::max<int64_t>(P->max_nnz, 1));
    P->cap = cap;
    int64_t capp = std::max<int64_t>(1, cap - P->max_nnz);
    int64_t minc = opts.min_chunks;
    if (minc <= 0) minc = std::min<int64_t>(64, std::max<int64_t>(1, total * 12 / (128ll << 20)));
    if (minc > 1) capp = std::min<int64_t>(capp, std::max<int64_t>(1, (total + minc - 1) / minc));
    if (opts.chunk_nnz > 0) capp = std::min<int64_t>(capp, std::max<int64_t>(1, opts.chunk_nnz - P->max_nnz));
    capp = std::max<int64_t>(capp, 1);

    P->chunk_rows.clear();
    P->chunk_offs.clear();
    if (total > 0) {
        const int64_t nids = total / capp + 1;
        // temporary arrays at the start of the (not yet used) ring region
        const size_t save = P->used;
        int64_t *bounds = P->alloc<int64_t>(nids + 1, "chunk bounds");
        int64_t *offs = P->alloc<int64_t>(nids + 1, "chunk offsets");
        launch_cut(P->crp, R, capp, bounds, nids, s);
        launch_gather(P->crp, bounds, nids + 1, offs, s);
        CKL("cut");
        std::vector<int64_t> hb(nids + 1), ho(nids + 1);
        CK(cudaMemcpyAsync(hb.data(), bounds, sizeof(int64_t) * (nids + 1), cudaMemcpyDeviceToHost, s));
        CK(cudaMemcpyAsync(ho.data(), offs, sizeof(int64_t) * (nids + 1), cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        P->used = save;
        // chunk boundaries = the distinct bounds (an id whose rows are empty repeats a bound)
        P->chunk_rows.push_back(hb[0]);
        P->chunk_offs.push_back(ho[0]);
        for (int64_t c = 1; c <= nids; ++c) {
            if (hb[c] == P->chunk_rows.back()) continue;
            if (ho[c] - P->chunk_offs.back() > cap) fail(SPGEMM_ERR_STATE, "internal: chunk exceeds the ring capacity");
            P->chunk_rows.push_back(hb[c]);
            P->chunk_offs.push_back(ho[c]);
        }
        if (P->chunk_rows.front() != 0 || P->chunk_rows.back() != R)
            fail(SPGEMM_ERR_STATE, "internal: chunk bounds do not cover the rows");
    }

    // ring buffers
    P->ring_col.resize(P->ring);
    P->ring_val.resize(P->ring);
    if (total > 0) {
        for (int r = 0; r < P->ring; ++r) {
            P->ring_val[r] = P->alloc<double>(cap, "ring values");
            P->ring_col[r] = P->alloc<int32_t>(cap, "ring col_idx");
        }
        P->ring_bytes = size_t(P->ring) * size_t(cap) * 12;
    }
    if (P->profile) {
        P->stats.clear();
        P->add_stat("count", elapsed(pe.ev[1], pe.ev[2]), 0);
        P->add_stat("sym_w", elapsed(pe.ev[4], pe.ev[5]), 0);
        P->add_stat("sym_b", elapsed(pe.ev[5], pe.ev[6]), 0);
        P->add_stat("sym_g", elapsed(pe.ev[6], pe.ev[7]), 0);
        P->add_stat("scan", elapsed(pe.ev[8], pe.ev[9]), 0);
        P->add_stat("plan_total", elapsed(pe.ev[0], pe.ev[9]), 0);
    }
}

int64_t num_chunks(const spgemm_plan_s *P) {
    return P->chunk_rows.empty() ? 0 : int64_t(P->chunk_rows.size()) - 1;
}

// Enqueue the numeric pass of chunk c into ring slot b on the compute stream.
void enqueue_numeric(spgemm_plan_s *P, int64_t c, int b, cudaEvent_t *ev) {
    NumArgs na{P->A,          P->B,           P->crp,     P->chunk_rows[c], P->chunk_rows[c + 1],
               P->ring_col[b], P->ring_val[b], P->listB,   P->listG,         P->ctl + 1,
               P->gbits,      P->gvals,       P->gstride_bits, P->gstride_vals, P->gblocks,
               P->group};
    launch_numeric(na, P->num_sms, P->stream, ev);
    CKL("numeric");
}

void apply_base(spgemm_plan_s *P) {
    if (P->base_wanted != P->base_applied) {
        launch_add(P->crp, P->R, P->base_wanted - P->base_applied, P->stream);
        CKL("row_ptr base");
        P->base_applied = P->base_wanted;
    }
}

void check_numeric_errors(spgemm_plan_s *P) {
    unsigned err = 0;
    CK(cudaMemcpyAsync(&err, &P->ctl[1].err, sizeof(unsigned), cudaMemcpyDeviceToHost, P->stream));
    CK(cudaStreamSynchronize(P->stream));
    if (err) fail(SPGEMM_ERR_STATE, "internal: numeric pass produced a row whose nnz differs from the symbolic pass");
}

// The pipeline: numeric(c) on the compute stream into slot c % ring, D2H(c) on the copy stream.
void do_execute(spgemm_plan_s *P, int64_t *rp_out, int32_t *col_out, double *val_out) {
    if (P->failed) fail(SPGEMM_ERR_STATE, "plan is in a failed state");
    DeviceGuard g(P->device);
    const int64_t nch = num_chunks(P);
    if (P->nnz > 0 && (!col_out || !val_out)) fail(SPGEMM_ERR_INVALID_ARGUMENT, "col_idx/values output is NULL");
    apply_base(P);
    CK(cudaEventRecord(P->ev_ready, P->stream));
    CK(cudaStreamWaitEvent(P->copy, P->ev_ready, 0));
    const int per = 5;
    EvSet pe(P->profile, int(nch) * per + 4);
    if (P->profile) CK(cudaEventRecord(pe.ev[nch * per], P->copy));
    if (rp_out) CK(cudaMemcpyAsync(rp_out, P->crp, sizeof(int64_t) * (P->R + 1), cudaMemcpyDeviceToHost, P->copy));
    const int64_t base0 = P->chunk_offs.empty() ? 0 : P->chunk_offs[0];
    for (int64_t c = 0; c < nch; ++c) {
        const int b = int(c % P->ring);
        if (c >= P->ring) CK(cudaStreamWaitEvent(P->stream, P->ev_d2h[b], 0));
        enqueue_numeric(P, c, b, P->profile ? pe.ptr() + c * per : nullptr);
        CK(cudaEventRecord(P->ev_num[b], P->stream));
        CK(cudaStreamWaitEvent(P->copy, P->ev_num[b], 0));
        const int64_t o = P->chunk_offs[c] - base0, n = P->chunk_offs[c + 1] - P->chunk_offs[c];
        if (P->profile) CK(cudaEventRecord(pe.ev[c * per + 4], P->copy));
        if (n > 0) {
            CK(cudaMemcpyAsync(col_out + o, P->ring_col[b], sizeof(int32_t) * n, cudaMemcpyDeviceToHost, P->copy));
            CK(cudaMemcpyAsync(val_out + o, P->ring_val[b], sizeof(double) * n, cudaMemcpyDeviceToHost, P->copy));
        }
        CK(cudaEventRecord(P->ev_d2h[b], P->copy));
        if (P->profile && c + 1 == nch) CK(cudaEventRecord(pe.ev[nch * per + 1], P->copy));
    }
    if (P->profile && nch == 0) CK(cudaEventRecord(pe.ev[nch * per + 1], P->copy));
    CK(cudaStreamSynchronize(P->copy));
    check_numeric_errors(P);
    if (P->profile) {
        for (const char *n : {"num_w", "num_b", "num_g", "d2h", "execute_total"}) {
            for (auto &s : P->stats)
                if (s.name == n) s = Stat{n, 0, 0, 0};
        }
        for (int64_t c = 0; c < nch; ++c) {
            cudaEvent_t *e = pe.ptr() + c * per;
            P->add_stat("num_w", elapsed(e[0], e[1]), 0);
            P->add_stat("num_b", elapsed(e[1], e[2]), 0);
            P->add_stat("num_g", elapsed(e[2], e[3]), 0);
            // d2h: from the copy stream's start of this chunk's copy to the next record on it
            cudaEvent_t end = (c + 1 < nch) ? pe.ev[(c + 1) * per + 4] : pe.ev[nch * per + 1];
            P->add_stat("d2h_span", elapsed(e[4], end), double(P->chunk_offs[c + 1] - P->chunk_offs[c]) * 12);
        }
        P->add_stat("execute_total", elapsed(pe.ev[nch * per], pe.ev[nch * per + 1]), double(P->nnz) * 12 + 8.0 * (P->R + 1));
    }
}

void do_execute_stream(spgemm_plan_s *P, spgemm_chunk_cb cb, void *user) {
    if (P->failed) fail(SPGEMM_ERR_STATE, "plan is in a failed state");
    if (!cb) fail(SPGEMM_ERR_INVALID_ARGUMENT, "callback is NULL");
    DeviceGuard g(P->device);
    const int64_t nch = num_chunks(P);
    apply_base(P);
    int64_t maxn = 0, maxr = 0;
    for (int64_t c = 0; c < nch; ++c) {
        maxn = std::max(maxn, P->chunk_offs[c + 1] - P->chunk_offs[c]);
        maxr = std::max(maxr, P->chunk_rows[c + 1] - P->chunk_rows[c]);
    }
    const int ring = P->ring;
    std::vector<void *> stage(ring, nullptr);
    struct Release {
        std::vector<void *> &v;
        ~Release() {
            for (auto p : v) pin_release(p);
        }
    } rel{stage};
    const size_t per_slot = size_t(maxn) * 12 + size_t(maxr + 1) * 8 + 1024;
    for (int r = 0; r < ring; ++r) stage[r] = pin_acquire(per_slot);
    auto slot_val = [&](int b) { return reinterpret_cast<double *>(stage[b]); };
    auto slot_col = [&](int b) { return reinterpret_cast<int32_t *>((char *)stage[b] + size_t(maxn) * 8); };
    auto slot_rp = [&](int b) {
        return reinterpret_cast<int64_t *>((char *)stage[b] + ((size_t(maxn) * 12 + 7) & ~size_t(7)));
    };
    CK(cudaEventRecord(P->ev_ready, P->stream));
    CK(cudaStreamWaitEvent(P->copy, P->ev_ready, 0));
    auto enqueue = [&](int64_t c) {
        const int b = int(c % ring);
        enqueue_numeric(P, c, b, nullptr);
        CK(cudaEventRecord(P->ev_num[b], P->stream));
        CK(cudaStreamWaitEvent(P->copy, P->ev_num[b], 0));
        const int64_t n = P->chunk_offs[c + 1] - P->chunk_offs[c];
        const int64_t r0 = P->chunk_rows[c], r1 = P->chunk_rows[c + 1];
        CK(cudaMemcpyAsync(slot_rp(b), P->crp + r0, sizeof(int64_t) * (r1 - r0 + 1), cudaMemcpyDeviceToHost, P->copy));
        if (n > 0) {
            CK(cudaMemcpyAsync(slot_col(b), P->ring_col[b], sizeof(int32_t) * n, cudaMemcpyDeviceToHost, P->copy));
            CK(cudaMemcpyAsync(slot_val(b), P->ring_val[b], sizeof(double) * n, cudaMemcpyDeviceToHost, P->copy));
        }
        CK(cudaEventRecord(P->ev_d2h[b], P->copy));
    };
    // keep `ring` chunks in flight; the host consumes chunk c while chunks c+1.. run
    int64_t issued = 0;
    for (; issued < std::min<int64_t>(nch, ring); ++issued) enqueue(issued);
    for (int64_t c = 0; c < nch; ++c) {
        const int b = int(c % ring);
        CK(cudaEventSynchronize(P->ev_d2h[b]));
        int64_t *rp = slot_rp(b);
        const int64_t r0 = P->chunk_rows[c], r1 = P->chunk_rows[c + 1];
        const int64_t first = rp[0];
        for (int64_t k = 0; k <= r1 - r0; ++k) rp[k] -= first;
        const int rc = cb(user, P->row_begin + r0, P->row_begin + r1, rp, slot_col(b), slot_val(b), rp[r1 - r0]);
        if (rc != 0) {
            CK(cudaStreamSynchronize(P->copy));
            fail(SPGEMM_ERR_CALLBACK, "chunk sink returned " + std::to_string(rc));
        }
        if (issued < nch) enqueue(issued++);
    }
    CK(cudaStreamSynchronize(P->copy));
    check_numeric_errors(P);
}

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
    spgemm_status st = guarded([&] {
        P = new spgemm_plan_s();
        do_plan(A, B, budget, opts, P);
    });
    if (prev >= 0) cudaSetDevice(prev);
    if (st != SPGEMM_OK) {
        delete P;
        return st;
    }
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
    info->max_row_nnz = P->max_nnz;
    info->max_row_products = P->max_u;
    info->num_chunks = (int32_t)num_chunks(P);
    info->ring = P->ring;
    info->chunk_capacity = P->cap;
    info->arena_bytes = (int64_t)P->arena_bytes;
    info->arena_used = (int64_t)P->used;
    info->ring_bytes = (int64_t)P->ring_bytes;
    info->rows_warp = P->rows_w;
    info->rows_block = P->rows_b;
    info->rows_global = P->rows_g;
    return SPGEMM_OK;
}

spgemm_status spgemm_plan_chunks(spgemm_plan_t P, int64_t *rows, int64_t *offs) {
    if (!P || !rows || !offs) {
        g_err = "NULL argument";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    const int64_t base0 = P->chunk_offs.empty() ? 0 : P->chunk_offs[0];
    if (P->chunk_rows.empty()) {
        rows[0] = 0;
        offs[0] = 0;
        return SPGEMM_OK;
    }
    for (size_t k = 0; k < P->chunk_rows.size(); ++k) {
        rows[k] = P->chunk_rows[k];
        offs[k] = P->chunk_offs[k] - base0;
    }
    return SPGEMM_OK;
}

spgemm_status spgemm_execute_into(spgemm_plan_t P, int64_t *row_ptr, int32_t *col_idx, double *values) {
    if (!P) {
        g_err = "plan is NULL";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    spgemm_status st = guarded([&] { do_execute(P, row_ptr, col_idx, values); });
    if (st != SPGEMM_OK && st != SPGEMM_ERR_INVALID_ARGUMENT) P->failed = true;
    return st;
}

spgemm_status spgemm_execute(spgemm_plan_t P, spgemm_csr_out *C) {
    if (!P || !C) {
        g_err = "NULL argument";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    spgemm_status st = guarded([&] {
        DeviceGuard g(P->device);
        if (!P->h_rp) {
            if (cudaHostAlloc(&P->h_rp, sizeof(int64_t) * (P->R + 1), 0) != cudaSuccess ||
                cudaHostAlloc(&P->h_col, sizeof(int32_t) * std::max<int64_t>(P->nnz, 1), 0) != cudaSuccess ||
                cudaHostAlloc(&P->h_val, sizeof(double) * std::max<int64_t>(P->nnz, 1), 0) != cudaSuccess) {
                cudaGetLastError();
                fail(SPGEMM_ERR_HOST_ALLOC, "pinned allocation of the output failed");
            }
        }
        do_execute(P, P->h_rp, P->h_col, P->h_val);
        C->nrows = P->R;
        C->ncols = P->ncols;
        C->nnz = P->nnz;
        C->row_ptr = P->h_rp;
        C->col_idx = P->h_col;
        C->values = P->h_val;
    });
    if (st != SPGEMM_OK && st != SPGEMM_ERR_INVALID_ARGUMENT && st != SPGEMM_ERR_HOST_ALLOC) P->failed = true;
    return st;
}

spgemm_status spgemm_execute_stream(spgemm_plan_t P, spgemm_chunk_cb cb, void *user) {
    if (!P) {
        g_err = "plan is NULL";
        return SPGEMM_ERR_INVALID_ARGUMENT;
    }
    spgemm_status st = guarded([&] { do_execute_stream(P, cb, user); });
    if (st == SPGEMM_ERR_CUDA || st == SPGEMM_ERR_STATE) P->failed = true;
    return st;
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
    spgemm_plan_t P = nullptr;
    spgemm_status st = spgemm_plan(A, B, budget, opts, &P);
    if (st != SPGEMM_OK) return st;
    if (nnz_out) *nnz_out = P->nnz;
    if (P->nnz > cap) {
        g_err = "output capacity " + std::to_string(cap) + " < nnz(C) = " + std::to_string(P->nnz);
        spgemm_free(P);
        return SPGEMM_ERR_CAPACITY;
    }
    st = spgemm_execute_into(P, row_ptr, col_idx, values);
    spgemm_free(P);
    return st;
}

spgemm_status spgemm_stats(spgemm_plan_t P, spgemm_kernel_stat *out, int32_t max, int32_t *n) {
    if (!P || !n) {
        g_err = "NULL argument";
        return SPGEMM_ERR_INVALID_ARGUMENT;
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

void spgemm_free(spgemm_plan_t P) {
    if (!P) return;
    int prev = -1;
    cudaGetDevice(&prev);
    cudaSetDevice(P->device);
    delete P;
    if (prev >= 0) cudaSetDevice(prev);
}

void spgemm_release_cache(void) {
    std::lock_guard<std::mutex> lk(g_pin_mu);
    std::vector<PinnedBlock> keep;
    for (auto &b : g_pins) {
        if (b.used) keep.push_back(b);
        else cudaFreeHost(b.p);
    }
    g_pins.swap(keep);
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
