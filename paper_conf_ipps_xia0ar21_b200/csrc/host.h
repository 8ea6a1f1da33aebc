// host.h -- host-side internals shared by api.cu (ABI, planner, chunk pipeline) and panels.cu
// (column-panel mode): error handling, pinned-memory and CUDA-object pools, the plan object.
// Not part of the public ABI (include/spgemm.h).
#pragma once
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include <mutex>
#include <string>
#include <vector>

#include "../../include/spgemm.h"
#include "internal.h"

// NVTX range for the host side of the pipeline (plan, execute, each unit's enqueue, the wait for a
// unit's total, every sink callback), so that an Nsight Systems timeline shows the host thread next
// to the compute / analysis / copy streams.  nvtx3 is header-only: without an attached tool each
// push/pop is a no-op call.
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange &) = delete;
    NvtxRange &operator=(const NvtxRange &) = delete;
};

namespace spgh {
using namespace spg;

// spare elements per ring slot for the alignment pad of an output chunk (run_pipeline)
constexpr int64_t RING_PAD = 32;

extern thread_local std::string g_err;

struct Err {
    spgemm_status st;
    std::string msg;
};

[[noreturn]] inline void fail(spgemm_status st, const std::string &msg) { throw Err{st, msg}; }

inline void ck(cudaError_t e, const char *what) {
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

// pinned host staging cache (api.cu): blocks are reused across plans until spgemm_release_cache
void *pin_acquire(size_t n);
void pin_release(void *p);

struct Stat {
    std::string name;
    int launches = 0;
    double ms = 0, bytes = 0;
};

double elapsed(cudaEvent_t a, cudaEvent_t b);  // ms, 0 on error

// ------------------------------------------------ reusable CUDA objects (per device, pooled)
// Streams and events are created on first use and handed from plan to plan: creating and
// destroying ~100 events and 3 streams per multiply cost ~1-2 ms of host time per step, serial
// with the pipeline.  A plan takes one Res at spgemm_plan and returns it at spgemm_free.
struct Res {
    int device = -1;
    bool used = false;
    cudaStream_t copy = nullptr, astream = nullptr, hstream = nullptr, own = nullptr;
    enum { PLAIN = 0, TIMING = 1, PIECE = 2 };
    std::vector<cudaEvent_t> pool[3];
    // n events of pool `kind` starting at index `from`; grows the pool as needed
    std::vector<cudaEvent_t> events(int kind, size_t from, size_t n) {
        auto &v = pool[kind];
        while (v.size() < from + n) {
            cudaEvent_t e;
            CK(cudaEventCreateWithFlags(&e, kind == TIMING ? cudaEventDefault : cudaEventDisableTiming));
            v.push_back(e);
        }
        return std::vector<cudaEvent_t>(v.begin() + from, v.begin() + from + n);
    }
    cudaStream_t stream(cudaStream_t &slot) {
        if (!slot) CK(cudaStreamCreateWithFlags(&slot, cudaStreamNonBlocking));
        return slot;
    }
    void destroy() {
        for (auto &v : pool)
            for (auto e : v) cudaEventDestroy(e);
        for (auto st : {copy, astream, hstream, own})
            if (st) cudaStreamDestroy(st);
    }
};
Res *res_acquire(int device);
void res_release(Res *r);

struct EvSet {  // timing events (profile mode only), borrowed from the plan's Res
    std::vector<cudaEvent_t> ev;
    EvSet(bool on, Res *r, size_t from, size_t n) {
        if (on) ev = r->events(Res::TIMING, from, n);
    }
    cudaEvent_t *at(size_t k) { return ev.empty() ? nullptr : ev.data() + k; }
    void rec(size_t k, cudaStream_t s) {
        if (!ev.empty()) CK(cudaEventRecord(ev[k], s));
    }
};


struct Sink {
    spgemm_chunk_cb cb = nullptr;
    void *user = nullptr;
};

}  // namespace spgh

using namespace spgh;

struct Panels;
void delete_panels(Panels *);

struct spgemm_plan_s {
    int device = 0, num_sms = 148;
    Res *res = nullptr;  // pooled streams and events
    cudaStream_t stream = nullptr, copy = nullptr;
    std::vector<cudaEvent_t> ev_num, ev_d2h, ev_tot;
    cudaEvent_t ev_ready = nullptr;

    char *arena = nullptr;
    size_t arena_bytes = 0, used = 0;
    bool own_arena = false;

    DevCSR A{}, B{};
    int64_t R = 0, ncols = 0, nnzA = 0, nnzB = 0, row_begin = 0;
    int group = 32;
    bool fused = false;

    int64_t *bnd = nullptr, *crp = nullptr, *tmp = nullptr;
    int32_t *nnzr = nullptr, *listB = nullptr, *listG = nullptr;  // symbolic long-row lists
    int32_t *listBn = nullptr, *listGn = nullptr;                  // numeric long-row lists
    int32_t *listM = nullptr, *listMn = nullptr;                   // medium-tier lists (sym, num)
    cudaStream_t astream = nullptr;  // fused plans: symbolic passes run here, ahead of the numeric
    cudaStream_t hstream = nullptr;         // host B: value pieces H2D
    std::vector<cudaEvent_t> ev_piece;      // one per value piece, in upload order
    std::vector<int64_t> bpiece_rows;       // B row boundaries of the pieces
    std::vector<int> chunk_wait;            // per chunk: last piece its numeric pass reads (-1: none)
    bool a_alias = false;
    // host cut (fused C = A x A with host operands and short rows): chunks cut on the host from
    // A.row_ptr; each chunk's count pass runs inside execute after the pieces it reads landed
    bool host_cut = false;
    std::vector<cudaEvent_t> ev_col;        // one per structure piece (row_ptr + col_idx), upload order
    const int64_t *hA_rp = nullptr;         // borrowed host A (the plan's rows start at hA_rp[0])
    const int32_t *hA_col = nullptr;
    Ctl *ctl = nullptr;  // [0] count / symbolic passes, [1] numeric passes

    uint32_t *gbits = nullptr, *gbits_sym = nullptr;
    double *gvals = nullptr;
    unsigned long long *gcnt = nullptr;  // split dense rows: counters (2 x gblocks x (KG_SWEEP + 1))
    int32_t *cur_sym = nullptr, *cur_num = nullptr;  // pieced CTA tier: cursor scratch
    int64_t curstride = 0, max_deg = 0;
    int bblocks_sym = 0, bblocks_num = 0;
    int64_t gstride_bits = 0, gstride_vals = 0;
    int gblocks = 0;

    int ring = 2;
    int64_t cap = 0;
    size_t ring_bytes = 0;
    std::vector<int32_t *> ring_col;
    std::vector<double *> ring_val;

    std::vector<int64_t> chunk_rows;  // num_chunks + 1 row boundaries
    std::vector<int64_t> chunk_offs;  // num_chunks + 1 offsets relative to the slice (known after
                                      // plan for two-phase plans, after an execution for fused)
    int64_t nnz = -1, products = 0, max_nnz = 0, max_u = 0, max_bound = 0, sum_bound = 0;
    int64_t rows_w = 0, rows_b = 0, rows_g = 0, rows_m = 0;
    int64_t num_groups = 0;  // output chunks (copies) of the last execution
    int64_t panel_units = 0; // column-panel plans: numeric units (chunks C[i][j]) over all panels
    std::vector<int64_t> unit_order;  // order = 1: units by decreasing flops (empty: row order)
    int64_t base_applied = 0, base_wanted = 0;
    int64_t *h_small = nullptr;  // pinned + mapped: [0] base; chunk j: [1 + 2j] end offset,
    int64_t *d_small = nullptr;  //   [2 + 2j] max row nnz (fused; written by k_publish)
    std::vector<int64_t> chunk_maxb;  // fused: max row bound per chunk
    std::vector<int> tiers_sym, tiers_num;  // per unit: tier bits launched (profile statistics)

    int64_t *h_rp = nullptr;
    int32_t *h_col = nullptr;
    double *h_val = nullptr;

    bool profile = false;
    struct Pending {  // profile mode: events of the last execution, evaluated on demand
        bool active = false;
        std::vector<cudaEvent_t> ev;
        int64_t nch = 0, total = 0;
        size_t per = 0;
        bool overflow = false;
        std::vector<int64_t> offs;
        std::vector<int64_t> group_last;  // last unit of every output chunk (copy events live there)
        std::vector<int64_t> group_nnz;   // nonzeros of every output chunk
    } pend;
    std::vector<Stat> stats;
    std::vector<double> timeline;  // profile: 6 times (ms) per chunk of the last execution
    bool failed = false;
    struct Panels *pan = nullptr;  // column-panel mode (B cut into column panels), else NULL
    int col_panels = 1;            // panels of B (1: B used whole)

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
    void clear_stats(std::initializer_list<const char *> names) {
        std::vector<Stat> keep;
        for (auto &s : stats) {
            bool drop = false;
            for (auto n : names) drop |= s.name == n;
            if (!drop) keep.push_back(s);
        }
        stats.swap(keep);
    }
    int64_t num_chunks() const { return chunk_rows.empty() ? 0 : int64_t(chunk_rows.size()) - 1; }
    ~spgemm_plan_s() {
        for (auto st : {stream, copy, astream, hstream})
            if (st) cudaStreamSynchronize(st);
        res_release(res);
        delete_panels(pan);
        if (own_arena && arena) cudaFree(arena);
        if (h_rp) cudaFreeHost(h_rp);
        if (h_col) cudaFreeHost(h_col);
        if (h_val) cudaFreeHost(h_val);
        pin_release(h_small);
    }
};

namespace spgh {
void check_csr(const spgemm_csr *M, const char *name);
void check_rows_host(const spgemm_csr *M, const char *name);
// column-panel mode (panels.cu)
void do_panel_plan(const spgemm_csr *Ah, const spgemm_csr *Bh, size_t budget, const spgemm_opts *o, spgemm_plan_s *P);
int64_t run_panels(spgemm_plan_s *P, int64_t *rp_out, int32_t *col_out, double *val_out, int64_t capacity,
                   const Sink *sink, bool *overflow);
}  // namespace spgh
