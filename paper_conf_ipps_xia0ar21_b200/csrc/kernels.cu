// kernels.cu -- sm_100a kernels of the out-of-core chunked SpGEMM hot path.
//
// Steps (DESIGN.md §8 rows; PAPER.md anchors):
//   S2 count     k_count        products per row ("row analysis", §III-B; Alg. 1 line-4 trip count)
//   S3 tiering   inside k_sym_w / k_num_w: rows too long for a warp are appended to the CTA (B) or
//                dense-global (G) list on the device -- the paper's host-side row grouping after a
//                D2H (§III-B, §IV-B) is replaced by device-side lists, no transfer.
//   S4 symbolic  k_sym_w / k_sym_b / k_sym_g   (hash set of column ids -> nnz per row, §II-B)
//   S5 scan      k_scan_{reduce,top,apply}     (row offsets of C, §III-B)
//   S6 numeric   k_num_w / k_num_b / k_num_g   (hash / dense accumulation, §II-B, §III-B)
//   S7 sort      in the numeric kernels: in-place compaction + bitonic sort by column (§II-B)
//
// No tensor cores: this is not a dense contraction.  Hash tables live in shared memory (W, B
// tiers); the G tier is a dense bitmap + fp64 array over all columns in arena scratch (the
// "dense accumulation" of §II-B L107 / §III-B, used here for the longest rows).
#include <climits>
#include <cstddef>
#include <cstdio>
#include <cstdlib>

#include <atomic>
#include <type_traits>

#include "internal.h"

namespace spg {

static std::atomic<long long> g_launches{0};
long long kernel_launches() { return g_launches.load(); }
#define LAUNCHED(n) g_launches.fetch_add((n), std::memory_order_relaxed)

#define FULLMASK 0xffffffffu

// Device-side bounds checks of the checked build (libspgemm_b200_checked.so, -DSPGEMM_CHECKS;
// compute-sanitizer is not available on the GPU pool): a failed check prints its site and traps.
// In the product build they compile to nothing.
#ifdef SPGEMM_CHECKS
#define SPG_CHECK(cond)                                                                                   \
    do {                                                                                                  \
        if (!(cond)) {                                                                                    \
            printf("SPG_CHECK failed: %s (%s:%d) block %d thread %d\n", #cond, __FILE__, __LINE__,       \
                   (int)blockIdx.x, (int)threadIdx.x);                                                    \
            __trap();                                                                                     \
        }                                                                                                 \
    } while (0)
#else
#define SPG_CHECK(cond) \
    do {                \
    } while (0)
#endif
constexpr int32_t EMPTY = -1;

// Home slot of column c in a table of 2^lg slots: multiplicative (Fibonacci) hashing.  (A variant
// whose low 5 bits XOR-fold c's digits, so that a stencil row's columns fall in distinct shared
// memory banks, cut bank conflicts by 22% but cost 8 more instructions per probe; the W kernels
// are issue-bound, not LSU-bound, so it was slower -- profiles/r01/ncu_*_h1.md.)
__device__ __forceinline__ uint32_t hslot(int32_t c, int lg) {
    return ((uint32_t)c * 0x9E3779B1u) >> (32 - lg);
}

// log2 of the table size for a row with `bound` distinct keys: load factor <= 1/2, >= 32 slots.
// (At load 3/4 linear probing's unsuccessful searches average 8.5 probes and a warp waits for its
// slowest lane; with CR ~ 1 -- R-MAT, C3 -- nearly every product is an unsuccessful search.)
__device__ __forceinline__ int table_log2(int64_t bound, int maxlg) {
    const int64_t need = 2 * bound;
    if (need <= 32) return 5;
    return need >= (int64_t(1) << maxlg) ? maxlg : 64 - __clzll(need - 1);
}

// symbolic insert: returns 1 if `c` was not yet in the table
__device__ __forceinline__ int sym_insert(int32_t *keys, int32_t c, int lg) {
    const uint32_t mask = (1u << lg) - 1;
    uint32_t h = hslot(c, lg);
    volatile int32_t *vk = keys;
    while (true) {
        int32_t k = vk[h];
        if (k == c) return 0;
        if (k == EMPTY) {
            int32_t old = atomicCAS(&keys[h], EMPTY, c);
            if (old == EMPTY) return 1;
            if (old == c) return 0;
        }
        h = (h + 1) & mask;
    }
}

// numeric insert-or-add (Alg. 1 lines 6-10 with a hash map instead of a list)
__device__ __forceinline__ void num_insert(int32_t *keys, double *vals, int32_t c, double v, int lg) {
    const uint32_t mask = (1u << lg) - 1;
    uint32_t h = hslot(c, lg);
    volatile int32_t *vk = keys;
    while (true) {
        int32_t k = vk[h];
        if (k == c) break;
        if (k == EMPTY) {
            int32_t old = atomicCAS(&keys[h], EMPTY, c);
            if (old == EMPTY || old == c) break;
        }
        h = (h + 1) & mask;
    }
    atomicAdd(&vals[h], v);
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) v += __shfl_xor_sync(FULLMASK, v, d);
    return v;
}

// Dynamic row claim of the CTA tiers: the next index of the tier's list for the whole CTA (all
// threads call; two barriers).  Row costs are heavy-tailed on power-law inputs (a pieced row of
// 10^5 nonzeros next to rows of 10^3), so a static stride left CTAs idle behind the unlucky one
// (per-unit launches of the symbolic CTA tier took 1.8x the single-launch time on C3).
__device__ __forceinline__ unsigned cta_claim(unsigned *ctr, unsigned *s_idx) {
    __syncthreads();  // every thread has read the previous claim
    if (threadIdx.x == 0) *s_idx = atomicAdd(ctr, 1u);
    __syncthreads();
    return *s_idx;
}

// exclusive block scan of one int64 per thread; s has >= 33 entries; returns exclusive prefix,
// *total = block sum.  All threads must call.
template <int NT>
__device__ __forceinline__ int64_t block_excl_scan(int64_t v, int64_t *s, int64_t *total) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    int64_t x = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        int64_t t = __shfl_up_sync(FULLMASK, x, d);
        if (lane >= d) x += t;
    }
    if (lane == 31) s[wid] = x;
    __syncthreads();
    if (wid == 0) {
        int64_t w = lane < NT / 32 ? s[lane] : 0;
        int64_t y = w;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            int64_t t = __shfl_up_sync(FULLMASK, y, d);
            if (lane >= d) y += t;
        }
        if (lane < NT / 32) s[lane] = y - w;
        if (lane == 31) s[32] = y;
    }
    __syncthreads();
    int64_t r = x - v + s[wid];
    *total = s[32];
    __syncthreads();
    return r;
}

// ------------------------------------------------------------------ warp product iterator (W tier)
//
// Visits every intermediate product A_ik * B_kj of row i with one warp (Alg. 1 lines 3-5).
//  * A entries are fetched 32 at a time (one per lane) together with their B row bounds and staged
//    in the warp's shared-memory slot `st`, so the A.col -> B.rp dependency is paid once per 32
//    entries; a round then reads its entry with ONE broadcast LDS.128: the B row's start and length
//    packed in one word (start < 2^40, length < 2^24) next to the A value.  (Separate arrays of
//    column / value pointers, lengths and A values cost four LDS per round: 11 % of num_w's shared
//    wavefronts on C2, profiles/r02/; the LSU data pipe -- shared memory, shuffles, L1 -- is what
//    bounds these kernels.)
//  * Lanes form 32/G subgroups; subgroup g takes one B row per round and its lanes take G
//    consecutive entries of it (coalesced).  U rounds are loaded before any is consumed, so U
//    independent B-row loads are in flight per warp (latency, not bandwidth, bounds this loop).
//  * f(ok, col, value) is called once per round by every lane, followed by __syncwarp() when SYNC
//    (the numeric pass: a round's value updates must land before the next round's; the symbolic
//    pass only inserts keys with atomicCAS and needs no ordering between rounds).  With
//    G == 32 all active lanes of a round hold entries of ONE B row, i.e. distinct columns
//    (rows are sorted and unique), which lets the numeric pass update values without atomics.
constexpr int AST_LSH = 40;  // packed staged entry (numeric pass): B row start | length << 40
struct __align__(16) AStage {
    union {
        ulonglong2 e[32];  // numeric: .x = start of B row A.col[entry] | its length << 40, .y = A value
        struct {           // symbolic (issue-bound, not LSU-bound: no unpacking, two broadcast LDS)
            const int32_t *pc[32];
            int32_t len[32];
        } s;
    };
};
__device__ __forceinline__ void ast_unpack(const ulonglong2 &x, int64_t &bs, int32_t &len, double &a) {
    bs = (int64_t)(x.x & ((1ull << AST_LSH) - 1));
    len = (int32_t)(x.x >> AST_LSH);
    a = __longlong_as_double((long long)x.y);
}

template <int G, int U, bool VALS, bool SYNC, typename F>
__device__ __forceinline__ void warp_row_products(const DevCSR &A, const DevCSR &B, int64_t i, AStage *st, F &&f) {
    constexpr int R = 32 / G;  // B rows per round
    const int lane = threadIdx.x & 31;
    const int sub = lane / G, sl = lane % G;
    const int64_t as = A.rp[i], ae = A.rp[i + 1];
    for (int64_t pb = as; pb < ae; pb += 32) {
        const int64_t e = pb + lane;
        int64_t len = 0, bs = 0;
        double av = 0.0;
        if (e < ae) {
            const int32_t k = __ldg(&A.col[e]);
            bs = __ldg(&B.rp[k]);
            len = __ldg(&B.rp[k + 1]) - bs;
            if (VALS) av = __ldg(&A.val[e]);
        }
        // rows longer than a group need the remainder loop below (never on the stencils)
        const bool any_long = __any_sync(FULLMASK, len > G);
        __syncwarp();  // the previous batch's rounds have read their entries
        // lanes past the row's end stage empty rows
        if (VALS) {
            st->e[lane] = make_ulonglong2((unsigned long long)bs | ((unsigned long long)len << AST_LSH),
                                          (unsigned long long)__double_as_longlong(av));
        } else {
            st->s.pc[lane] = B.col + bs;
            st->s.len[lane] = (int32_t)len;
        }
        __syncwarp();
        const int nb = (int)(ae - pb < 32 ? ae - pb : 32);
        for (int t = 0; t < nb; t += R * U) {  // R * U divides 32, so src < 32
            int32_t c[U];
            double a[U], v[U];
            bool ok[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int src = t + u * R + sub;
                if (VALS) {
                    int64_t s0;
                    int32_t ln;
                    ast_unpack(st->e[src], s0, ln, a[u]);
                    ok[u] = sl < ln;
                    c[u] = ok[u] ? __ldg(B.col + s0 + sl) : 0;
                    v[u] = ok[u] ? __ldg(B.val + s0 + sl) : 0.0;
                } else {
                    ok[u] = sl < st->s.len[src];
                    c[u] = ok[u] ? __ldg(st->s.pc[src] + sl) : 0;
                }
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                f(ok[u], c[u], VALS ? a[u] * v[u] : 0.0);
                if (SYNC) __syncwarp();
            }
            if (any_long) {
#pragma unroll 1
                for (int u = 0; u < U; ++u) {
                    // remainder of B rows longer than G (uniform trip count across the warp)
                    const int src = t + u * R + sub;
                    int64_t s2 = 0;
                    int32_t ln2;
                    double a2 = 0.0;
                    if (VALS) {
                        ast_unpack(st->e[src], s2, ln2, a2);
                    } else {
                        s2 = st->s.pc[src] - B.col;
                        ln2 = st->s.len[src];
                    }
                    for (int o = G;; o += G) {
                        if (!__any_sync(FULLMASK, o < ln2)) break;
                        const int q = o + sl;
                        const bool okk = q < ln2;
                        const int32_t cc = okk ? __ldg(B.col + s2 + q) : 0;
                        const double vv = (VALS && okk) ? __ldg(B.val + s2 + q) : 0.0;
                        f(okk, cc, VALS ? a2 * vv : 0.0);
                        if (SYNC) __syncwarp();
                    }
                }
            }
        }
    }
}

// ------------------------------------------------------------------ CTA product iterator (B/G)
//
// Visits every product of row i with a whole CTA, load-balanced: A entries are taken PBATCH at a
// time, a block scan of their B-row segment lengths flattens the products, and thread t handles
// products t, t + NT, ...  (coalesced B loads), locating its A entry by binary search in shared
// memory.  One warp per A entry would leave the CTA waiting on the longest B row -- a hub row of a
// power-law graph holds thousands of entries.  seg(e, k, s0, e0, s, en) picks the segment [s, en)
// of B row k = [s0, e0) that entry e (its index within the row) contributes: the whole row, or
// one column piece of it (PieceSeg).
constexpr int PBATCH = 512;
template <int PB>
struct ProdSmemT {
    int64_t off[PB + 1];
    int64_t bs[PB];
    double a[PB];
    int64_t scan[40];
    unsigned next;  // next claim of 64 products (dynamic distribution over the warps)
};
using ProdSmem = ProdSmemT<PBATCH>;

struct WholeSeg {
    __device__ __forceinline__ void operator()(int, int32_t, int64_t s0, int64_t e0, int64_t &s, int64_t &en) const {
        s = s0;
        en = e0;
    }
};

// Column piece [.., hi) of every B row, resumed at the entry's cursor (offset within the B row
// of the first column not yet consumed by earlier pieces); the end of the segment -- the first
// column >= hi, by binary search -- is left in nxt[e] for the next piece (the paper's col_offset,
// P:L182).  cur / nxt live in this CTA's global scratch slot.
struct PieceSeg {
    const int32_t *bcol;
    const int32_t *cur;
    int32_t *nxt;
    int32_t hi;
    __device__ __forceinline__ void operator()(int e, int32_t, int64_t s0, int64_t e0, int64_t &s, int64_t &en) const {
        SPG_CHECK(cur[e] >= 0 && s0 + cur[e] <= e0);
        s = s0 + cur[e];
        int64_t lo = s, h = e0;
        if (lo < h) {
            // the row's last column is loaded next to the first midpoint (independent loads): in
            // the row's last piece -- and for every B row that ends before hi -- the search ends
            // there, instead of after log2(length) dependent loads
            const int64_t m = (lo + h) >> 1;
            const int32_t cl = __ldg(&bcol[h - 1]), cm = __ldg(&bcol[m]);
            if (cl < hi) {
                lo = h;
            } else {
                if (cm < hi) lo = m + 1;
                else h = m;
                h = min(h, e0 - 1);  // bcol[e0 - 1] >= hi
                while (lo < h) {
                    const int64_t m2 = (lo + h) >> 1;
                    if (__ldg(&bcol[m2]) < hi) lo = m2 + 1;
                    else h = m2;
                }
            }
        }
        en = lo;
        nxt[e] = (int32_t)(lo - s0);
    }
};

// f(col, value) or f(col, value, q) with q the product's index in the flattened sequence of the
// range (0 .. total-1, batch after batch).  Returns the total number of products (every thread).
template <int NT, bool VALS, int PB, typename SEG, typename F>
__device__ __forceinline__ int64_t range_products(const DevCSR &A, const DevCSR &B, int64_t as, int64_t ae,
                                                  ProdSmemT<PB> &sm, const SEG &seg, F &&f) {
    constexpr int PER = PB / NT;
    static_assert(PER * NT == PB, "batch must be a multiple of the CTA size");
    constexpr bool WITH_Q = std::is_invocable<F, int32_t, double, int64_t>::value;
    int64_t qbase = 0;
    for (int64_t pb = as; pb < ae; pb += PB) {
        const int nb = (int)(ae - pb < PB ? ae - pb : PB);
        int64_t lens[PER];
        int64_t sum = 0;
#pragma unroll
        for (int r = 0; r < PER; ++r) {
            const int e = threadIdx.x * PER + r;
            int64_t bs = 0, len = 0;
            double av = 0.0;
            if (e < nb) {
                const int32_t k = __ldg(&A.col[pb + e]);
                int64_t s, en;
                seg((int)(pb - as) + e, k, __ldg(&B.rp[k]), __ldg(&B.rp[k + 1]), s, en);
                bs = s;
                len = en - s;
                if (VALS) av = __ldg(&A.val[pb + e]);
            }
            if (e < PB) {
                sm.bs[e] = bs;
                if (VALS) sm.a[e] = av;
            }
            lens[r] = len;
            sum += len;
        }
        int64_t tot;
        int64_t run = block_excl_scan<NT>(sum, sm.scan, &tot);
#pragma unroll
        for (int r = 0; r < PER; ++r) {
            const int e = threadIdx.x * PER + r;
            if (e < nb) sm.off[e] = run;
            run += lens[r];
        }
        constexpr int NW = NT / 32;
        if (threadIdx.x == 0) {
            sm.off[nb] = tot;
            sm.next = NW;  // claims 0 .. NW-1 are the warps' first ones
        }
        __syncthreads();
        // Each warp claims 64 consecutive products at a time (two steps of 32: coalesced B loads)
        // from a shared counter, so a warp whose inserts probed longer takes fewer claims -- with a
        // static stride the warps left the batch up to a step apart and the barrier after it was
        // the top stall of the CTA kernels (14 % of num_b's and 24 % of sym_b's stall samples,
        // profiles/r02/NOTES.md).  Software-pipelined: the next claim and its gathers are issued
        // before the current products are consumed, so up to four B loads per lane are in flight
        // while the hash inserts run (a cp.async double buffer of the same gathers was slower).
        // Four groups of 8 lanes find the segments of the first and last product of each step;
        // every lane then searches only that window (usually 1-3 segments) instead of all nb A
        // entries of the batch.
        const int lane = threadIdx.x & 31;
        auto locate = [&](int64_t qb, int64_t (&pos)[2], double (&a)[2], bool (&ok)[2]) {
            // the four window ends (first / last product of each step) are found by four groups of
            // 8 lanes in parallel, an 8-ary search over off[0, nb) (3 levels for PB = 512) -- the
            // whole warp busy, instead of 4 lanes walking a 9-level binary search while 28 idle
            const int grp = lane >> 3, k = lane & 7;
            const int64_t q0 = qb + (grp >> 1) * 32;
            const int64_t qq = (grp & 1) ? min(q0 + 31, tot - 1) : min(q0, tot - 1);
            int lo = 0;  // invariant: off[lo] <= qq, answer in [lo, lo + S * 8)
#pragma unroll
            for (int S = PB / 8;; S = S >= 8 ? S / 8 : 1) {
                const int idx = lo + k * S;
                const bool le = idx < nb && sm.off[idx] <= qq;
                const unsigned m = (__ballot_sync(FULLMASK, le) >> (grp * 8)) & 0xffu;
                lo += (__popc(m) - 1) * S;
                if (S == 1) break;
            }
#pragma unroll
            for (int u = 0; u < 2; ++u) {
                const int64_t q = qb + u * 32 + lane;
                const int wlo = __shfl_sync(FULLMASK, lo, 16 * u), whi = __shfl_sync(FULLMASK, lo, 16 * u + 8) + 1;
                ok[u] = q < tot;
                pos[u] = 0;
                a[u] = 0.0;
                if (ok[u]) {
                    int l2 = wlo, h2 = whi;
                    while (h2 - l2 > 1) {
                        const int mid = (l2 + h2) >> 1;
                        if (sm.off[mid] <= q) l2 = mid;
                        else h2 = mid;
                    }
                    pos[u] = sm.bs[l2] + (q - sm.off[l2]);
                    SPG_CHECK(l2 >= 0 && l2 < nb && q >= sm.off[l2] && q < sm.off[l2 + 1]);
                    SPG_CHECK(pos[u] >= B.rp[0] && pos[u] < B.rp[B.nrows]);
                    if (VALS) a[u] = sm.a[l2];
                }
            }
        };
        int64_t qb = (int64_t)(threadIdx.x >> 5) * 64;  // warp-uniform
        if (qb < tot) {
            int64_t pos[2];
            double av[2];
            bool ok[2];
            int32_t c[2];
            double v[2];
            locate(qb, pos, av, ok);
#pragma unroll
            for (int u = 0; u < 2; ++u) {
                c[u] = ok[u] ? __ldg(&B.col[pos[u]]) : 0;
                v[u] = (VALS && ok[u]) ? av[u] * __ldg(&B.val[pos[u]]) : 0.0;
            }
            int64_t qc = qb;  // first product of the claim being consumed
            while (true) {
                unsigned nc = 0;
                if (lane == 0) nc = atomicAdd(&sm.next, 1u);
                const int64_t qn = (int64_t)__shfl_sync(FULLMASK, nc, 0) * 64;
                int32_t cn[2] = {0, 0};
                double vn[2] = {0.0, 0.0};
                bool okn[2] = {false, false};
                if (qn < tot) {  // next claim's gathers first
                    locate(qn, pos, av, okn);
#pragma unroll
                    for (int u = 0; u < 2; ++u) {
                        cn[u] = okn[u] ? __ldg(&B.col[pos[u]]) : 0;
                        vn[u] = (VALS && okn[u]) ? av[u] * __ldg(&B.val[pos[u]]) : 0.0;
                    }
                }
#pragma unroll
                for (int u = 0; u < 2; ++u)
                    if (ok[u]) {
                        if constexpr (WITH_Q) f(c[u], v[u], qbase + qc + u * 32 + lane);
                        else f(c[u], v[u]);
                    }
                if (qn >= tot) break;
                qc = qn;
#pragma unroll
                for (int u = 0; u < 2; ++u) {
                    c[u] = cn[u];
                    v[u] = vn[u];
                    ok[u] = okn[u];
                }
            }
        }
        qbase += tot;
        __syncthreads();
    }
    return qbase;
}

// all products of row i (A entries [A.rp[i], A.rp[i+1]))
template <int NT, bool VALS, int PB, typename SEG, typename F>
__device__ __forceinline__ int64_t block_row_products(const DevCSR &A, const DevCSR &B, int64_t i,
                                                      ProdSmemT<PB> &sm, const SEG &seg, F &&f) {
    return range_products<NT, VALS>(A, B, A.rp[i], A.rp[i + 1], sm, seg, f);
}

template <int NT, bool VALS, int PB, typename F>
__device__ __forceinline__ int64_t block_row_products(const DevCSR &A, const DevCSR &B, int64_t i,
                                                      ProdSmemT<PB> &sm, F &&f) {
    return range_products<NT, VALS>(A, B, A.rp[i], A.rp[i + 1], sm, WholeSeg{}, f);
}

// find-or-insert of a column in a warp-private table; returns the slot
__device__ __forceinline__ uint32_t find_slot(int32_t *keys, int32_t c, int lg) {
    const uint32_t mask = (1u << lg) - 1;
    uint32_t h = hslot(c, lg);
    volatile int32_t *vk = keys;
    while (true) {
        const int32_t k = vk[h];
        if (k == c) return h;
        if (k == EMPTY) {
            const int32_t old = atomicCAS(&keys[h], EMPTY, c);
            if (old == EMPTY || old == c) return h;
        }
        h = (h + 1) & mask;
    }
}

// Warp-uniform find-or-insert (W tier): every lane of the warp calls it (inactive lanes with
// ok = false); all lanes probe in lockstep -- one predicated LDS (+ predicated CAS on an empty
// slot) per step and one uniform vote to leave -- instead of a divergent per-lane loop, whose
// reconvergence barriers and branch resolution dominated the stalls of the W kernels (ncu).
// Returns the slot (undefined for inactive lanes); *fresh = 1 if this lane inserted the key.
__device__ __forceinline__ uint32_t warp_find_slot(int32_t *keys, int32_t c, int lg, bool ok, int *fresh) {
    const uint32_t mask = (1u << lg) - 1;
    uint32_t h = hslot(c, lg);
    volatile int32_t *vk = keys;
    bool done = !ok;
    int ins = 0;
    while (true) {
        if (!done) {
            int32_t k = vk[h];
            if (k == EMPTY) {
                k = atomicCAS(&keys[h], EMPTY, c);
                if (k == EMPTY) {
                    ins = 1;
                    k = c;
                }
            }
            if (k == c) done = true;
            else h = (h + 1) & mask;
        }
        if (__all_sync(FULLMASK, done)) break;
    }
    *fresh = ins;
    return h;
}

// vectorised fill of n (multiple of 4) int32 / n (even) doubles with a warp
__device__ __forceinline__ void warp_fill_keys(int32_t *keys, int n) {
    const int lane = threadIdx.x & 31;
    int4 *k4 = reinterpret_cast<int4 *>(keys);
    for (int t = lane; t < (n >> 2); t += 32) k4[t] = make_int4(EMPTY, EMPTY, EMPTY, EMPTY);
}
__device__ __forceinline__ void warp_fill_zero(double *v, int n) {
    const int lane = threadIdx.x & 31;
    double2 *v2 = reinterpret_cast<double2 *>(v);
    for (int t = lane; t < (n >> 1); t += 32) v2[t] = make_double2(0.0, 0.0);
}

// ------------------------------------------------------------------------------------------ S2

// COUNT_G lanes per row, 32 / COUNT_G rows per warp step, entries of a row strided over its
// lanes: a warp has the A-column loads and B.row_ptr gathers of 8 rows in flight at once (one row
// per warp left this pass latency-bound: 0.41 ms for C2's 2 M rows of 27 entries; 8 lanes per
// row 0.23 ms, 4 lanes 0.13 ms).  Rows longer than COUNT_LONG entries (power-law hubs) are done
// afterwards by the whole warp, one at a time, so that no 4-lane group walks a 10^4-entry row.
constexpr int COUNT_G = 4, COUNT_LONG = 256;
__device__ __forceinline__ void count_row_done(int64_t acc, int64_t deg, int64_t ncols, unsigned long long &lsum,
                                               unsigned long long &lmax, unsigned long long &lmaxb,
                                               unsigned long long &ldeg) {
    lsum += acc;
    lmax = max(lmax, (unsigned long long)acc);
    lmaxb = max(lmaxb, (unsigned long long)min(acc, ncols));
    ldeg = max(ldeg, (unsigned long long)deg);
}
// raw = 1: u[i] = the product count itself (spgemm_row_products); 0: the row bound min(u_i, ncols)
__global__ void __launch_bounds__(256) k_count(DevCSR A, DevCSR B, int64_t *__restrict__ u, Ctl *ctl, int raw) {
    const int lane = threadIdx.x & 31, sl = lane % COUNT_G;
    const int64_t ngroups = (int64_t)gridDim.x * (blockDim.x / COUNT_G);
    unsigned long long lsum = 0, lmax = 0, lmaxb = 0, ldeg = 0;
    const int64_t g0 = (int64_t)blockIdx.x * (blockDim.x / COUNT_G) + threadIdx.x / COUNT_G;
    // warp-uniform trip count (the shuffles below need every lane of the warp)
    const int64_t gw = g0 - (lane / COUNT_G);
    for (int64_t base = gw; base < A.nrows; base += ngroups) {
        const int64_t i = base + lane / COUNT_G;
        int64_t acc = 0, s = 0, e = 0;
        if (i < A.nrows) {
            s = A.rp[i];
            e = A.rp[i + 1];
            if (e - s <= COUNT_LONG) {
#pragma unroll 4
                for (int64_t p = s + sl; p < e; p += COUNT_G) {
                    const int32_t k = __ldg(&A.col[p]);
                    acc += __ldg(&B.rp[k + 1]) - __ldg(&B.rp[k]);
                }
            }
        }
#pragma unroll
        for (int o = COUNT_G / 2; o > 0; o >>= 1) acc += __shfl_xor_sync(FULLMASK, acc, o);
        const bool lng = i < A.nrows && e - s > COUNT_LONG;
        if (sl == 0 && i < A.nrows && !lng) {
            u[i] = raw ? acc : min(acc, B.ncols);  // the row's nnz bound: distinct columns <= min(products, ncols)
            count_row_done(acc, e - s, B.ncols, lsum, lmax, lmaxb, ldeg);
        }
        unsigned lm = __ballot_sync(FULLMASK, lng && sl == 0);
        while (lm) {  // long rows of this step: the whole warp, one row at a time
            const int src = __ffs(lm) - 1;
            lm &= lm - 1;
            const int64_t ri = __shfl_sync(FULLMASK, i, src);
            const int64_t rs = __shfl_sync(FULLMASK, s, src), re = __shfl_sync(FULLMASK, e, src);
            int64_t a2 = 0;
            for (int64_t p = rs + lane; p < re; p += 32) {
                const int32_t k = __ldg(&A.col[p]);
                a2 += __ldg(&B.rp[k + 1]) - __ldg(&B.rp[k]);
            }
            a2 = warp_sum(a2);
            if (lane == 0) {
                u[ri] = raw ? a2 : min(a2, B.ncols);
                count_row_done(a2, re - rs, B.ncols, lsum, lmax, lmaxb, ldeg);
            }
        }
    }
    // warp reduction of the block maxima / sums, one atomic each per warp
    lsum = warp_sum(lsum);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        lmax = max(lmax, __shfl_xor_sync(FULLMASK, lmax, o));
        lmaxb = max(lmaxb, __shfl_xor_sync(FULLMASK, lmaxb, o));
        ldeg = max(ldeg, __shfl_xor_sync(FULLMASK, ldeg, o));
    }
    if (lane == 0 && lsum) {
        atomicAdd(&ctl->sum_u, lsum);
        atomicMax(&ctl->max_u, lmax);
        atomicMax(&ctl->max_bound, lmaxb);
    }
    if (lane == 0 && ldeg) atomicMax(&ctl->max_deg, ldeg);
}

// --------------------------------------------------------------------------------- validation

// Rows of M must have lo <= rp[i] <= rp[i+1] <= lo + nnz (lo = *rp0, the first row_ptr entry of
// the caller's whole array, so a row panel or a device base is checked against the caller's
// allocation) and strictly increasing columns in [0, ncols).  A row whose offsets are out of that
// range is flagged without reading its columns (no access outside the caller's arrays).
__global__ void k_validate(DevCSR M, const int64_t *rp0, int64_t nnz, Ctl *ctl) {
    const int lane = threadIdx.x & 31;
    const int64_t lo = *rp0, hi = lo + nnz;
    const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t i = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < M.nrows; i += nw) {
        const int64_t s = M.rp[i], e = M.rp[i + 1];
        bool bad = e < s || s < lo || e > hi;
        if (!bad)
            for (int64_t p = s + lane; p < e; p += 32) {
                const int32_t c = M.col[p];
                if (c < 0 || c >= M.ncols || (p > s && M.col[p - 1] >= c)) bad = true;
            }
        if (__any_sync(FULLMASK, bad) && lane == 0) atomicOr(&ctl->err, 2u);
    }
}

__global__ void k_rebase(int64_t *rp, int64_t n, int64_t sub) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        rp[i] -= sub;
}

__global__ void k_add(int64_t *rp, int64_t n, int64_t d) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        rp[i] += d;
}

// ------------------------------------------------------------------------ tier classification

// rows too long for a warp: the medium tier (bound <= capM, when enabled), the CTA tier (one piece
// up to capB; column pieces up to capS when the pass has cursor scratch and the row's A entries
// fit it), the dense tier beyond
// The B list holds the pieced rows from its front and the one-piece rows from its back (cap = the
// pass's row count), so that the dynamic claims take the expensive rows first and the cheap ones
// fill the tail (longest-first; a pieced row can take 30x a one-piece row).
__device__ __forceinline__ void push_long(int64_t i, int64_t bound, const DevCSR &A, int64_t capM, int64_t capB,
                                          int64_t capS, const int32_t *cursor, int64_t curstride, int32_t *listM,
                                          int32_t *listB, int32_t *listG, Ctl *ctl, int64_t cap) {
    if (listM != nullptr && bound <= capM) {
        unsigned idx = atomicAdd(&ctl->nM, 1u);
        SPG_CHECK(idx < cap);
        listM[idx] = (int32_t)i;
        return;
    }
    const bool pieces_ok = cursor != nullptr && bound <= capS && A.rp[i + 1] - A.rp[i] <= curstride;
    if (bound <= capB) {
        unsigned idx = atomicAdd(&ctl->nBl, 1u);
        SPG_CHECK(idx < cap);
        listB[cap - 1 - idx] = (int32_t)i;
    } else if (pieces_ok) {
        unsigned idx = atomicAdd(&ctl->nB, 1u);
        SPG_CHECK(idx < cap);
        listB[idx] = (int32_t)i;
    } else {
        unsigned idx = atomicAdd(&ctl->nG, 1u);
        SPG_CHECK(idx < cap);
        listG[idx] = (int32_t)i;
    }
}

// ----------------------------------------------------------------------------- S4 symbolic, W
//
// One warp per row; rows are claimed ROW_BATCH at a time from a global counter (dynamic load
// balance for skewed rows).  Lanes form 32/G groups of G: each group takes one A entry A_ik and
// its lanes stride over B_k* (coalesced col loads).  Keys go to the warp's shared-memory table.

template <int G>
__global__ void __launch_bounds__(WARPS_W * 32) k_sym_w(SymArgs a) {
    extern __shared__ __align__(16) int32_t smem_i[];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    int32_t *keys = smem_i + wid * TW_SYM;
    AStage *ast = reinterpret_cast<AStage *>(smem_i + WARPS_W * TW_SYM) + wid;
    const int64_t R = a.r1 - a.r0;
    unsigned long long lmax = 0, nw = 0, nlong = 0;
    constexpr int MAXLG = 10;  // log2(TW_SYM)
    while (true) {
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(&a.ctl->row_ctr, (unsigned long long)a.batch);
        base = __shfl_sync(FULLMASK, base, 0);
        if ((int64_t)base >= R) break;
        const int64_t end = min((int64_t)base + a.batch, R);
        for (int64_t li = (int64_t)base; li < end; ++li) {
            const int64_t i = a.r0 + li;
            const int64_t bound = a.bnd[i];
            if (bound == 0) {
                if (lane == 0) a.nnz[i] = 0;
                continue;
            }
            if (bound > CAPW_SYM) {
                if (lane == 0) {
                    push_long(i, bound, a.A, CAPM_SYM, CAPB_SYM, CAPS_SYM, a.cursor, a.curstride, a.listM, a.listB,
                              a.listG, a.ctl, R);
                    nlong++;
                }
                continue;
            }
            const int lg = table_log2(bound, MAXLG);
            const int T = 1 << lg;
            warp_fill_keys(keys, T);
            __syncwarp();
            int cnt = 0;
            warp_row_products<G, (G == 32 ? 4 : 2), false, false>(a.A, a.B, i, ast, [&](bool ok, int32_t c, double) {
                int fresh;
                warp_find_slot(keys, c, lg, ok, &fresh);
                cnt += fresh;
            });
            cnt = warp_sum(cnt);
            if (lane == 0) {
                a.nnz[i] = cnt;
                lmax = max(lmax, (unsigned long long)cnt);
                nw++;
            }
            __syncwarp();
        }
    }
    if (lane == 0) {
        if (lmax) {
            atomicMax(&a.ctl->max_nnz, lmax);
            atomicMax(&a.ctl->pass_max, lmax);
        }
        if (nw) atomicAdd(&a.ctl->rows_w, nw);
    }
}

// ----------------------------------------------------------------------------- S4 symbolic, B

// Insert with an occupancy count (CTA tables): *ins counts fresh keys; past `limit` the piece is
// abandoned (*ovf = 1) and later inserts are skipped, so a table never fills beyond
// limit + (threads in flight) and probing always ends.  Returns the slot, or -1 if skipped.
// The count is aggregated per warp (one shared atomic per group of converged lanes instead of one
// per fresh key: on R-MAT rows nearly every product is a fresh key, and 512 threads incrementing
// one shared counter serialised the CTA tier).
__device__ __forceinline__ int insert_counted(int32_t *keys, int32_t c, int lg, int *ins, int limit,
                                              volatile int *ovf) {
    int h = -1, fresh = 0;
    if (!*ovf) {
        const uint32_t mask = (1u << lg) - 1;
        uint32_t hh = hslot(c, lg);
        volatile int32_t *vk = keys;
        while (true) {
            const int32_t k = vk[hh];
            if (k == c) break;
            if (k == EMPTY) {
                const int32_t old = atomicCAS(&keys[hh], EMPTY, c);
                if (old == EMPTY) {
                    fresh = 1;
                    break;
                }
                if (old == c) break;
            }
            hh = (hh + 1) & mask;
        }
        h = (int)hh;
    }
    const unsigned m = __activemask();
    const unsigned b = __ballot_sync(m, fresh);
    if (b && (threadIdx.x & 31) == __ffs(m) - 1) {
        const int cnt = __popc(b);
        if (atomicAdd(ins, cnt) + cnt > limit) *ovf = 1;
    }
    return h;
}

// [cmin, cmax] of row i's columns: the first and last column of every B row it touches
template <int NT>
__device__ __forceinline__ void row_col_span(const DevCSR &A, const DevCSR &B, int64_t i, int *s_span) {
    if (threadIdx.x == 0) {
        s_span[0] = INT_MAX;
        s_span[1] = -1;
    }
    __syncthreads();
    int mn = INT_MAX, mx = -1;
    for (int64_t p = A.rp[i] + threadIdx.x; p < A.rp[i + 1]; p += NT) {
        const int32_t k = __ldg(&A.col[p]);
        const int64_t s0 = __ldg(&B.rp[k]), e0 = __ldg(&B.rp[k + 1]);
        if (e0 > s0) {
            mn = min(mn, __ldg(&B.col[s0]));
            mx = max(mx, __ldg(&B.col[e0 - 1]));
        }
    }
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) {
        mn = min(mn, __shfl_xor_sync(FULLMASK, mn, d));
        mx = max(mx, __shfl_xor_sync(FULLMASK, mx, d));
    }
    if ((threadIdx.x & 31) == 0) {
        atomicMin(&s_span[0], mn);
        atomicMax(&s_span[1], mx);
    }
    __syncthreads();
}

// Column pieces of a long row (both passes): P = ceil(bound / target) pieces of equal width over
// the row's column span, processed in column order; a piece whose table passes its limit is
// halved and redone (the cursors advance only when a piece succeeds).  piece(lo, hi) runs the
// products of the piece and returns false on overflow; done(lo, hi) consumes a successful piece.
template <int NT, typename PIECE, typename DONE>
__device__ __forceinline__ void row_pieces(const DevCSR &A, const DevCSR &B, int64_t i, int64_t bound, int target,
                                           int32_t *cur, const int32_t *nxt, int *s_span, PIECE &&piece,
                                           DONE &&done) {
    row_col_span<NT>(A, B, i, s_span);
    const int64_t cmin = s_span[0], cmax = s_span[1];
    const int64_t deg = A.rp[i + 1] - A.rp[i];
    for (int64_t e = threadIdx.x; e < deg; e += NT) cur[e] = 0;
    __syncthreads();
    if (cmax < cmin) return;  // no products
    const int64_t P = (bound + target - 1) / target;
    const int64_t width = (cmax - cmin + P) / P;
    for (int64_t lo = cmin; lo <= cmax;) {
        int64_t hi = min(lo + width, cmax + 1);
        while (!piece((int32_t)lo, (int32_t)hi)) {
            __syncthreads();
            hi = lo + ((hi - lo) / 2 > 1 ? (hi - lo) / 2 : 1);
        }
        done();
        for (int64_t e = threadIdx.x; e < deg; e += NT) cur[e] = nxt[e];
        __syncthreads();
        lo = hi;
    }
}

__global__ void __launch_bounds__(THREADS_B, 1024 / THREADS_B) k_sym_b(SymArgs a) {
    extern __shared__ __align__(16) int32_t keys[];
    __shared__ ProdSmem psm;
    __shared__ int s_ins, s_ovf, s_span[2];
    constexpr int MAXLG = TB_SYM == 16384 ? 14 : TB_SYM == 8192 ? 13 : 12;  // log2(TB_SYM)
    static_assert((1 << MAXLG) == TB_SYM, "table size");
    constexpr int LIMIT = (TB_SYM / 4) * 3;
    int32_t *cur = a.cursor ? a.cursor + (int64_t)blockIdx.x * 2 * a.curstride : nullptr;
    int32_t *nxt = cur ? cur + a.curstride : nullptr;
    const unsigned nh = *(volatile unsigned *)&a.ctl->nB, n = nh + *(volatile unsigned *)&a.ctl->nBl;
    const int64_t R = a.r1 - a.r0;
    __shared__ unsigned s_idx;
    for (unsigned idx = cta_claim(&a.ctl->bctr, &s_idx); idx < n; idx = cta_claim(&a.ctl->bctr, &s_idx)) {
        const int64_t i = a.listB[idx < nh ? int64_t(idx) : R - 1 - int64_t(idx - nh)];
        const int64_t bound = a.bnd[i];
        int64_t total = 0;
        // one table pass over the products of [lo, hi) (whole row: seg = WholeSeg)
        auto pass = [&](int lg, const auto &seg, int limit) {
            const int T = 1 << lg;
            int4 *k4 = reinterpret_cast<int4 *>(keys);
            for (int t = threadIdx.x; t < T / 4; t += THREADS_B) k4[t] = make_int4(EMPTY, EMPTY, EMPTY, EMPTY);
            if (threadIdx.x == 0) {
                s_ins = 0;
                s_ovf = 0;
            }
            __syncthreads();
            // a whole row's table cannot overflow (>= 2 x bound slots): fresh keys are counted per
            // thread and reduced once, instead of a ballot + shared atomic per insert
            constexpr bool whole = std::is_same<std::decay_t<decltype(seg)>, WholeSeg>::value;
            int mine = 0;
            block_row_products<THREADS_B, false>(a.A, a.B, i, psm, seg, [&](int32_t c, double) {
                if (whole) mine += sym_insert(keys, c, lg);
                else insert_counted(keys, c, lg, &s_ins, limit, &s_ovf);
            });  // ends with a barrier
            if (whole) {
                mine = warp_sum(mine);
                if ((threadIdx.x & 31) == 0 && mine) atomicAdd(&s_ins, mine);
                __syncthreads();
            }
            return s_ovf == 0;
        };
        if (bound <= CAPB_SYM) {
            pass(table_log2(bound, MAXLG), WholeSeg{}, INT_MAX);
            total = s_ins;
        } else {
            row_pieces<THREADS_B>(
                a.A, a.B, i, bound, PIECE_SYM, cur, nxt, s_span,
                [&](int32_t lo, int32_t hi) { return pass(MAXLG, PieceSeg{a.B.col, cur, nxt, hi}, LIMIT); },
                [&]() { total += s_ins; });
        }
        if (threadIdx.x == 0) {
            a.nnz[i] = (int32_t)total;
            atomicMax(&a.ctl->max_nnz, (unsigned long long)total);
            atomicMax(&a.ctl->pass_max, (unsigned long long)total);
            atomicAdd(&a.ctl->rows_b, 1ull);
        }
        __syncthreads();
    }
}

// ----------------------------------------------------------------------------- S4 symbolic, M
//
// Rows whose bound exceeds a warp's table but fits a TM_SYM table at load <= 1/2: one 128-thread CTA
// per row with a 16 KB table, so that ~11 rows are in flight per SM instead of the B tier's 2 (on
// R-MAT most long rows have a few hundred to two thousand products).  The same
// flattened, load-balanced product iterator as the B tier, with a 128-entry A batch; fresh keys
// are counted per thread (sym_insert's return) and reduced once per row.
constexpr int PBATCH_M = THREADS_M;

__global__ void __launch_bounds__(THREADS_M) k_sym_m(SymArgs a) {
    extern __shared__ __align__(16) int32_t keys[];
    __shared__ ProdSmemT<PBATCH_M> psm;
    __shared__ int s_cnt;
    constexpr int MAXLG = 12;  // log2(TM_SYM)
    static_assert((1 << MAXLG) == TM_SYM, "table size");
    const unsigned n = *(volatile unsigned *)&a.ctl->nM;
    unsigned long long lmax = 0, nrow = 0;
    __shared__ unsigned s_idx;
    for (unsigned idx = cta_claim(&a.ctl->mctr, &s_idx); idx < n; idx = cta_claim(&a.ctl->mctr, &s_idx)) {
        const int64_t i = a.listM[idx];
        const int lg = table_log2(a.bnd[i], MAXLG);
        const int T = 1 << lg;
        for (int t = threadIdx.x; t < T; t += THREADS_M) keys[t] = EMPTY;
        if (threadIdx.x == 0) s_cnt = 0;
        __syncthreads();
        int cnt = 0;
        block_row_products<THREADS_M, false>(a.A, a.B, i, psm,
                                             [&](int32_t c, double) { cnt += sym_insert(keys, c, lg); });
        cnt = warp_sum(cnt);  // (block_row_products ended with a barrier: every insert is done)
        if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(&s_cnt, cnt);
        __syncthreads();
        if (threadIdx.x == 0) {
            a.nnz[i] = s_cnt;
            lmax = max(lmax, (unsigned long long)s_cnt);
            nrow++;
        }
    }
    if (threadIdx.x == 0 && nrow) {
        atomicMax(&a.ctl->max_nnz, lmax);
        atomicMax(&a.ctl->pass_max, lmax);
        atomicAdd(&a.ctl->rows_m, nrow);
    }
}

// ----------------------------------------------------------------------------- S4 symbolic, G
// Dense bitmap over all columns in this CTA's arena slot; atomicOr's return tells whether the
// column is new.  The bitmap is cleared again before the next row (by re-walking the products
// when that is cheaper than a sweep).

__global__ void __launch_bounds__(THREADS_G) k_sym_g(SymArgs a) {
    __shared__ int64_t s_scan[40];
    __shared__ ProdSmem psm;
    uint32_t *bm = a.gscratch + (int64_t)blockIdx.x * a.gstride;
    const unsigned n = *(volatile unsigned *)&a.ctl->nG;
    const int64_t nwords = (a.B.ncols + 31) / 32;
    __shared__ unsigned s_idx;
    // the first gblocks rows of the list were done by the split kernels (k_sym_g1 / g2)
    for (unsigned idx = a.gblocks + cta_claim(&a.ctl->gctr, &s_idx); idx < n;
         idx = a.gblocks + cta_claim(&a.ctl->gctr, &s_idx)) {
        const int64_t i = a.listG[idx];
        int cnt = 0;
        block_row_products<THREADS_G, false>(a.A, a.B, i, psm, [&](int32_t c, double) {
            const uint32_t bit = 1u << (c & 31);
            const uint32_t old = atomicOr(&bm[c >> 5], bit);
            cnt += (old & bit) ? 0 : 1;
        });
        int64_t tot;
        block_excl_scan<THREADS_G>(cnt, s_scan, &tot);
        if (threadIdx.x == 0) {
            a.nnz[i] = (int32_t)tot;
            atomicMax(&a.ctl->max_nnz, (unsigned long long)tot);
            atomicMax(&a.ctl->pass_max, (unsigned long long)tot);
            atomicAdd(&a.ctl->rows_g, 1ull);
        }
        // clear (block_excl_scan ended with a barrier, so all atomics of this row are done)
        if (a.bnd[i] < nwords) {  // bnd = min(products, ncols): re-walk only when cheaper than a sweep
            block_row_products<THREADS_G, false>(a.A, a.B, i, psm, [&](int32_t c, double) { bm[c >> 5] = 0u; });
        } else {
            for (int64_t w = threadIdx.x; w < nwords; w += THREADS_G) bm[w] = 0u;
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------- S4 / S6 dense tier, split rows
//
// A dense-tier row (beyond the pieced CTA tier: the hubs of C3-C5, up to 3e6 products each) is
// shared by KG_PARTS CTAs, each taking 1/KG_PARTS of the row's A entries, all accumulating into
// the row's own dense slot (bitmap + fp64 over all columns, L2 atomics); the slot is then swept
// in KG_SWEEP column ranges by as many CTAs (numeric: a count kernel and a write kernel, the
// ranges' offsets from the counts).  One CTA per row made every unit wait for its largest hub:
// C3 has ~60 such rows per unit, so most SMs idled (ncu: 25 % warps active) and the tier took
// 0.8 s of a 3 s step.  Row r of the tier's list uses slot r (r < gblocks); the list's rows
// beyond the slots take the one-CTA-per-row kernels (k_sym_g / k_num_g) afterwards.

__device__ __forceinline__ void part_range(const DevCSR &A, int64_t i, int64_t &p0, int64_t &p1) {
    const int64_t as = A.rp[i], d = A.rp[i + 1] - as;
    p0 = as + d * blockIdx.y / gridDim.y;
    p1 = as + d * (blockIdx.y + 1) / gridDim.y;
}

__global__ void __launch_bounds__(THREADS_G) k_sym_g1(SymArgs a) {
    const unsigned n = *(volatile unsigned *)&a.ctl->nG, r = blockIdx.x;
    if (r >= n || r >= (unsigned)a.gblocks) return;
    __shared__ ProdSmem psm;
    __shared__ int s_cnt;
    const int64_t i = a.listG[r];
    uint32_t *bm = a.gscratch + (int64_t)r * a.gstride;
    int64_t p0, p1;
    part_range(a.A, i, p0, p1);
    if (threadIdx.x == 0) s_cnt = 0;
    __syncthreads();
    int cnt = 0;
    range_products<THREADS_G, false>(a.A, a.B, p0, p1, psm, WholeSeg{}, [&](int32_t c, double) {
        const uint32_t bit = 1u << (c & 31);
        cnt += (atomicOr(&bm[c >> 5], bit) & bit) ? 0 : 1;  // fresh column: the bit was clear
    });
    cnt = warp_sum(cnt);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(&s_cnt, cnt);
    __syncthreads();
    if (threadIdx.x == 0 && s_cnt) atomicAdd(&a.gcnt[r * (KG_SWEEP + 1)], (unsigned long long)s_cnt);
}

// the row's nnz out, the slot's bitmap range cleared
__global__ void __launch_bounds__(THREADS_G2) k_sym_g2(SymArgs a) {
    const unsigned n = *(volatile unsigned *)&a.ctl->nG, r = blockIdx.x;
    if (r >= n || r >= (unsigned)a.gblocks) return;
    const int64_t nwords = (a.B.ncols + 31) / 32;
    uint32_t *bm = a.gscratch + (int64_t)r * a.gstride;
    const int64_t w0 = nwords * blockIdx.y / gridDim.y, w1 = nwords * (blockIdx.y + 1) / gridDim.y;
    for (int64_t w = w0 + threadIdx.x; w < w1; w += THREADS_G2) bm[w] = 0u;
    if (blockIdx.y == 0 && threadIdx.x == 0) {
        const int64_t i = a.listG[r];
        unsigned long long *gc = &a.gcnt[r * (KG_SWEEP + 1)];
        const unsigned long long tot = *gc;
        *gc = 0;
        a.nnz[i] = (int32_t)tot;
        atomicMax(&a.ctl->max_nnz, tot);
        atomicMax(&a.ctl->pass_max, tot);
        atomicAdd(&a.ctl->rows_g, 1ull);
    }
}

__global__ void __launch_bounds__(THREADS_G) k_num_g1(NumArgs a) {
    const unsigned n = *(volatile unsigned *)&a.ctl->nG, r = blockIdx.x;
    if (r >= n || r >= (unsigned)a.gblocks) return;
    __shared__ ProdSmem psm;
    const int64_t i = a.listG[r];
    uint32_t *bm = a.gbits + (int64_t)r * a.gstride_bits;
    double *dv = a.gvals + (int64_t)r * a.gstride_vals;
    int64_t p0, p1;
    part_range(a.A, i, p0, p1);
    range_products<THREADS_G, true>(a.A, a.B, p0, p1, psm, WholeSeg{}, [&](int32_t c, double v) {
        SPG_CHECK(c >= 0 && c < a.B.ncols);
        atomicOr(&bm[c >> 5], 1u << (c & 31));
        atomicAdd(&dv[c], v);
    });
}

// set bits of each column range of the slot
__global__ void __launch_bounds__(THREADS_G2) k_num_g2(NumArgs a) {
    const unsigned n = *(volatile unsigned *)&a.ctl->nG, r = blockIdx.x;
    if (r >= n || r >= (unsigned)a.gblocks) return;
    __shared__ int64_t s_scan[40];
    const int64_t nwords = (a.B.ncols + 31) / 32;
    const uint32_t *bm = a.gbits + (int64_t)r * a.gstride_bits;
    const int64_t w0 = nwords * blockIdx.y / gridDim.y, w1 = nwords * (blockIdx.y + 1) / gridDim.y;
    int64_t c = 0;
    for (int64_t w = w0 + threadIdx.x; w < w1; w += THREADS_G2) c += __popc(__ldcg(&bm[w]));
    int64_t tot;
    block_excl_scan<THREADS_G2>(c, s_scan, &tot);
    if (threadIdx.x == 0) a.gcnt[r * (KG_SWEEP + 1) + 1 + blockIdx.y] = (unsigned long long)tot;
}

// each column range written at its offset in the row (sorted: ranges and bits in column order);
// the slot range restored to zero
__global__ void __launch_bounds__(THREADS_G2) k_num_g3(NumArgs a) {
    const unsigned n = *(volatile unsigned *)&a.ctl->nG, r = blockIdx.x;
    if (r >= n || r >= (unsigned)a.gblocks) return;
    __shared__ int64_t s_scan[40];
    const int64_t i = a.listG[r];
    const int64_t o = a.crp[i], len = a.crp[i + 1] - o;
    const int64_t off0 = a.crp[a.r0];
    int32_t *oc = a.out_col + (o - off0);
    double *ov = a.out_val + (o - off0);
    const int64_t nwords = (a.B.ncols + 31) / 32;
    uint32_t *bm = a.gbits + (int64_t)r * a.gstride_bits;
    double *dv = a.gvals + (int64_t)r * a.gstride_vals;
    unsigned long long *gc = &a.gcnt[r * (KG_SWEEP + 1) + 1];
    int64_t cnt = 0, all = 0;
    for (int k = 0; k < (int)gridDim.y; ++k) {
        const int64_t ck = (int64_t)gc[k];
        if (k < (int)blockIdx.y) cnt += ck;
        all += ck;
    }
    const int64_t w0 = nwords * blockIdx.y / gridDim.y, w1 = nwords * (blockIdx.y + 1) / gridDim.y;
    for (int64_t wb = w0; wb < w1; wb += THREADS_G2) {
        const int64_t w = wb + threadIdx.x;
        uint32_t word = w < w1 ? __ldcg(&bm[w]) : 0u;
        int64_t tot;
        const int64_t ex = block_excl_scan<THREADS_G2>(__popc(word), s_scan, &tot);
        if (word) {
            int64_t pos = cnt + ex;
            bm[w] = 0u;
            while (word) {
                const int b = __ffs(word) - 1;
                word &= word - 1;
                const int64_t c = w * 32 + b;
                if (pos < len) {
                    oc[pos] = (int32_t)c;
                    ov[pos] = __ldcg(&dv[c]);
                }
                dv[c] = 0.0;
                ++pos;
            }
        }
        cnt += tot;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        if (blockIdx.y + 1 == gridDim.y && all != len) atomicOr(&a.ctl->err, 1u);
    }
}

__global__ void k_gcnt_clear(unsigned long long *gcnt, const Ctl *ctl, int slots) {
    // numeric range counts of the used slots back to zero (after k_num_g3 read them)
    const unsigned n = min(*(volatile const unsigned *)&ctl->nG, (unsigned)slots);
    for (unsigned t = blockIdx.x * blockDim.x + threadIdx.x; t < n * (KG_SWEEP + 1); t += gridDim.x * blockDim.x)
        gcnt[t] = 0ull;
}

// ------------------------------------------------------------------------------------- S5 scan
// y[0] holds the base on entry (device-resident: the previous chunk's end offset, or the slice
// base); y[1 + t] = y[0] + x[0] + ... + x[t] for t < n.  Three passes: tile sums, one-CTA scan of
// the tile sums (reads the base on the device, so chunks can be scanned back to back without a
// host round trip), and the tile-local scans.

template <typename T>
__global__ void __launch_bounds__(1024) k_scan_reduce(const T *__restrict__ x, int64_t n, int64_t *__restrict__ part) {
    __shared__ int64_t s[40];
    const int64_t b0 = (int64_t)blockIdx.x * SCAN_TILE;
    int64_t v = 0;
#pragma unroll
    for (int t = 0; t < SCAN_TILE / 1024; ++t) {
        const int64_t i = b0 + (int64_t)threadIdx.x * (SCAN_TILE / 1024) + t;
        if (i < n) v += (int64_t)x[i];
    }
    int64_t tot;
    block_excl_scan<1024>(v, s, &tot);
    if (threadIdx.x == 0) part[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(1024) k_scan_top(int64_t *part, int64_t nb, const int64_t *y0) {
    __shared__ int64_t s[40];
    int64_t carry = *y0;
    for (int64_t b0 = 0; b0 < nb; b0 += 1024) {
        const int64_t i = b0 + threadIdx.x;
        const int64_t v = i < nb ? part[i] : 0;
        int64_t tot;
        const int64_t ex = block_excl_scan<1024>(v, s, &tot);
        if (i < nb) part[i] = carry + ex;
        carry += tot;
    }
}

template <typename T>
__global__ void __launch_bounds__(1024) k_scan_apply(const T *__restrict__ x, int64_t n,
                                                     const int64_t *__restrict__ part, int64_t *__restrict__ y) {
    __shared__ int64_t s[40];
    constexpr int PER = SCAN_TILE / 1024;
    const int64_t b0 = (int64_t)blockIdx.x * SCAN_TILE + (int64_t)threadIdx.x * PER;
    int64_t v[PER];
    int64_t sum = 0;
#pragma unroll
    for (int t = 0; t < PER; ++t) {
        v[t] = (b0 + t < n) ? (int64_t)x[b0 + t] : 0;
        sum += v[t];
    }
    int64_t tot;
    int64_t run = block_excl_scan<1024>(sum, s, &tot) + part[blockIdx.x];
#pragma unroll
    for (int t = 0; t < PER; ++t) {
        run += v[t];
        if (b0 + t < n) y[1 + b0 + t] = run;
    }
}

// ------------------------------------------------------------------------------- chunk cutting

__global__ void k_fill(int64_t *b, int64_t n, int64_t v) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        b[i] = v;
}

__global__ void k_cut(const int64_t *__restrict__ crp, int64_t n, int64_t capp, int64_t *__restrict__ bounds,
                      int64_t nids) {
    const int64_t off0 = crp[0];
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t ci = (crp[i] - off0) / capp;
        const int64_t cp = i == 0 ? -1 : (crp[i - 1] - off0) / capp;
        for (int64_t c = cp + 1; c <= ci && c < nids; ++c) bounds[c] = i;
    }
}

// ------------------------------------------------------------------------------ S7 sort helpers

// warp bitonic sort of (keys, vals)[0..N) ascending by key, N a power of two >= 32
__device__ __forceinline__ void warp_bitonic(int32_t *keys, double *vals, int N) {
    const int lane = threadIdx.x & 31;
    for (int k = 2; k <= N; k <<= 1)
        for (int j = k >> 1; j > 0; j >>= 1) {
            for (int q = lane; q < (N >> 1); q += 32) {
                const int t = ((q & ~(j - 1)) << 1) | (q & (j - 1));
                const int p = t | j;
                const int32_t x = keys[t], y = keys[p];
                const bool up = (t & k) == 0;
                if ((x > y) == up) {
                    keys[t] = y;
                    keys[p] = x;
                    const double vx = vals[t];
                    vals[t] = vals[p];
                    vals[p] = vx;
                }
            }
            __syncwarp();
        }
}

template <int NT>
__device__ __forceinline__ void block_bitonic(int32_t *keys, double *vals, int N) {
    for (int k = 2; k <= N; k <<= 1)
        for (int j = k >> 1; j > 0; j >>= 1) {
            for (int q = threadIdx.x; q < (N >> 1); q += NT) {
                const int t = ((q & ~(j - 1)) << 1) | (q & (j - 1));
                const int p = t | j;
                const int32_t x = keys[t], y = keys[p];
                const bool up = (t & k) == 0;
                if ((x > y) == up) {
                    keys[t] = y;
                    keys[p] = x;
                    const double vx = vals[t];
                    vals[t] = vals[p];
                    vals[p] = vx;
                }
            }
            __syncthreads();
        }
}

__device__ __forceinline__ int pow2_at_least(int64_t n, int lo) {
    const int v = n <= 1 ? 1 : 1 << (64 - __clzll(n - 1));
    return v < lo ? lo : v;
}

// ------------------------------------------------------------------------------ S6 numeric, W

// Register bitonic sort of 32*E packed keys held E per lane (element e = r*32 + lane), ascending;
// partners within a lane for j >= 32, across lanes (shfl_xor) for j < 32.
template <typename K, int E>
__device__ __forceinline__ void reg_bitonic(K (&x)[E]) {
    const int lane = threadIdx.x & 31;
    constexpr int N = 32 * E;
#pragma unroll
    for (int k = 2; k <= N; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            if (j >= 32) {
#pragma unroll
                for (int r = 0; r < E; ++r) {
                    const int p = r ^ (j >> 5);
                    if (p > r) {
                        const bool up = (((r << 5) | lane) & k) == 0;
                        const K u = x[r], v = x[p];
                        const bool sw = (u > v) == up;
                        x[r] = sw ? v : u;
                        x[p] = sw ? u : v;
                    }
                }
            } else {
#pragma unroll
                for (int r = 0; r < E; ++r) {
                    const K y = __shfl_xor_sync(FULLMASK, x[r], j);
                    const bool up = (((r << 5) | lane) & k) == 0;
                    const bool keep_min = ((lane & j) == 0) == up;
                    x[r] = keep_min ? (y < x[r] ? y : x[r]) : (y > x[r] ? y : x[r]);
                }
            }
        }
    }
}

// load n packed keys (column << SB | slot) from smem or global memory, sort them in registers and
// write the row out in column order: col from the key, value gathered from its hash slot in
// shared memory (S7, §II-B).  pk may alias ov: all loads complete before any store.
// PK_G / V_G: keys / values live in global memory and are read at L2 (ld.cg): they were written
// or atomically updated in this row, possibly through other SMs' stale L1 views.
template <typename K, int E, int SB = 9, bool PK_G = false, bool V_G = false>
__device__ __forceinline__ void sort_emit(const K *pk, int n, const double *vals, int32_t *oc, double *ov) {
    const int lane = threadIdx.x & 31;
    K x[E];
#pragma unroll
    for (int r = 0; r < E; ++r) {
        const int e = (r << 5) | lane;
        x[r] = e < n ? (PK_G ? __ldcg(pk + e) : pk[e]) : ~K(0);
    }
    __syncwarp();
    reg_bitonic<K, E>(x);
#pragma unroll
    for (int r = 0; r < E; ++r) {
        const int e = (r << 5) | lane;
        if (e < n) {
            SPG_CHECK((int)(x[r] & ((K(1) << SB) - 1u)) < (1 << SB));
            oc[e] = (int32_t)(x[r] >> SB);
            const int slot = (int)(x[r] & ((K(1) << SB) - 1u));
            ov[e] = V_G ? __ldcg(vals + slot) : vals[slot];
        }
    }
}

// one warp sorts and emits a bucket of m packed keys (E chosen from m <= 512)
template <int SB, bool PK_G, bool V_G>
__device__ __forceinline__ void sort_emit_any(const unsigned long long *pk, int m, const double *vals, int32_t *oc,
                                              double *ov) {
    const int E = pow2_at_least((m + 31) / 32, 1);
    switch (E) {
        case 1: sort_emit<unsigned long long, 1, SB, PK_G, V_G>(pk, m, vals, oc, ov); break;
        case 2: sort_emit<unsigned long long, 2, SB, PK_G, V_G>(pk, m, vals, oc, ov); break;
        case 4: sort_emit<unsigned long long, 4, SB, PK_G, V_G>(pk, m, vals, oc, ov); break;
        case 8: sort_emit<unsigned long long, 8, SB, PK_G, V_G>(pk, m, vals, oc, ov); break;
        default: sort_emit<unsigned long long, 16, SB, PK_G, V_G>(pk, m, vals, oc, ov); break;
    }
}

template <int G, bool WIDE>
__global__ void __launch_bounds__(WARPS_W * 32, 4) k_num_w(NumArgs a) {
    extern __shared__ __align__(16) double smem_d[];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    AStage *ast = reinterpret_cast<AStage *>(smem_d) + wid;  // A-entry staging first (16-B aligned)
    double *vals = smem_d + WARPS_W * (sizeof(AStage) / sizeof(double)) + wid * TW_NUM;
    int32_t *keys = reinterpret_cast<int32_t *>(smem_d + WARPS_W * (sizeof(AStage) / sizeof(double)) +
                                                WARPS_W * TW_NUM) + wid * TW_NUM;
    // WIDE (ncols > 2^23): 64-bit packed keys staged after the key tables
    unsigned long long *stage = reinterpret_cast<unsigned long long *>(
                                    reinterpret_cast<int32_t *>(smem_d + WARPS_W * (sizeof(AStage) / sizeof(double)) +
                                                                WARPS_W * TW_NUM) + WARPS_W * TW_NUM) +
                                wid * TW_NUM;
    constexpr int MAXLG = 9;  // log2(TW_NUM)
    const int64_t R = a.r1 - a.r0;
    const int64_t off0 = a.crp[a.r0];
    while (true) {
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(&a.ctl->row_ctr, (unsigned long long)a.batch);
        base = __shfl_sync(FULLMASK, base, 0);
        if ((int64_t)base >= R) break;
        const int64_t end = min((int64_t)base + a.batch, R);
        for (int64_t li = (int64_t)base; li < end; ++li) {
            const int64_t i = a.r0 + li;
            const int64_t o = a.crp[i];
            const int64_t n = a.crp[i + 1] - o;
            if (n == 0) continue;
            if (n > CAPW_NUM) {
                if (lane == 0)
                    push_long(i, n, a.A, CAPM_NUM, CAPB_NUM, CAPS_NUM, a.cursor, a.curstride, a.listM, a.listB, a.listG,
                              a.ctl, R);
                continue;
            }
            const int lg = table_log2(a.tload == 0 ? n : a.tload == 1 ? (3 * n) / 2 : 2 * n, MAXLG);
            const int T = 1 << lg;
            warp_fill_keys(keys, T);
            warp_fill_zero(vals, T);
            __syncwarp();
            warp_row_products<G, (G == 32 ? 4 : 2), true, true>(a.A, a.B, i, ast, [&](bool ok, int32_t c, double v) {
                if (G == 32) {
                    // one B row per round: distinct columns -> distinct slots -> plain RMW
                    int fresh;
                    const uint32_t h = warp_find_slot(keys, c, lg, ok, &fresh);
                    if (ok) vals[h] += v;
                } else {
                    const unsigned act = __ballot_sync(FULLMASK, ok);
                    if (ok) {
                        const uint32_t h = find_slot(keys, c, lg);
                        const unsigned peers = __match_any_sync(act, c);
                        if (__popc(peers) == 1) vals[h] += v;
                        else atomicAdd(&vals[h], v);
                    }
                }
            });
            __syncwarp();
            // compaction of the occupied slots into packed sort keys (column << 9 | slot): in place
            // in `keys` for 32-bit keys (destination <= source, a round of 32 slots is read before
            // any of it is written), into the warp's staging array for 64-bit keys.  Values stay
            // in their slots and are gathered by slot after the sort.
            int cnt = 0;
            const unsigned lt = (1u << lane) - 1u;
            if (T >= 128) {
                // 128 slots per step, 4 per lane (one LDS.128); the order of the packed keys is
                // free (they are sorted next), so each of the 4 sub-slots is compacted by its own ballot
                for (int t0 = 0; t0 < T; t0 += 128) {
                    const int4 k4 = reinterpret_cast<const int4 *>(keys + t0)[lane];
                    const int32_t kk[4] = {k4.x, k4.y, k4.z, k4.w};
                    __syncwarp();  // the whole window is read before any write (dst < t0 + 128)
#pragma unroll
                    for (int r = 0; r < 4; ++r) {
                        const bool occ = kk[r] != EMPTY;
                        const unsigned bal = __ballot_sync(FULLMASK, occ);
                        if (occ) {
                            const int dst = cnt + __popc(bal & lt);
                            const unsigned slot = (unsigned)(t0 + 4 * lane + r);
                            if (WIDE) stage[dst] = ((unsigned long long)(uint32_t)kk[r] << 9) | slot;
                            else reinterpret_cast<uint32_t *>(keys)[dst] = ((uint32_t)kk[r] << 9) | slot;
                        }
                        cnt += __popc(bal);
                    }
                    __syncwarp();
                }
            } else {
                for (int t0 = 0; t0 < T; t0 += 32) {
                    const int32_t k = keys[t0 + lane];
                    const bool occ = k != EMPTY;
                    const unsigned bal = __ballot_sync(FULLMASK, occ);
                    const int dst = cnt + __popc(bal & lt);
                    __syncwarp();
                    if (occ) {
                        if (WIDE) stage[dst] = ((unsigned long long)(uint32_t)k << 9) | (unsigned)(t0 + lane);
                        else reinterpret_cast<uint32_t *>(keys)[dst] = ((uint32_t)k << 9) | (uint32_t)(t0 + lane);
                    }
                    cnt += __popc(bal);
                    __syncwarp();
                }
            }
            if (cnt != n) {
                if (lane == 0) atomicOr(&a.ctl->err, 1u);
                continue;
            }
            int32_t *oc = a.out_col + (o - off0);
            double *ov = a.out_val + (o - off0);
            const int E = pow2_at_least((n + 31) / 32, 1);
            if (WIDE) {
                switch (E) {
                    case 1: sort_emit<unsigned long long, 1>(stage, (int)n, vals, oc, ov); break;
                    case 2: sort_emit<unsigned long long, 2>(stage, (int)n, vals, oc, ov); break;
                    case 4: sort_emit<unsigned long long, 4>(stage, (int)n, vals, oc, ov); break;
                    case 8: sort_emit<unsigned long long, 8>(stage, (int)n, vals, oc, ov); break;
                    default: sort_emit<unsigned long long, 16>(stage, (int)n, vals, oc, ov); break;
                }
            } else {
                const uint32_t *pk = reinterpret_cast<const uint32_t *>(keys);
                switch (E) {
                    case 1: sort_emit<uint32_t, 1>(pk, (int)n, vals, oc, ov); break;
                    case 2: sort_emit<uint32_t, 2>(pk, (int)n, vals, oc, ov); break;
                    case 4: sort_emit<uint32_t, 4>(pk, (int)n, vals, oc, ov); break;
                    case 8: sort_emit<uint32_t, 8>(pk, (int)n, vals, oc, ov); break;
                    default: sort_emit<uint32_t, 16>(pk, (int)n, vals, oc, ov); break;
                }
            }
            __syncwarp();
        }
    }
}

// ------------------------------------------------------------------------------ S6 numeric, B

template <int NT>
struct CtaSortSmemT {
    int mm[3], occ[NT / 32];
    int64_t scan[40];
};

// fine-bucket cursors of the CTA sort: 8 NT buckets, two 16-bit cursors per word (positions are
// < 2^16); one array serves as histogram, bucket start, staging cursor and -- once staged -- bucket
// end (= the next bucket's start).  They alias the product iterator's ProdSmem (not in use while
// a table is sorted).
template <int NT>
struct SortCntT {
    union {
        uint32_t arr[4 * NT];
        struct {
            int cnt[64], cur[64], start[64];  // coarse buckets of the clustered-column fallback
        } co;
    };
    int esc_w[8][NT / 32];  // esc_sort_emit: per owner round and warp, the distinct count
};
template <int NT, int PB>
union ProdOrSortT {
    ProdSmemT<PB> psm;
    SortCntT<NT> sc;
};

template <typename T>
__device__ __forceinline__ T warp_incl_scan(T x) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const T y = __shfl_up_sync(FULLMASK, x, d);
        if (lane >= d) x += y;
    }
    return x;
}

// S7 for a CTA table of T <= 2^SB slots holding n keys (+ values).  Fast path: rank inside fine
// column buckets, entirely in shared memory -- every thread holds its SPT = 2^SB / NT slots' keys
// in registers, so the key table itself becomes the staging array once it has been read:
//   histogram of fine buckets (~4 keys each) -> bucket starts (block scan) -> each key staged in
//   its bucket as (offset within the bucket << SB | slot) -> rank = bucket start + the number of
//   smaller staged words in the bucket -> column and value written to their final position.
// (The previous version staged the keys in the global output and ranked from there: 56 % of
// k_num_b's instructions and 47 % of its stall samples on C3, profiles/r02/ncu_numb_c3_before.md.)
// A bucket over 64 keys (clustered columns) takes coarse buckets sorted by warps in registers,
// staged in the output value area; a coarse bucket over 512 keys the general path (compaction +
// shared-memory bitonic).  Writes oc/ov [0, n); returns false (nothing written) if the table does
// not hold exactly n keys.  All threads call; ends with a barrier; the key table is clobbered.
// ZV: the value table is left all zero (each value is cleared where it is read; the rare paths
// clear the whole table), so that the next pass need not refill it.
__device__ __forceinline__ void cswap_u32(uint32_t &a, uint32_t &b) {
    const uint32_t x = min(a, b), y = max(a, b);
    a = x;
    b = y;
}
template <int SB, int NT = THREADS_B, bool ZV = false>
__device__ bool cta_sort_emit(int32_t *keys, double *vals, int T, int64_t n, int32_t *oc, double *ov,
                              CtaSortSmemT<NT> &ss, SortCntT<NT> &sc) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    constexpr int NW = NT / 32;
    constexpr int SPT = (1 << SB) / NT;  // table slots per thread
    static_assert(SPT * NT == (1 << SB), "table size must be a multiple of the CTA size");
    constexpr int PLMAX = NT == 1024 ? 13 : NT == 512 ? 12 : NT == 256 ? 11 : NT == 128 ? 10 : 9;  // 2^PLMAX = 8 NT
    static_assert((1 << PLMAX) == 8 * NT, "eight fine buckets per thread");
    // fine buckets (~1 key each): 2^pl of them, bucket of key k = (k - lo) >> sh
    const int pl = min(PLMAX, max(5, 32 - __clz((int)max((int64_t)1, n) - 1)));
    for (int w = threadIdx.x; w < (1 << (pl - 1)); w += NT) sc.arr[w] = 0u;
    const int P = min(64, max(1, (int)((n + 255) / 256)));
    if (threadIdx.x == 0) {
        ss.mm[0] = INT_MAX;
        ss.mm[1] = -1;
    }
    int32_t kr[SPT];  // slot j * NT + threadIdx.x
#pragma unroll
    for (int j = 0; j < SPT; ++j) {
        const int t = j * NT + threadIdx.x;
        kr[j] = t < T ? keys[t] : EMPTY;
    }
    __syncthreads();
    {
        int lmin = INT_MAX, lmax = -1, occ = 0;
#pragma unroll
        for (int j = 0; j < SPT; ++j)
            if (kr[j] != EMPTY) {
                lmin = min(lmin, kr[j]);
                lmax = max(lmax, kr[j]);
                ++occ;
            }
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) {
            lmin = min(lmin, __shfl_xor_sync(FULLMASK, lmin, d));
            lmax = max(lmax, __shfl_xor_sync(FULLMASK, lmax, d));
            occ += __shfl_xor_sync(FULLMASK, occ, d);
        }
        if (lane == 0) {
            atomicMin(&ss.mm[0], lmin);
            atomicMax(&ss.mm[1], lmax);
            ss.occ[wid] = occ;
        }
    }
    __syncthreads();
    int occ_total = 0;
#pragma unroll
    for (int w = 0; w < NW; ++w) occ_total += ss.occ[w];
    if (occ_total != n || n == 0) {
        if (ZV && occ_total != n)
            for (int t = threadIdx.x; t < T; t += NT) vals[t] = 0.0;
        __syncthreads();
        return occ_total == n;
    }
    const int64_t lo = ss.mm[0], span = (int64_t)ss.mm[1] - lo + 1;
    {
        const int lspan = 64 - __clzll(span - 1);  // 2^lspan >= span
        const int sh = max(0, lspan - pl);
        // histogram (16-bit counters, two per word)
#pragma unroll
        for (int j = 0; j < SPT; ++j)
            if (kr[j] != EMPTY) {
                const uint32_t b = (uint32_t)(((int64_t)kr[j] - lo) >> sh);
                atomicAdd(&sc.arr[b >> 1], 1u << ((b & 1u) << 4));
            }
        __syncthreads();
        // bucket starts: thread t owns words 4t .. 4t+3 (buckets 8t .. 8t+7)
        const int w0 = 4 * threadIdx.x;
        const bool mine = w0 < (1 << (pl - 1));
        uint32_t wv[4];
        int sum = 0, big = 0;
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            wv[q] = mine ? sc.arr[w0 + q] : 0u;
            const int c0 = (int)(wv[q] & 0xffffu), c1 = (int)(wv[q] >> 16);
            sum += c0 + c1;
            big = max(big, max(c0, c1));
        }
        int64_t tot;
        int run = (int)block_excl_scan<NT>(sum, ss.scan, &tot);  // ends with a barrier
        if (mine) {
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int c0 = (int)(wv[q] & 0xffffu), c1 = (int)(wv[q] >> 16);
                sc.arr[w0 + q] = (uint32_t)run | ((uint32_t)(run + c0) << 16);
                run += c0 + c1;
            }
        }
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) big = max(big, __shfl_xor_sync(FULLMASK, big, d));
        if (lane == 0) ss.occ[wid] = big;
        __syncthreads();
        int bmax = 0;
#pragma unroll
        for (int w = 0; w < NW; ++w) bmax = max(bmax, ss.occ[w]);
        if (bmax <= 64 && sh + SB <= 31) {
            // stage (every key is in registers: the key table is free) -- the word
            // (offset within the bucket << SB | slot) at the bucket's next position
            uint32_t *stg = reinterpret_cast<uint32_t *>(keys);
            const uint32_t relmask = (1u << sh) - 1u;
#pragma unroll
            for (int j = 0; j < SPT; ++j)
                if (kr[j] != EMPTY) {
                    const uint32_t d = (uint32_t)((int64_t)kr[j] - lo);
                    const uint32_t b = d >> sh, hs = (b & 1u) << 4;
                    const int pos = (int)((atomicAdd(&sc.arr[b >> 1], 1u << hs) >> hs) & 0xffffu);
                    SPG_CHECK(b < (1u << pl) && pos >= 0 && pos < n);
                    stg[pos] = ((d & relmask) << SB) | (uint32_t)(j * NT + threadIdx.x);
                }
            __syncthreads();
            // every bucket b = [end(b - 1), end(b)) sorted in place by its owner thread (b mod NT;
            // ~1 key per bucket, so mostly nothing to do) and written out: consecutive lanes own
            // consecutive buckets, so one-key buckets give coalesced stores.  (Ranking every key
            // against its bucket-mates made each warp wait for its lane with the largest bucket:
            // 17 % of num_b's instructions, profiles/r02/ncu_numb_c3_v4.)
            // A bucket of <= 4 keys (99.6 % at ~1 key per bucket) is sorted by a 5-comparator network
            // on predicated loads -- every lane the same instructions; a larger bucket by insertion
            // sort.  (The per-bucket loops alone made each warp wait for its lane with the largest
            // bucket: the owner loop was 25 % of num_b's instructions at 3.8 active lanes per
            // instruction, profiles/r02/NOTES.md.)
            const int nb_used = (int)(((span - 1) >> sh) + 1);
            const uint32_t slotmask = (1u << SB) - 1u;
            for (int b = threadIdx.x; b < nb_used; b += NT) {
                const int e0 = (int)((sc.arr[b >> 1] >> ((b & 1) << 4)) & 0xffffu);
                const int s0 = b == 0 ? 0 : (int)((sc.arr[(b - 1) >> 1] >> (((b - 1) & 1) << 4)) & 0xffffu);
                const int m = e0 - s0;
                const int64_t cb = lo + ((int64_t)b << sh);
                if (m <= 4) {
                    uint32_t w[4];
#pragma unroll
                    for (int q = 0; q < 4; ++q) w[q] = q < m ? stg[s0 + q] : 0xffffffffu;
                    cswap_u32(w[0], w[1]);
                    cswap_u32(w[2], w[3]);
                    cswap_u32(w[0], w[2]);
                    cswap_u32(w[1], w[3]);
                    cswap_u32(w[1], w[2]);
#pragma unroll
                    for (int q = 0; q < 4; ++q)
                        if (q < m) {
                            const uint32_t sl = w[q] & slotmask;
                            SPG_CHECK(s0 + q < n && (int)sl < T);
                            oc[s0 + q] = (int32_t)(cb + (w[q] >> SB));
                            ov[s0 + q] = vals[sl];
                            if (ZV) vals[sl] = 0.0;
                        }
                } else {
                    for (int p = s0 + 1; p < e0; ++p) {  // insertion sort of the bucket's staged words
                        const uint32_t v = stg[p];
                        int q = p - 1;
                        while (q >= s0 && stg[q] > v) {
                            stg[q + 1] = stg[q];
                            --q;
                        }
                        stg[q + 1] = v;
                    }
                    for (int p = s0; p < e0; ++p) {
                        const uint32_t x = stg[p];
                        SPG_CHECK(p < n && (int)(x & slotmask) < T);
                        oc[p] = (int32_t)(cb + (x >> SB));
                        ov[p] = vals[x & slotmask];
                        if (ZV) vals[x & slotmask] = 0.0;
                    }
                }
            }
            __syncthreads();
            return true;
        }
    }
    // skewed columns (a fine bucket over 64 keys): coarse buckets sorted by warps in registers
    // (their counters alias the fine-bucket cursors, no longer read past the last barrier)
    if (threadIdx.x < 64) sc.co.cnt[threadIdx.x] = 0;
    __syncthreads();
    for (int t = threadIdx.x; t < T; t += NT) {
        const int32_t k = keys[t];
        if (k != EMPTY) atomicAdd(&sc.co.cnt[(int)(((int64_t)k - lo) * P / span)], 1);
    }
    __syncthreads();
    if (wid == 0) {  // bucket starts (lane l owns buckets l and l + 32) and the largest bucket
        const int c0 = lane < P ? sc.co.cnt[lane] : 0, c1 = lane + 32 < P ? sc.co.cnt[lane + 32] : 0;
        const int i0 = warp_incl_scan(c0), i1 = warp_incl_scan(c1);
        const int tot0 = __shfl_sync(FULLMASK, i0, 31);
        if (lane < P) sc.co.start[lane] = sc.co.cur[lane] = i0 - c0;
        if (lane + 32 < P) sc.co.start[lane + 32] = sc.co.cur[lane + 32] = tot0 + i1 - c1;
        int big = max(c0, c1);
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) big = max(big, __shfl_xor_sync(FULLMASK, big, d));
        if (lane == 0) ss.mm[2] = big;
    }
    __syncthreads();
    if (ss.mm[2] <= 512) {
        unsigned long long *stage = reinterpret_cast<unsigned long long *>(ov);
        for (int t = threadIdx.x; t < T; t += NT) {
            const int32_t k = keys[t];
            if (k != EMPTY) {
                const int pos = atomicAdd(&sc.co.cur[(int)(((int64_t)k - lo) * P / span)], 1);
                stage[pos] = ((unsigned long long)(uint32_t)k << SB) | (unsigned)t;
            }
        }
        __syncthreads();  // staged keys (global) visible to the block
        for (int b = wid; b < P; b += NW) {
            const int st = sc.co.start[b], m = sc.co.cnt[b];
            if (m == 0) continue;
            sort_emit_any<SB, true, false>(stage + st, m, vals, oc + st, ov + st);
        }
        __syncthreads();
        if (ZV) {
            for (int t = threadIdx.x; t < T; t += NT)
                if (keys[t] != EMPTY) vals[t] = 0.0;
            __syncthreads();
        }
        return true;
    }
    // general path: in-place compaction + shared-memory bitonic sort
    int64_t cnt = 0;
    for (int t0 = 0; t0 < T; t0 += NT) {
        const int t = t0 + threadIdx.x;
        const int32_t k = t < T ? keys[t] : EMPTY;
        const double v = t < T ? vals[t] : 0.0;
        const int occ = k != EMPTY;
        int64_t tot;
        const int64_t ex = block_excl_scan<NT>(occ, ss.scan, &tot);  // ends with a barrier
        if (occ) {
            keys[cnt + ex] = k;
            vals[cnt + ex] = v;
        }
        cnt += tot;
        __syncthreads();
    }
    const int N = pow2_at_least(n, 32);
    for (int t = (int)n + threadIdx.x; t < N; t += NT) keys[t] = INT_MAX;
    __syncthreads();
    block_bitonic<NT>(keys, vals, N);
    for (int t = threadIdx.x; t < n; t += NT) {
        oc[t] = keys[t];
        ov[t] = vals[t];
    }
    __syncthreads();
    if (ZV) {
        for (int t = threadIdx.x; t < T; t += NT) vals[t] = 0.0;
        __syncthreads();
    }
    return true;
}

// ------------------------------------------------------------ S6+S7 by sorting the products (ESC)
//
// The numeric CTA tier's rows and pieces are nearly all-distinct on power-law inputs (C3: 1.06
// products per nonzero), so accumulating them in a hash table and then sorting the table does the
// work twice: every product is an unsuccessful hash search with a CAS, and then every key is
// bucket-sorted.  Here the products themselves are sorted (expand - sort - compress): the product
// iterator stores product q's column and value at index q (no atomics, no probing; consecutive
// lanes, consecutive q), the products are bucketed by column (~1 per fine bucket, a histogram, a
// scan and a staging pass as in cta_sort_emit), each bucket is sorted by (column, q) and equal
// columns merged -- values summed in product order -- and a prefix over the buckets' distinct
// counts places every bucket's output.  Up to ESC_CAP products per pass (16 B each: value, column,
// staged word, in the 96 KB of the hash table).
constexpr int ESC_CAP = TB_NUM * 12 / 16;  // 6144

// u products in pc / pv [0, u) with columns in [lo, hi]; writes the distinct columns in order and
// their summed values to oc / ov.  Returns the number of distinct columns, -1 if some fine bucket
// holds more than 64 products (clustered or heavily repeated columns: the caller uses the hash
// path), -2 if there are more than nmax distinct columns (nothing written).  All threads call;
// ends with a barrier; stg and the sort counters are clobbered.
template <int NT>
__device__ int esc_sort_emit(const int32_t *pc, const double *pv, uint32_t *stg, int u, int32_t lo, int32_t hi,
                             int64_t nmax, int32_t *oc, double *ov, CtaSortSmemT<NT> &ss, SortCntT<NT> &sc) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    constexpr int NW = NT / 32;
    constexpr int PLMAX = NT == 1024 ? 13 : NT == 512 ? 12 : NT == 256 ? 11 : NT == 128 ? 10 : 9;  // 2^PLMAX = 8 NT
    if (u == 0) return 0;
    const int QB = 32 - __clz(max(u, 2) - 1);  // bits of a product index (2^QB >= u)
    const int pl = min(PLMAX, max(5, QB));     // 2^pl fine buckets, ~1 product each
    const int64_t span = (int64_t)hi - lo + 1;
    const int lspan = span <= 1 ? 0 : 64 - __clzll(span - 1);
    const int sh = max(0, lspan - pl);         // sh + QB <= lspan + 1 <= 32
    const uint32_t relmask = (1u << sh) - 1u, qmask = (1u << QB) - 1u;
    for (int w = threadIdx.x; w < (1 << (pl - 1)); w += NT) sc.arr[w] = 0u;
    __syncthreads();
    for (int q = threadIdx.x; q < u; q += NT) {  // histogram (16-bit counters, two per word)
        const uint32_t b = (uint32_t)(pc[q] - lo) >> sh;
        atomicAdd(&sc.arr[b >> 1], 1u << ((b & 1u) << 4));
    }
    __syncthreads();
    {  // bucket starts: thread t owns words 4t .. 4t+3 (buckets 8t .. 8t+7)
        const int w0 = 4 * threadIdx.x;
        const bool mine = w0 < (1 << (pl - 1));
        uint32_t wv[4];
        int sum = 0, big = 0;
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            wv[q] = mine ? sc.arr[w0 + q] : 0u;
            const int c0 = (int)(wv[q] & 0xffffu), c1 = (int)(wv[q] >> 16);
            sum += c0 + c1;
            big = max(big, max(c0, c1));
        }
        int64_t tot;
        int run = (int)block_excl_scan<NT>(sum, ss.scan, &tot);  // ends with a barrier
        if (mine) {
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int c0 = (int)(wv[q] & 0xffffu), c1 = (int)(wv[q] >> 16);
                sc.arr[w0 + q] = (uint32_t)run | ((uint32_t)(run + c0) << 16);
                run += c0 + c1;
            }
        }
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) big = max(big, __shfl_xor_sync(FULLMASK, big, d));
        if (lane == 0) ss.occ[wid] = big;
        __syncthreads();
        int bmax = 0;
#pragma unroll
        for (int w = 0; w < NW; ++w) bmax = max(bmax, ss.occ[w]);
        if (bmax > 64) {
            __syncthreads();
            return -1;
        }
    }
    for (int q = threadIdx.x; q < u; q += NT) {  // stage (offset in the bucket << QB | q) in its bucket
        const uint32_t d = (uint32_t)(pc[q] - lo);
        const uint32_t b = d >> sh, hs = (b & 1u) << 4;
        const int pos = (int)((atomicAdd(&sc.arr[b >> 1], 1u << hs) >> hs) & 0xffffu);
        SPG_CHECK(b < (1u << pl) && pos >= 0 && pos < u);
        stg[pos] = ((d & relmask) << QB) | (uint32_t)q;
    }
    __syncthreads();
    // owner pass 1 (bucket b = k NT + thread): sort in place by (column, q), count distinct columns
    const int nb_used = (int)(((span - 1) >> sh) + 1);
    auto bucket = [&](int b, int &s0, int &e0) {
        e0 = (int)((sc.arr[b >> 1] >> ((b & 1) << 4)) & 0xffffu);
        s0 = b == 0 ? 0 : (int)((sc.arr[(b - 1) >> 1] >> (((b - 1) & 1) << 4)) & 0xffffu);
    };
    int pos0[8];  // per round: the exclusive prefix of the distinct counts (-> first output position)
#pragma unroll
    for (int k = 0; k < 8; ++k) {
        const int b = k * NT + threadIdx.x;
        int dd = 0;
        if (b < nb_used) {
            int s0, e0;
            bucket(b, s0, e0);
            const int m = e0 - s0;
            if (m <= 4) {
                uint32_t w[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) w[q] = q < m ? stg[s0 + q] : 0xffffffffu;
                cswap_u32(w[0], w[1]);
                cswap_u32(w[2], w[3]);
                cswap_u32(w[0], w[2]);
                cswap_u32(w[1], w[3]);
                cswap_u32(w[1], w[2]);
                dd = m > 0;
#pragma unroll
                for (int q = 0; q < 4; ++q)
                    if (q < m) {
                        stg[s0 + q] = w[q];
                        if (q > 0) dd += (w[q] >> QB) != (w[q - 1] >> QB);
                    }
            } else {
                // insertion sort by column only: a large bucket is mostly repeats of a few (hub)
                // columns, already in order among themselves (their values are summed in any order,
                // as by the hash path's atomics)
                for (int p = s0 + 1; p < e0; ++p) {
                    const uint32_t v = stg[p];
                    int q = p - 1;
                    while (q >= s0 && (stg[q] >> QB) > (v >> QB)) {
                        stg[q + 1] = stg[q];
                        --q;
                    }
                    stg[q + 1] = v;
                }
                dd = 1;
                for (int p = s0 + 1; p < e0; ++p) dd += (stg[p] >> QB) != (stg[p - 1] >> QB);
            }
        }
        const int inc = warp_incl_scan(dd);
        pos0[k] = inc - dd;
        if (lane == 31) sc.esc_w[k][wid] = inc;
    }
    __syncthreads();
    // every warp scans the per-warp totals of each round itself (one barrier instead of two)
    int total = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) {
        const int x = lane < NW ? sc.esc_w[k][lane] : 0;
        const int y = warp_incl_scan(x);
        pos0[k] += total + __shfl_sync(FULLMASK, y - x, wid);
        total += __shfl_sync(FULLMASK, y, 31);
    }
    if (total > nmax) {
        __syncthreads();
        return -2;
    }
    // owner pass 2: merge equal columns (values summed in product order) and write the bucket
#pragma unroll
    for (int k = 0; k < 8; ++k) {
        const int b = k * NT + threadIdx.x;
        int s0 = 0, e0 = 0;
        if (b < nb_used) bucket(b, s0, e0);
        const int m = e0 - s0;
        if (m > 0) {
            const int64_t cb = lo + ((int64_t)b << sh);
            int pos = pos0[k];
            uint32_t prev = stg[s0];
            double acc = pv[prev & qmask];
            prev >>= QB;
            if (m <= 4) {
#pragma unroll
                for (int q = 1; q < 4; ++q)
                    if (q < m) {
                        const uint32_t x = stg[s0 + q];
                        const double v = pv[x & qmask];
                        if ((x >> QB) != prev) {
                            SPG_CHECK(pos < total);
                            oc[pos] = (int32_t)(cb + prev);
                            ov[pos] = acc;
                            ++pos;
                            prev = x >> QB;
                            acc = v;
                        } else {
                            acc += v;
                        }
                    }
            } else {
                for (int p = s0 + 1; p < e0; ++p) {
                    const uint32_t x = stg[p];
                    const double v = pv[x & qmask];
                    if ((x >> QB) != prev) {
                        SPG_CHECK(pos < total);
                        oc[pos] = (int32_t)(cb + prev);
                        ov[pos] = acc;
                        ++pos;
                        prev = x >> QB;
                        acc = v;
                    } else {
                        acc += v;
                    }
                }
            }
            SPG_CHECK(pos < total);
            oc[pos] = (int32_t)(cb + prev);
            ov[pos] = acc;
        }
    }
    __syncthreads();
    return total;
}

__global__ void __launch_bounds__(THREADS_BN, 1024 / THREADS_BN) k_num_b(NumArgs a) {
    extern __shared__ __align__(16) double smem_d[];
    double *vals = smem_d;                                          // hash path: TB_NUM values
    int32_t *keys = reinterpret_cast<int32_t *>(smem_d + TB_NUM);   // ... and TB_NUM keys
    double *pv = smem_d;                                            // ESC path (same 96 KB): values,
    int32_t *pc = reinterpret_cast<int32_t *>(smem_d + ESC_CAP);    // columns and staged words of
    uint32_t *stg = reinterpret_cast<uint32_t *>(pc + ESC_CAP);     // up to ESC_CAP products
    static_assert(ESC_CAP * 16 <= TB_NUM * 12, "ESC staging fits the table");
    __shared__ ProdOrSortT<THREADS_BN, PBATCH_BN> u;
    ProdSmemT<PBATCH_BN> &psm = u.psm;
    __shared__ CtaSortSmemT<THREADS_BN> ss;
    __shared__ int s_ins, s_ovf, s_span[2];
    constexpr int MAXLG = TB_NUM == 16384 ? 14 : TB_NUM == 8192 ? 13 : TB_NUM == 4096 ? 12 : 11;  // log2(TB_NUM)
    static_assert((1 << MAXLG) == TB_NUM, "table size");
    constexpr int LIMIT = (TB_NUM / 4) * 3;
    int32_t *cur = a.cursor ? a.cursor + (int64_t)blockIdx.x * 2 * a.curstride : nullptr;
    int32_t *nxt = cur ? cur + a.curstride : nullptr;
    const unsigned nh = *(volatile unsigned *)&a.ctl->nB, nrows = nh + *(volatile unsigned *)&a.ctl->nBl;
    const int64_t R = a.r1 - a.r0;
    const int64_t off0 = a.crp[a.r0];
    __shared__ unsigned s_idx;
    // the value table is zeroed once here and kept zero by cta_sort_emit<.., ZV> (each value cleared
    // where the sort reads it); only a piece abandoned on overflow leaves it dirty
    auto zero_vals = [&]() {
        double2 *v2 = reinterpret_cast<double2 *>(vals);
        for (int t = threadIdx.x; t < TB_NUM / 2; t += THREADS_BN) v2[t] = make_double2(0.0, 0.0);
    };
    zero_vals();  // (cta_claim's barrier follows)
    bool dirty = false;
    for (unsigned idx = cta_claim(&a.ctl->bctr, &s_idx); idx < nrows; idx = cta_claim(&a.ctl->bctr, &s_idx)) {
        const int64_t i = a.listB[idx < nh ? int64_t(idx) : R - 1 - int64_t(idx - nh)];
        const int64_t o = a.crp[i];
        const int64_t n = a.crp[i + 1] - o;
        int32_t *oc = a.out_col + (o - off0);
        double *ov = a.out_val + (o - off0);
        auto pass = [&](int lg, const auto &seg, int limit) {
            const int T = 1 << lg;
            if (dirty) zero_vals();
            dirty = false;
            int4 *k4 = reinterpret_cast<int4 *>(keys);
            for (int t = threadIdx.x; t < T / 4; t += THREADS_BN) k4[t] = make_int4(EMPTY, EMPTY, EMPTY, EMPTY);
            if (threadIdx.x == 0) {
                s_ins = 0;
                s_ovf = 0;
            }
            __syncthreads();
            // a whole row's key count is known (n) and its table cannot overflow: no counting
            constexpr bool whole = std::is_same<std::decay_t<decltype(seg)>, WholeSeg>::value;
            block_row_products<THREADS_BN, true>(a.A, a.B, i, psm, seg, [&](int32_t c, double v) {
                if (whole) {
                    atomicAdd(&vals[find_slot(keys, c, lg)], v);
                } else {
                    const int h = insert_counted(keys, c, lg, &s_ins, limit, &s_ovf);
                    if (h >= 0) atomicAdd(&vals[h], v);
                }
            });  // ends with a barrier
            dirty = s_ovf != 0;
            return !dirty;
        };
        // ESC pass over the products of seg: 1 = done (*m distinct columns written to ocw / ovw),
        // 0 = more than ESC_CAP products, -1 = a fine bucket over 64 products, -2 = more than nmax
        // distinct columns.  It overwrites the hash tables (dirty).
        auto esc_pass = [&](const auto &seg, int64_t nmax, int32_t *ocw, double *ovw, int &m) {
            if (threadIdx.x == 0) {
                ss.mm[0] = INT_MAX;
                ss.mm[1] = -1;
            }
            dirty = true;
            __syncthreads();
            int lmin = INT_MAX, lmax = -1;
            const int64_t nprod = block_row_products<THREADS_BN, true>(
                a.A, a.B, i, psm, seg, [&](int32_t c, double v, int64_t q) {
                    if (q < ESC_CAP) {
                        pc[q] = c;
                        pv[q] = v;
                        lmin = min(lmin, (int)c);
                        lmax = max(lmax, (int)c);
                    }
                });  // ends with a barrier
            if (nprod > ESC_CAP) return 0;
#pragma unroll
            for (int d = 16; d > 0; d >>= 1) {
                lmin = min(lmin, __shfl_xor_sync(FULLMASK, lmin, d));
                lmax = max(lmax, __shfl_xor_sync(FULLMASK, lmax, d));
            }
            if ((threadIdx.x & 31) == 0 && lmax >= 0) {
                atomicMin(&ss.mm[0], lmin);
                atomicMax(&ss.mm[1], lmax);
            }
            __syncthreads();
            const int r = esc_sort_emit<THREADS_BN>(pc, pv, stg, (int)nprod, ss.mm[0], ss.mm[1], nmax, ocw, ovw, ss,
                                                    u.sc);
            m = r;
            return r >= 0 ? 1 : r;
        };
        bool ok = true;
        if (n <= CAPB_NUM) {
            int m = 0;
            const int r = esc_pass(WholeSeg{}, n, oc, ov, m);
            if (r == 1) {
                ok = m == n;
            } else if (r == -2) {
                ok = false;
            } else {  // too many products or clustered columns: hash table + table sort
                const int lg = table_log2(n, MAXLG);
                pass(lg, WholeSeg{}, INT_MAX);
                ok = cta_sort_emit<MAXLG, THREADS_BN, true>(keys, vals, 1 << lg, n, oc, ov, ss, u.sc);
            }
        } else {
            int64_t written = 0;
            int esc_m = 0;  // >= 0: the piece was written by the ESC pass; -1: by the hash path
            row_pieces<THREADS_BN>(
                a.A, a.B, i, n, PIECE_NUM, cur, nxt, s_span,
                [&](int32_t lo, int32_t hi) {
                    const PieceSeg sg{a.B.col, cur, nxt, hi};
                    int m = 0;
                    const int r = esc_pass(sg, n - written, oc + written, ov + written, m);
                    if (r == 0) return false;  // too many products: the piece is halved
                    if (r == 1) {
                        esc_m = m;
                        return true;
                    }
                    if (r == -2) {
                        esc_m = 0;
                        ok = false;
                        return true;
                    }
                    esc_m = -1;  // clustered columns: this piece through the hash table
                    return pass(MAXLG, sg, LIMIT);
                },
                [&]() {
                    if (esc_m >= 0) {
                        written += esc_m;
                        return;
                    }
                    const int m = s_ins;
                    if (written + m <= n) {
                        ok &= cta_sort_emit<MAXLG, THREADS_BN, true>(keys, vals, TB_NUM, m, oc + written, ov + written,
                                                                     ss, u.sc);
                    } else {
                        ok = false;
                        dirty = true;
                    }
                    written += m;
                });
            ok &= written == n;
        }
        if (!ok && threadIdx.x == 0) atomicOr(&a.ctl->err, 1u);
        __syncthreads();
    }
}

// ------------------------------------------------------------------------------ S6 numeric, M
// One 128-thread CTA per row of CAPW_NUM < nnz <= CAPM_NUM (24 KB table: ~8 rows in flight per SM),
// the B tier's product iterator and bucket sort at 128 threads.

__global__ void __launch_bounds__(THREADS_M, 6) k_num_m(NumArgs a) {
    extern __shared__ __align__(16) double smem_d[];
    double *vals = smem_d;
    int32_t *keys = reinterpret_cast<int32_t *>(smem_d + TM_NUM);
    __shared__ ProdOrSortT<THREADS_M, PBATCH_M> u;
    __shared__ CtaSortSmemT<THREADS_M> ss;
    constexpr int MAXLG = 11;  // log2(TM_NUM)
    static_assert((1 << MAXLG) == TM_NUM, "table size");
    const unsigned nrows = *(volatile unsigned *)&a.ctl->nM;
    const int64_t off0 = a.crp[a.r0];
    __shared__ unsigned s_idx;
    {  // zero once; cta_sort_emit<.., ZV> keeps the value table zero (cta_claim's barrier follows)
        double2 *v2 = reinterpret_cast<double2 *>(vals);
        for (int t = threadIdx.x; t < TM_NUM / 2; t += THREADS_M) v2[t] = make_double2(0.0, 0.0);
    }
    for (unsigned idx = cta_claim(&a.ctl->mctr, &s_idx); idx < nrows; idx = cta_claim(&a.ctl->mctr, &s_idx)) {
        const int64_t i = a.listM[idx];
        const int64_t o = a.crp[i];
        const int64_t n = a.crp[i + 1] - o;
        const int lg = table_log2(n, MAXLG);
        const int T = 1 << lg;
        int4 *k4 = reinterpret_cast<int4 *>(keys);
        for (int t = threadIdx.x; t < T / 4; t += THREADS_M) k4[t] = make_int4(EMPTY, EMPTY, EMPTY, EMPTY);
        __syncthreads();
        block_row_products<THREADS_M, true>(a.A, a.B, i, u.psm, [&](int32_t c, double v) {
            atomicAdd(&vals[find_slot(keys, c, lg)], v);
        });  // ends with a barrier
        const bool ok = cta_sort_emit<MAXLG, THREADS_M, true>(keys, vals, T, n, a.out_col + (o - off0),
                                                        a.out_val + (o - off0), ss, u.sc);
        if (!ok && threadIdx.x == 0) atomicOr(&a.ctl->err, 1u);
        __syncthreads();
    }
}

// ------------------------------------------------------------------------------ S6 numeric, G
// Dense accumulation over all columns (§II-B): bitmap for structure (values may cancel to
// 0.0 and must still be stored), fp64 array for values, in this CTA's arena slot.  Output is
// produced in column order by sweeping the bitmap, which also restores the slot to zero.

__global__ void __launch_bounds__(THREADS_G) k_num_g(NumArgs a) {
    __shared__ int64_t s_scan[40];
    __shared__ ProdSmem psm;
    uint32_t *bm = a.gbits + (int64_t)blockIdx.x * a.gstride_bits;
    double *dv = a.gvals + (int64_t)blockIdx.x * a.gstride_vals;
    const unsigned nrows = *(volatile unsigned *)&a.ctl->nG;
    const int64_t nwords = (a.B.ncols + 31) / 32;
    const int64_t off0 = a.crp[a.r0];
    __shared__ unsigned s_idx;
    // the first gblocks rows of the list were done by the split kernels (k_num_g1 .. g3)
    for (unsigned idx = a.gblocks + cta_claim(&a.ctl->gctr, &s_idx); idx < nrows;
         idx = a.gblocks + cta_claim(&a.ctl->gctr, &s_idx)) {
        const int64_t i = a.listG[idx];
        const int64_t o = a.crp[i];
        const int64_t n = a.crp[i + 1] - o;
        block_row_products<THREADS_G, true>(a.A, a.B, i, psm, [&](int32_t c, double v) {
            atomicOr(&bm[c >> 5], 1u << (c & 31));
            atomicAdd(&dv[c], v);
        });
        int32_t *oc = a.out_col + (o - off0);
        double *ov = a.out_val + (o - off0);
        int64_t cnt = 0;
        for (int64_t w0 = 0; w0 < nwords; w0 += THREADS_G) {
            const int64_t w = w0 + threadIdx.x;
            uint32_t word = w < nwords ? __ldcg(&bm[w]) : 0u;
            int64_t tot;
            const int64_t ex = block_excl_scan<THREADS_G>(__popc(word), s_scan, &tot);
            if (word) {
                int64_t pos = cnt + ex;
                bm[w] = 0u;
                while (word) {
                    const int b = __ffs(word) - 1;
                    word &= word - 1;
                    const int64_t c = w * 32 + b;
                    if (pos < n) {
                        oc[pos] = (int32_t)c;
                        ov[pos] = __ldcg(&dv[c]);
                    }
                    dv[c] = 0.0;
                    ++pos;
                }
            }
            cnt += tot;
        }
        if (cnt != n && threadIdx.x == 0) atomicOr(&a.ctl->err, 1u);
        __syncthreads();
    }
}

// ------------------------------------------------------------------------------------ launchers

size_t symw_smem() { return size_t(WARPS_W) * (TW_SYM * sizeof(int32_t) + sizeof(AStage)); }
size_t numw_smem(bool wide) {
    return size_t(WARPS_W) * (TW_NUM * (sizeof(int32_t) + sizeof(double) + (wide ? sizeof(unsigned long long) : 0)) +
                              sizeof(AStage));
}
size_t symb_smem() { return size_t(TB_SYM) * sizeof(int32_t); }
size_t numb_smem() { return size_t(TB_NUM) * (sizeof(int32_t) + sizeof(double)); }
size_t symm_smem() { return size_t(TM_SYM) * sizeof(int32_t); }
size_t numm_smem() { return size_t(TM_NUM) * (sizeof(int32_t) + sizeof(double)); }

bool medium_enabled() {  // read per pass (host side), so that a test can switch it
    const char *v = getenv("SPGEMM_NO_MEDIUM");
    return !(v && v[0] == '1');
}

template <int G>
static void set_attrs_w() {
    cudaFuncSetAttribute(k_sym_w<G>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)symw_smem());
    cudaFuncSetAttribute(k_num_w<G, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)numw_smem(false));
    cudaFuncSetAttribute(k_num_w<G, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)numw_smem(true));
}

const Grids &grids(int device, int num_sms) {
    static Grids cache[64];
    static bool init[64] = {false};
    if (device < 0 || device >= 64) device = 0;
    if (!init[device]) {
        set_attrs_w<4>();
        set_attrs_w<8>();
        set_attrs_w<16>();
        set_attrs_w<32>();
        cudaFuncSetAttribute(k_sym_b, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)symb_smem());
        cudaFuncSetAttribute(k_num_b, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)numb_smem());
        cudaFuncSetAttribute(k_sym_m, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)symm_smem());
        cudaFuncSetAttribute(k_num_m, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)numm_smem());
        Grids g;
        int occ = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_count, 256, 0);
        g.count_blocks = num_sms * (occ > 0 ? occ : 1);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_sym_w<8>, WARPS_W * 32, symw_smem());
        g.symw_blocks = num_sms * (occ > 0 ? occ : 1);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_num_w<32, false>, WARPS_W * 32, numw_smem(false));
        g.numw_blocks = num_sms * (occ > 0 ? occ : 1);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_sym_b, THREADS_B, symb_smem());
        g.symb_blocks = num_sms * (occ > 0 ? occ : 1);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_num_b, THREADS_BN, numb_smem());
        g.numb_blocks = num_sms * (occ > 0 ? occ : 1);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_sym_m, THREADS_M, symm_smem());
        g.symm_blocks = num_sms * (occ > 0 ? occ : 1);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_num_m, THREADS_M, numm_smem());
        g.numm_blocks = num_sms * (occ > 0 ? occ : 1);
        cache[device] = g;
        init[device] = true;
    }
    return cache[device];
}

// rows a warp claims per atomic: large batches amortise the counter, small ones keep every SM
// busy on small chunks (at least ~4 claims per resident warp)
static int batch_for(int64_t rows, int full_blocks) {
    const int64_t warps = int64_t(full_blocks) * WARPS_W;
    int64_t b = rows / (warps * 4);
    return (int)(b < 1 ? 1 : (b > ROW_BATCH ? ROW_BATCH : b));
}

static int grid_for(int64_t n, int threads, int cap) {
    int64_t b = (n + threads - 1) / threads;
    if (b < 1) b = 1;
    return (int)(b < cap ? b : cap);
}

void launch_count(const DevCSR &A, const DevCSR &B, int64_t *u, Ctl *ctl, cudaStream_t s, bool raw) {
    if (A.nrows == 0) return;
    int dev = 0;
    cudaGetDevice(&dev);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int blocks = grid_for(A.nrows, 256 / COUNT_G, grids(dev, sms).count_blocks);
    k_count<<<blocks, 256, 0, s>>>(A, B, u, ctl, raw ? 1 : 0);
    LAUNCHED(1);
}

void launch_validate(const DevCSR &M, const int64_t *rp0, int64_t nnz, Ctl *ctl, cudaStream_t s) {
    if (M.nrows == 0) return;
    k_validate<<<grid_for(M.nrows, 8, 148 * 16), 256, 0, s>>>(M, rp0, nnz, ctl);
    LAUNCHED(1);
}

void launch_rebase(int64_t *rp, int64_t n, int64_t sub, cudaStream_t s) {
    if (n == 0 || sub == 0) return;
    k_rebase<<<grid_for(n, 256, 148 * 8), 256, 0, s>>>(rp, n, sub);
    LAUNCHED(1);
}

void launch_add(int64_t *crp, int64_t n, int64_t delta, cudaStream_t s) {
    if (delta == 0) return;
    k_add<<<grid_for(n + 1, 256, 148 * 8), 256, 0, s>>>(crp, n + 1, delta);
    LAUNCHED(1);
}

template <int G>
static void sym_w(const SymArgs &a, int blocks, cudaStream_t s) {
    k_sym_w<G><<<blocks, WARPS_W * 32, symw_smem(), s>>>(a);
    LAUNCHED(1);
}
template <int G>
static void num_w(const NumArgs &a, int blocks, cudaStream_t s) {
    if (a.B.ncols > (int64_t(1) << 23)) k_num_w<G, true><<<blocks, WARPS_W * 32, numw_smem(true), s>>>(a);
    else k_num_w<G, false><<<blocks, WARPS_W * 32, numw_smem(false), s>>>(a);
    LAUNCHED(1);
}
static int env_int(const char *name, int dflt) {
    const char *v = getenv(name);
    return (v && *v) ? atoi(v) : dflt;
}

static int group_for(const DevCSR &B, int64_t nnzB) {
    const double avg = B.nrows > 0 ? double(nnzB) / double(B.nrows) : 0.0;
    if (avg <= 5.0) return 4;
    if (avg <= 10.0) return 8;
    if (avg <= 20.0) return 16;
    return 32;
}

static inline void rec(cudaEvent_t *ev, int k, cudaStream_t s) {
    if (ev) cudaEventRecord(ev[k], s);
}

void launch_symbolic(const SymArgs &a, int num_sms, cudaStream_t s, cudaEvent_t *ev) {
    const int64_t rows = a.r1 - a.r0;
    if (rows <= 0) {
        for (int k = 0; k < 5; ++k) rec(ev, k, s);
        return;
    }
    int dev = 0;
    cudaGetDevice(&dev);
    const Grids &g = grids(dev, num_sms);
    static_assert(offsetof(Ctl, err) == CTL_RESET, "Ctl layout");
    cudaMemsetAsync(&a.ctl->row_ctr, 0, CTL_RESET, s);  // row_ctr, list lengths, pass_max, claim cursors
    SymArgs aw = a;
    if (!(a.tiers & 4)) aw.listM = nullptr;
    aw.batch = batch_for(rows, g.symw_blocks);
    const int wblocks = grid_for(rows, WARPS_W * aw.batch, g.symw_blocks);
    rec(ev, 0, s);
    switch (a.group) {
        case 4: sym_w<4>(aw, wblocks, s); break;
        case 8: sym_w<8>(aw, wblocks, s); break;
        case 16: sym_w<16>(aw, wblocks, s); break;
        default: sym_w<32>(aw, wblocks, s); break;
    }
    rec(ev, 1, s);
    if (aw.listM) {
        k_sym_m<<<g.symm_blocks, THREADS_M, symm_smem(), s>>>(aw);
        LAUNCHED(1);
    }
    rec(ev, 2, s);
    if (a.tiers & 1) {
        k_sym_b<<<a.cursor ? a.bblocks : g.symb_blocks, THREADS_B, symb_smem(), s>>>(a);
        LAUNCHED(1);
    }
    rec(ev, 3, s);
    // the dense tier: rows beyond the pieced CTA tier, and rows whose A entries do not fit the
    // cursor scratch (possible whenever the pass has CTA-tier rows; the kernel exits at once
    // when its list is empty)
    if ((a.tiers & 3) && a.gblocks > 0) {
        k_sym_g1<<<dim3(a.gblocks, KG_PARTS), THREADS_G, 0, s>>>(a);
        k_sym_g2<<<dim3(a.gblocks, KG_SWEEP), THREADS_G2, 0, s>>>(a);
        k_sym_g<<<a.gblocks, THREADS_G, 0, s>>>(a);  // rows beyond the slots (usually none)
        LAUNCHED(3);
    }
    rec(ev, 4, s);
}

void launch_numeric(const NumArgs &a, int num_sms, cudaStream_t s, cudaEvent_t *ev) {
    const int64_t rows = a.r1 - a.r0;
    if (rows <= 0) {
        for (int k = 0; k < 5; ++k) rec(ev, k, s);
        return;
    }
    int dev = 0;
    cudaGetDevice(&dev);
    const Grids &g = grids(dev, num_sms);
    cudaMemsetAsync(&a.ctl->row_ctr, 0, CTL_RESET, s);
    NumArgs aw = a;
    if (!(a.tiers & 4)) aw.listM = nullptr;
    static const int tload = env_int("SPGEMM_NUMW_TLOAD", 2);  // tuning knob
    aw.tload = tload;
    aw.batch = batch_for(rows, g.numw_blocks);
    const int wblocks = grid_for(rows, WARPS_W * aw.batch, g.numw_blocks);
    rec(ev, 0, s);
    switch (a.group) {
        case 4: num_w<4>(aw, wblocks, s); break;
        case 8: num_w<8>(aw, wblocks, s); break;
        case 16: num_w<16>(aw, wblocks, s); break;
        default: num_w<32>(aw, wblocks, s); break;
    }
    rec(ev, 1, s);
    if (aw.listM) {
        k_num_m<<<g.numm_blocks, THREADS_M, numm_smem(), s>>>(aw);
        LAUNCHED(1);
    }
    rec(ev, 2, s);
    if (a.tiers & 1) {
        k_num_b<<<a.cursor ? a.bblocks : g.numb_blocks, THREADS_BN, numb_smem(), s>>>(a);
        LAUNCHED(1);
    }
    rec(ev, 3, s);
    if ((a.tiers & 3) && a.gblocks > 0) {
        k_num_g1<<<dim3(a.gblocks, KG_PARTS), THREADS_G, 0, s>>>(a);
        k_num_g2<<<dim3(a.gblocks, KG_SWEEP), THREADS_G2, 0, s>>>(a);
        k_num_g3<<<dim3(a.gblocks, KG_SWEEP), THREADS_G2, 0, s>>>(a);
        k_gcnt_clear<<<grid_for(int64_t(a.gblocks) * (KG_SWEEP + 1), 256, 148), 256, 0, s>>>(a.gcnt, a.ctl, a.gblocks);
        k_num_g<<<a.gblocks, THREADS_G, 0, s>>>(a);  // rows beyond the slots (usually none)
        LAUNCHED(5);
    }
    rec(ev, 4, s);
}

template <typename T>
static void scan_impl(const T *x, int64_t n, int64_t *y, int64_t *tmp, cudaStream_t s) {
    if (n <= 0) return;
    const int64_t nb = (n + SCAN_TILE - 1) / SCAN_TILE;
    k_scan_reduce<T><<<(unsigned)nb, 1024, 0, s>>>(x, n, tmp);
    LAUNCHED(1);
    k_scan_top<<<1, 1024, 0, s>>>(tmp, nb, y);
    LAUNCHED(1);
    k_scan_apply<T><<<(unsigned)nb, 1024, 0, s>>>(x, n, tmp, y);
    LAUNCHED(1);
}

void launch_scan(const int32_t *x, int64_t n, int64_t *y, int64_t *tmp, cudaStream_t s) { scan_impl(x, n, y, tmp, s); }
void launch_scan64(const int64_t *x, int64_t n, int64_t *y, int64_t *tmp, cudaStream_t s) { scan_impl(x, n, y, tmp, s); }

void launch_cut(const int64_t *crp, int64_t n, int64_t cap_prime, int64_t *bounds, int64_t nids, cudaStream_t s) {
    k_fill<<<grid_for(nids + 1, 256, 148 * 4), 256, 0, s>>>(bounds, nids + 1, n);
    LAUNCHED(1);
    if (n > 0) {
        k_cut<<<grid_for(n, 256, 148 * 8), 256, 0, s>>>(crp, n, cap_prime, bounds, nids);
        LAUNCHED(1);
    }
}

int choose_group(const DevCSR &B, int64_t nnzB) { return group_for(B, nnzB); }

__global__ void k_publish(const int64_t *end, const Ctl *ctl, int64_t *host2) {
    // system-scope visibility: the host reads these after synchronising on an event
    volatile int64_t *h = host2;
    h[0] = *end;
    h[1] = (int64_t)ctl->pass_max;
    __threadfence_system();
}

void launch_publish(const int64_t *end, const Ctl *ctl, int64_t *host2, cudaStream_t s) {
    k_publish<<<1, 1, 0, s>>>(end, ctl, host2);
    LAUNCHED(1);
}

template <bool SUM>
__global__ void __launch_bounds__(256) k_seg_reduce(const int64_t *__restrict__ x, const int64_t *__restrict__ rows,
                                                    int64_t *__restrict__ out) {
    __shared__ int64_t s[8];
    const int64_t r0 = rows[blockIdx.x], r1 = rows[blockIdx.x + 1];
    int64_t m = 0;
    for (int64_t i = r0 + threadIdx.x; i < r1; i += blockDim.x) m = SUM ? m + x[i] : max(m, x[i]);
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) {
        const int64_t y = __shfl_xor_sync(FULLMASK, m, d);
        m = SUM ? m + y : max(m, y);
    }
    if ((threadIdx.x & 31) == 0) s[threadIdx.x >> 5] = m;
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < 8; ++w) m = SUM ? m + s[w] : max(m, s[w]);
        out[blockIdx.x] = m;
    }
}

// out[k] = largest column index in A's rows [rows[k], rows[k+1]) (-1 if they hold no entry): the
// last row of B a chunk reads.  Rows are sorted, so a row's largest column is its last entry:
// O(rows), not O(entries).
__global__ void __launch_bounds__(256) k_seg_max_col(DevCSR A, const int64_t *__restrict__ rows,
                                                     int64_t *__restrict__ out) {
    __shared__ int s[8];
    int m = -1;
    for (int64_t i = rows[blockIdx.x] + threadIdx.x; i < rows[blockIdx.x + 1]; i += blockDim.x) {
        const int64_t e = A.rp[i + 1];
        if (e > A.rp[i]) m = max(m, A.col[e - 1]);
    }
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) m = max(m, __shfl_xor_sync(FULLMASK, m, d));
    if ((threadIdx.x & 31) == 0) s[threadIdx.x >> 5] = m;
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < 8; ++w) m = max(m, s[w]);
        out[blockIdx.x] = max(m, s[0]);
    }
}

void launch_seg_max_col(const DevCSR &A, const int64_t *rows, int64_t nseg, int64_t *out, cudaStream_t s) {
    if (nseg <= 0) return;
    k_seg_max_col<<<(unsigned)nseg, 256, 0, s>>>(A, rows, out);
    LAUNCHED(1);
}

void launch_seg_max(const int64_t *x, const int64_t *rows, int64_t nseg, int64_t *out, cudaStream_t s) {
    if (nseg <= 0) return;
    k_seg_reduce<false><<<(unsigned)nseg, 256, 0, s>>>(x, rows, out);
    LAUNCHED(1);
}

void launch_seg_sum(const int64_t *x, const int64_t *rows, int64_t nseg, int64_t *out, cudaStream_t s) {
    if (nseg <= 0) return;
    k_seg_reduce<true><<<(unsigned)nseg, 256, 0, s>>>(x, rows, out);
    LAUNCHED(1);
}

__global__ void k_gather(const int64_t *__restrict__ crp, const int64_t *__restrict__ idx, int64_t n,
                         int64_t *__restrict__ out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = crp[idx[i]];
}

void launch_gather(const int64_t *crp, const int64_t *idx, int64_t n, int64_t *out, cudaStream_t s) {
    if (n > 0) {
        k_gather<<<grid_for(n, 256, 148 * 4), 256, 0, s>>>(crp, idx, n, out);
        LAUNCHED(1);
    }
}

// ------------------------------------------------------------- column panels of B (NEXT-1)
//
// When B does not fit the device budget, B is cut into column panels B[j] = B restricted to
// columns [lo_j, hi_j) (Alg. 3 line 4, §III-A, §III-D) and every chunk of C is
// A[i] x B[j].  The paper partitions B on the host in two stages (count per panel, then fill,
// L173) with a col_offset cursor per row (L182).  Here B streams through the device in row
// pieces: a histogram of column ids picks balanced panel boundaries, and each panel is built on
// the device by k_panel_len (two binary searches per row -- the cursor's job, without a
// sequential scan) + the chained scan + k_panel_fill.  Column ids stay global.

// hist[c >> shift] += 1 for the n column ids (nbins <= 4096; privatised in shared memory)
__global__ void __launch_bounds__(256) k_col_hist(const int32_t *__restrict__ col, int64_t n, int shift, int nbins,
                                                  unsigned long long *__restrict__ hist) {
    __shared__ unsigned int h[4096];
    for (int b = threadIdx.x; b < nbins; b += blockDim.x) h[b] = 0;
    __syncthreads();
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int32_t c = __ldg(&col[i]);
        if (c >= 0 && (c >> shift) < nbins) atomicAdd(&h[c >> shift], 1u);  // (invalid ids: flagged by k_validate)
    }
    __syncthreads();
    for (int b = threadIdx.x; b < nbins; b += blockDim.x)
        if (h[b]) atomicAdd(&hist[b], (unsigned long long)h[b]);
}

// first position p in [s, e) with col[p] >= c (e if none)
__device__ __forceinline__ int64_t lower_col(const int32_t *col, int64_t s, int64_t e, int32_t c) {
    while (s < e) {
        const int64_t m = (s + e) >> 1;
        if (__ldg(&col[m]) < c) s = m + 1;
        else e = m;
    }
    return s;
}

// len[k] = entries of row k of the piece with lo <= col < hi
__global__ void k_panel_len(DevCSR Bp, int32_t lo, int32_t hi, int32_t *__restrict__ len) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < Bp.nrows; k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t s = Bp.rp[k], e = Bp.rp[k + 1];
        const int64_t a = lower_col(Bp.col, s, e, lo);
        const int64_t b = lower_col(Bp.col, a, e, hi);
        len[k] = (int32_t)(b - a);
    }
}

// copy the panel's entries of every row of the piece to B[j] (rp = B[j]'s offsets of these rows);
// one warp per row, coalesced
__global__ void k_panel_fill(DevCSR Bp, int32_t lo, const int64_t *__restrict__ rp, int32_t *__restrict__ ocol,
                             double *__restrict__ oval) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
    for (int64_t k = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); k < Bp.nrows; k += nw) {
        const int64_t o = rp[k], n = rp[k + 1] - o;
        if (n == 0) continue;
        const int64_t a = lower_col(Bp.col, Bp.rp[k], Bp.rp[k + 1], lo);
        for (int64_t t = lane; t < n; t += 32) {
            ocol[o + t] = __ldg(&Bp.col[a + t]);
            oval[o + t] = __ldg(&Bp.val[a + t]);
        }
    }
}

// y[r] += x[r] (row totals accumulated over the panels); *mx = max over rows of the new y
__global__ void k_acc_i32(const int32_t *__restrict__ x, int32_t *__restrict__ y, int64_t n, unsigned long long *mx) {
    unsigned long long m = 0;
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        const int32_t t = y[r] + x[r];
        y[r] = t;
        m = max(m, (unsigned long long)t);
    }
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) m = max(m, __shfl_xor_sync(FULLMASK, m, d));
    if ((threadIdx.x & 31) == 0 && m && mx) atomicMax(mx, m);
}

// Chunk C[i][j] (rows [0, n) of a unit, packed in a ring slot at offsets crpj - crpj[0]) to its
// final place in host C: row r's piece lands after the pieces of panels j' < j of the same row,
// at crpt[r] + pre[r] (pre = sum of the row's earlier pieces).  The stores go straight into mapped pinned host memory
// over the host link (zero-copy), one warp per row -- a row's pieces are not contiguous in host
// C, so one copy-engine transfer per chunk cannot place them.
__global__ void k_scatter(const int32_t *__restrict__ scol, const double *__restrict__ sval,
                          const int64_t *__restrict__ crpj, const int32_t *__restrict__ pre,
                          const int64_t *__restrict__ crpt, int64_t n, int32_t *hcol, double *hval) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
    const int64_t base = crpj[0];
    for (int64_t r = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); r < n; r += nw) {
        const int64_t o = crpj[r] - base, len = crpj[r + 1] - crpj[r];
        if (len == 0) continue;
        const int64_t d = crpt[r] + pre[r];
        for (int64_t t = lane; t < len; t += 32) hcol[d + t] = scol[o + t];
        for (int64_t t = lane; t < len; t += 32) hval[d + t] = sval[o + t];
    }
}

void launch_col_hist(const int32_t *col, int64_t n, int shift, int nbins, unsigned long long *hist, cudaStream_t s) {
    if (n <= 0) return;
    k_col_hist<<<grid_for(n, 256 * 16, 148 * 4), 256, 0, s>>>(col, n, shift, nbins, hist);
    LAUNCHED(1);
}

void launch_panel_len(const DevCSR &Bp, int32_t lo, int32_t hi, int32_t *len, cudaStream_t s) {
    if (Bp.nrows <= 0) return;
    k_panel_len<<<grid_for(Bp.nrows, 256, 148 * 8), 256, 0, s>>>(Bp, lo, hi, len);
    LAUNCHED(1);
}

void launch_panel_fill(const DevCSR &Bp, int32_t lo, const int64_t *rp, int32_t *col, double *val, cudaStream_t s) {
    if (Bp.nrows <= 0) return;
    k_panel_fill<<<grid_for(Bp.nrows, 8, 148 * 16), 256, 0, s>>>(Bp, lo, rp, col, val);
    LAUNCHED(1);
}

void launch_acc_i32(const int32_t *x, int32_t *y, int64_t n, unsigned long long *mx, cudaStream_t s) {
    if (n <= 0) return;
    k_acc_i32<<<grid_for(n, 256, 148 * 8), 256, 0, s>>>(x, y, n, mx);
    LAUNCHED(1);
}

void launch_scatter(const int32_t *scol, const double *sval, const int64_t *crpj, const int32_t *pre,
                    const int64_t *crpt, int64_t n, int32_t *hcol, double *hval, int num_sms, cudaStream_t s) {
    if (n <= 0) return;
    k_scatter<<<grid_for(n, 8, num_sms * 4), 256, 0, s>>>(scol, sval, crpj, pre, crpt, n, hcol, hval);
    LAUNCHED(1);
}

}  // namespace spg
