"""bench.py -- C = A*A GFLOP/s (2 x intermediate products) including the D2H of all of C.

Default workload (N = 1): BASELINE.json configs[2] = R-MAT scale 22, edge factor 16, symmetric
(com-LiveJournal-like skew, 134 M nnz), C = A*A: 2.9e10 intermediate products and 2.7e10 nonzeros
of C = 0.33 TB, larger than host memory, so every output chunk streams into a pinned staging ring
and is handed to a sink that drops it (the paper's timing scope: "include the time for
transferring all chunks of the output matrix", §V-C).  This is the largest
configuration that fits one GPU ("1 GPU" in BASELINE.json); configs[0] is the oracle-sized case
and configs[1] / [3] / [4] are selectable with --config (C2 writes C into host memory).

One step = the whole hot path (DESIGN.md §2 rows S0-S10) through the C ABI: spgemm_plan (count,
chunk cut) + spgemm_execute_stream (per chunk: symbolic + scan, numeric + sort, D2H overlapped)
+ spgemm_free, on a fused plan.

  value  operands resident in HBM when the timed region starts (device operands);
  e2e    the same through the public API with HOST operands: the H2D of A (= B) from pinned host
         memory and the D2H of every chunk of C are inside the timed region.

Multi-GPU (torchrun, one rank per GPU, NCCL): rows of A are dealt as contiguous panels balanced by
intermediate products (each rank counts 1/N of the rows with the library's count kernel, one
all_gather gives everyone the same cuts); every rank drains its own chunks over its own host link;
in the e2e step every rank uploads 1/N of B and an NCCL all-gather over NVLink assembles B.  Total
work is fixed -> scaling "strong".

--impl reference runs the CPU oracle (the reference arm of this tier) on bounded samples.
"""
from __future__ import annotations

import argparse
import hashlib
import json
import os
import re
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

METRIC = json.load(open(os.path.join(ROOT, "BASELINE.json")))["metric"]
BUDGET_C2 = 2 << 30


# ---------------------------------------------------------------------------------------- helpers

def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=2, help="BASELINE.json configs index (2 = R-MAT s22, C = A*A)")
    ap.add_argument("--n", type=int, default=128, help="stencil edge for config 1")
    ap.add_argument("--scale", type=int, default=0, help="R-MAT scale override for configs 2/3 (tests)")
    ap.add_argument("--ring", type=int, default=3)
    ap.add_argument("--chunk-nnz", type=int, default=200_000_000,
                    help="sink mode: nonzeros per output chunk (pinned staging = ring x 12 B x this)")
    ap.add_argument("--e2e-steps", type=int, default=0, help="e2e steps (0 = --steps)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--two-phase", action="store_true", help="time the two-phase plan/execute path")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"])
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    return ap.parse_args()


class Clocks:
    """nvidia-smi sampler during the timed region (the profiling recipe's clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu, self.rows, self.p = gpu, [], None

    def __enter__(self):
        if os.environ.get("BENCH_CLOCKS", "1") == "0":  # diagnostic: no sampler process
            return self
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:  # noqa: BLE001
            self.p = None
        return self

    def _read(self):
        for line in self.p.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.p:
            time.sleep(0.25)
            self.p.terminate()
            try:
                self.p.wait(timeout=2)
            except Exception:  # noqa: BLE001
                self.p.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        ok = [r for r in self.rows if len(r) > 8 and r[1].replace(".", "").isdigit()]
        sm = [float(r[1]) for r in ok]
        mx = [float(r[2]) for r in ok if r[2].replace(".", "").isdigit()]
        pw = [float(r[3]) for r in ok if r[3].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in ok:
            for k, nm in enumerate(names):
                if r[5 + k].lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows),
                "power_w_median": float(np.median(pw)) if pw else None}


def probe_d2h(nbytes, dev, reps=2):
    """This box's pinned D2H rate (GB/s), measured in this process just before the timed region:
    copy-engine copies of `nbytes` (one output chunk's size) from HBM into a pinned buffer, best of
    `reps`, CUDA events on a side stream.  The step's link bound is judged against it."""
    import torch
    nbytes = int(min(max(nbytes, 1 << 20), 4 << 30))
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    src = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    src.fill_(7)
    s = torch.cuda.Stream(device=dev)
    best = None
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record(s)
            h.copy_(src, non_blocking=True)
            e1.record(s)
        s.synchronize()
        t = e0.elapsed_time(e1) / 1e3
        best = t if best is None else min(best, t)
    del src, h
    return nbytes / best / 1e9


def d2h_detail(tl, d2h_bytes):
    """Copy-engine view of the last timed step from its chunk timeline: when the first copy
    starts, how long the copy stream is busy vs idle between the first and last copy, and the
    rate while busy (separates a slow link from a starved one)."""
    if tl is None or len(tl) == 0:
        return None
    tl = tl[tl[:, 4] >= 0]  # copies are recorded on the last unit of each output chunk
    if len(tl) == 0:
        return None
    c0, c1 = tl[:, 4], tl[:, 5]
    busy = float(np.sum(c1 - c0))
    span = float(c1[-1] - c0[0])
    return {"first_copy_start_ms": float(c0[0]), "copy_span_ms": span, "copy_busy_ms": busy,
            "copy_idle_ms": span - busy, "rate_while_busy_GBps": d2h_bytes / (busy / 1e3) / 1e9 if busy > 0 else None,
            "copies": int(len(tl))}


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def load_config(args, gpu_gen=False):
    """(A, B, budget, name, sink): sink = True when C does not fit host memory (configs 2-4)."""
    c = args.config
    if c == 1:
        A = W.stencil_3d27(args.n)
        return A, A, BUDGET_C2, f"C2: 3-D 27-point stencil {args.n}^3, C=A*A, device budget 2 GiB (out-of-core)", False
    if c in (2, 3):
        scale = args.scale or (22 if c == 2 else 24)
        seed = 20210517 if c == 2 else 20210518
        A = W.rmat_torch(scale, 16, seed=seed) if gpu_gen else W.rmat(scale, 16, seed=seed)
        gen = "torch Philox on the GPU" if gpu_gen else "numpy PCG64"
        return A, A, 0, (f"C{c + 1}: R-MAT scale {scale} ef16 (0.45,0.2,0.2,0.15), symmetric, C=A*A through the "
                         f"sink ({gen} generator, seed {seed})"), True
    if c == 4:
        if gpu_gen:
            A = W.rmat_torch(24, col_scale=22, nedges=1 << 28, seed=11, symmetric=False)
            B = W.rmat_torch(22, col_scale=24, nedges=1 << 28, seed=12, symmetric=False)
        else:
            A = W.rmat_rect(24, 22, 1 << 28, seed=11)
            B = W.rmat_rect(22, 24, 1 << 28, seed=12)
        return A, B, 0, "C5: rect power-law A (2^24 x 2^22) x B (2^22 x 2^24), through the sink", True
    A, B, budget, name = W.config(c)
    return A, B, budget or 0, name, False


def tier_constants():
    """Tier thresholds of the kernels (csrc/internal.h), for the per-launch byte accounting."""
    txt = open(os.path.join(ROOT, "paper_conf_ipps_xia0ar21_b200", "csrc", "internal.h")).read()
    out = {}
    for k in ("CAPW_SYM", "CAPW_NUM", "CAPB_SYM", "CAPB_NUM", "PIECE_SYM", "PIECE_NUM", "CURSOR_MAX", "CAPM_SYM",
              "CAPM_NUM", "CAPS_SYM", "CAPS_NUM"):
        m = re.search(rf"\b{k}\s*=\s*(\d+)", txt)
        if m:
            out[k] = int(m.group(1))
    return out


def source_digest():
    """Digest of the kernel sources: a committed ncu counter is reported only for the code it was
    measured on."""
    h = hashlib.sha256()
    for f in ("kernels.cu", "internal.h"):
        h.update(open(os.path.join(ROOT, "paper_conf_ipps_xia0ar21_b200", "csrc", f), "rb").read())
    return h.hexdigest()[:16]


def row_products_np(A, B):
    """u_i = sum over A's row i of nnz(B_k*) (bench bookkeeping with numpy, not the oracle)."""
    bl = np.diff(B.row_ptr).astype(np.int64)
    deg = np.diff(A.row_ptr)
    if A.nnz == 0:
        return np.zeros(A.nrows, np.int64)
    u = np.add.reduceat(bl[A.col], np.minimum(A.row_ptr[:-1], A.nnz - 1))
    u[deg == 0] = 0
    return u


def tier_bytes(A, u, nnz_rows, r0, r1, info, kind):
    """Algorithmic bytes of the step per kernel class: Gustavson's row-by-row
    formulation (Alg. 1) reads per row its A entries (col [+ val]) and row_ptr pair, the
    B row_ptr pair of every A entry, one B entry per intermediate product (col + val = 12 B numeric,
    col = 4 B symbolic), and writes its output (12 B per C nonzero, or 4 B of nnz).  Rows are
    assigned to the tier the kernels assign them (the thresholds of csrc/internal.h)."""
    T = tier_constants()
    deg = np.diff(A.row_ptr[r0:r1 + 1]).astype(np.float64)
    uu = u[r0:r1].astype(np.float64)
    maxdeg = int(deg.max()) if len(deg) else 0
    curstride = (min(max(maxdeg, 1), T["CURSOR_MAX"]) + 31) & ~31
    if kind == "num":
        n = nnz_rows.astype(np.float64)
        per = 16.0 + 28.0 * deg + 12.0 * uu + 12.0 * n
        capw, capb, caps = T["CAPW_NUM"], T["CAPB_NUM"], T["CAPS_NUM"]
        key = n
    else:
        b = np.minimum(uu, A.ncols)
        per = 20.0 + 20.0 * deg + 4.0 * uu
        capw, capb, caps = T["CAPW_SYM"], T["CAPB_SYM"], T["CAPS_SYM"]
        key = b
    w = (key > 0) & (key <= capw)
    big = key > capw
    blk = big & ((key <= capb) | ((key <= caps) & (deg <= curstride)))
    g = big & ~blk
    out = {}
    for name, m in (("w", w), ("b", blk), ("g", g)):
        out[f"{kind}_{name}"] = {"bytes": float(per[m].sum()), "rows": int(m.sum()), "products": float(uu[m].sum())}
    capm = T.get("CAPM_NUM" if kind == "num" else "CAPM_SYM")
    if capm:  # medium CTA tier (csrc/internal.h): part of the "b" rows
        mm = blk & (key <= capm)
        out[f"{kind}_m"] = {"bytes": float(per[mm].sum()), "rows": int(mm.sum()), "products": float(uu[mm].sum())}
        out[f"{kind}_b"] = {"bytes": float(per[blk & ~mm].sum()), "rows": int((blk & ~mm).sum()),
                            "products": float(uu[blk & ~mm].sum())}
    return out


# ---------------------------------------------------------------------------------------- reference

def cpu_sample(A, B, seconds: float, threads=None):
    """Time the oracle (as it stands: structure pass + fp64 Alg. 1 values, no reference sums) on a
    contiguous block of rows sized for ~`seconds` of CPU work.  Returns a dict."""
    import oracle
    th = threads or oracle.default_threads()
    u = oracle.products(A, B, threads=th)
    cum = np.concatenate([[0], np.cumsum(u)])
    probe = int(np.searchsorted(cum, min(cum[-1], 2e7)))
    probe = max(1, min(probe, A.nrows))
    t0 = time.perf_counter()
    oracle.spgemm(A, B, rows=np.arange(probe), threads=th, with_ref=False)
    dt = max(time.perf_counter() - t0, 1e-6)
    rate = cum[probe] / dt
    want = min(float(cum[-1]), rate * seconds)
    nrows = int(np.searchsorted(cum, want))
    nrows = max(1, min(nrows, A.nrows))
    t0 = time.perf_counter()
    oracle.spgemm(A, B, rows=np.arange(nrows), threads=th, with_ref=False)
    dt = time.perf_counter() - t0
    prods = int(cum[nrows])
    return {"value": 2.0 * prods / dt / 1e9, "unit": "GFLOP/s", "cores": th, "kind": "oracle",
            "sample": f"rows 0..{nrows - 1} of {A.nrows} ({prods} of {int(cum[-1])} products, "
                      f"{100.0 * prods / max(1, cum[-1]):.1f}%), {dt:.2f} s",
            "seconds": dt, "products": prods}


def run_reference(args):
    world, rank, _ = dist_env()
    if rank != 0:
        return
    gpu_gen = False
    try:
        import torch
        gpu_gen = torch.cuda.is_available()  # the same matrix as our arm (torch generator on the GPU)
    except Exception:  # noqa: BLE001
        pass
    A, B, budget, name, _ = load_config(args, gpu_gen=gpu_gen)
    import oracle
    th = oracle.default_threads()
    per = max(2.0, min(args.cpu_seconds, 150.0 / max(1, args.steps + args.warmup)))
    for _ in range(args.warmup):
        cpu_sample(A, B, per / 4, th)
    vals = []
    last = None
    for _ in range(args.steps):
        last = cpu_sample(A, B, per, th)
        vals.append(last)
    prods = sum(v["products"] for v in vals)
    secs = sum(v["seconds"] for v in vals)
    value = 2.0 * prods / secs / 1e9
    line = {"metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * secs / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": name, "budget_bytes": budget}, "impl": "reference",
            "cpu_baseline": {"value": value, "unit": "GFLOP/s", "cores": th, "kind": "oracle",
                             "sample": last["sample"] + " per step"},
            "e2e": {"value": value, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------------------- ours

class SinkOut:
    """C larger than host memory: every output chunk lands in the library's pinned staging ring and
    is handed to this sink, which drops it (or, in the capture step, keeps per-row nnz and the
    sampled rows for the parity check)."""

    def __init__(self, r0, r1, sample_rows):
        self.r0, self.r1 = r0, r1
        self.sample = set(int(x) for x in sample_rows)
        self.capture = False
        self.nnz = 0
        self.rownnz = None
        self.kept = {}

    def cb(self, ra, rb, rp, col, val):
        self.nnz += int(rp[-1])
        if self.capture:
            self.rownnz[ra - self.r0:rb - self.r0] = np.diff(rp)
            for r in [x for x in self.sample if ra <= x < rb]:
                k = r - ra
                self.kept[r] = (col[rp[k]:rp[k + 1]].copy(), val[rp[k]:rp[k + 1]].copy())
        return 0

    def run(self, P, capture=False):
        self.nnz = 0
        self.capture = capture
        if capture:
            self.rownnz = np.zeros(self.r1 - self.r0, dtype=np.int64)
            self.kept = {}
        P.execute_stream(self.cb)
        return self.nnz


class HostOut:
    """C fits host memory (C1, C2): the rank's slice goes to pinned host arrays."""

    def __init__(self, rows, nnz):
        import torch
        t0 = time.perf_counter()
        self.rp = torch.empty(rows + 1, dtype=torch.int64, pin_memory=True)
        self.col = torch.empty(nnz, dtype=torch.int32, pin_memory=True)
        self.val = torch.empty(nnz, dtype=torch.float64, pin_memory=True)
        self.pin_s = time.perf_counter() - t0
        self.cap = nnz
        self.rownnz = None

    def run(self, P, capture=False):
        z = P.execute_capacity(self.rp, self.col, self.val, self.cap)
        if capture:
            self.rownnz = np.diff(self.rp.numpy())
        return z


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_xia0ar21_b200 import capi
    from paper_conf_ipps_xia0ar21_b200 import dist as pdist

    world, rank, local = dist_env()
    # one rank per GPU; --dist-backend gloo lets the multi-rank path run several ranks on one GPU
    # (a test of the control flow only: NCCL refuses two ranks on one device)
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(args.dist_backend)
    cdev = dev if (world > 1 and args.dist_backend == "nccl") else None  # collective tensors' device

    t_gen = time.perf_counter()
    A, B, budget, name, sink_mode = load_config(args, gpu_gen=True)
    gen_s = time.perf_counter() - t_gen
    same = A is B

    class Dev:
        pass

    def to_dev(M):
        # storage padded to a multiple of the world size: the e2e step refills these arrays with a
        # scatter (each rank uploads 1/world) + all-gather over NVLink (dist.scatter_allgather_csr)
        d = Dev()
        d.nrows, d.ncols = M.nrows, M.ncols
        d.store = []
        for nm, x in (("row_ptr", M.row_ptr), ("col", M.col), ("val", M.val)):
            t = torch.from_numpy(x)
            buf = torch.zeros(pdist.padded_len(t.numel(), world), dtype=t.dtype, device=dev)
            buf[:t.numel()].copy_(t)
            d.store.append(buf)
            setattr(d, nm, buf[:t.numel()])
        return d

    dB = to_dev(B)
    dA = dB if same else to_dev(A)
    stream = torch.cuda.current_stream()

    # flop-balanced row panels: each rank counts the products of 1/world of the rows with the
    # library's count kernel (spgemm_row_products), one all_gather, identical cuts everywhere
    if world > 1:
        s0, s1 = pdist.even_slices(A.nrows, world)[rank]
        u_loc, _ = capi.row_products(dA, dB, capi.opts(device=local, row_begin=s0, row_end=s1,
                                                       stream=stream.cuda_stream))
        u_all = pdist.allgather_rows(u_loc, A.nrows, device=cdev)
        panels = pdist.row_panels(A.row_ptr, world, weights=u_all)
    else:
        panels = [(0, A.nrows)]
    r0, r1 = panels[rank]

    # the budget covers every device byte of the multiply (reading R15): with resident
    # operands the arena gets the budget minus the operands' bytes; without a budget the arena is
    # 85 % of what is free (one arena for every step: cudaMalloc of ~150 GB is not part of a multiply)
    in_bytes = 8 * (B.nrows + 1) + 12 * B.nnz + (0 if same else 8 * (A.nrows + 1) + 12 * A.nnz)
    if budget:
        ws = torch.empty(budget - in_bytes, dtype=torch.uint8, device=dev)
    else:
        # ranks sharing one GPU (the gloo control-flow run) split its memory
        share = -(-int(os.environ.get("LOCAL_WORLD_SIZE", world)) // max(1, torch.cuda.device_count()))
        if world > 1:
            dist.barrier()  # every rank's operands are resident before anyone sizes its arena
        free = torch.cuda.mem_get_info()[0]
        if world > 1:
            dist.barrier()  # ... and every rank has read the free memory before anyone allocates
        ws = torch.empty(int(free * 0.85 / share), dtype=torch.uint8, device=dev)
    wbytes = ws.numel()
    fused = not args.two_phase
    chunk_nnz = args.chunk_nnz if sink_mode else 0

    def mk_opts(profile=False, base=0, workspace=None):
        return capi.opts(device=local, ring=args.ring, profile=profile, row_begin=r0, row_end=r1,
                         workspace=ws if workspace is None else workspace, stream=stream.cuda_stream,
                         row_ptr_base=base, fused=fused, chunk_nnz=chunk_nnz)

    # untimed: sizes (and for C2 the pinned host output, a one-time cost reported separately)
    u_np = row_products_np(A, B)
    products_local = int(u_np[r0:r1].sum())
    rng = np.random.default_rng(1)
    nloc = r1 - r0
    sample_rows = (np.unique(np.concatenate([[r0, r1 - 1], r0 + rng.integers(0, nloc, 64)])) if nloc
                   else np.zeros(0, np.int64))
    if sink_mode:
        out = SinkOut(r0, r1, sample_rows)
        pin_s = 0.0
    else:
        with capi.Plan(dA, dB, wbytes, capi.opts(device=local, ring=args.ring, row_begin=r0, row_end=r1,
                                                 workspace=ws, stream=stream.cuda_stream)) as P:
            nnz0 = P.info()["nnz"]
        out = HostOut(r1 - r0, nnz0)
        pin_s = out.pin_s

    host_ms = {"plan": [], "execute": [], "free": []}

    def step(profile=False, keep=False, capture=False):
        """One multiply (plan + execute + free).  keep: return the plan unfreed, so that its
        kernel times (CUDA events recorded inside the step) are read after the timed region."""
        h0 = time.perf_counter()
        P = capi.Plan(dA, dB, wbytes, mk_opts(profile))
        h1 = time.perf_counter()
        z = out.run(P, capture)
        if world > 1 and not sink_mode:
            b, _ = pdist.slice_bases(z, device=cdev)
            capi.rebase_host(out.rp, b)
        h2 = time.perf_counter()
        host_ms["plan"].append(1e3 * (h1 - h0))
        host_ms["execute"].append(1e3 * (h2 - h1))
        if keep:
            return P, z
        P.free()
        host_ms["free"].append(1e3 * (time.perf_counter() - h2))
        return None, z

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        step(profile=True)
    barrier()
    for v in host_ms.values():
        v.clear()
    d2h_est = 12 * (args.chunk_nnz if sink_mode else out.cap)
    link_live = probe_d2h(d2h_est, dev)
    launches0 = capi.kernel_launches()
    with Clocks(local) as clk:
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        w0 = time.perf_counter()
        e0.record(stream)
        for k in range(args.steps):
            last = step(profile=True, keep=(k == args.steps - 1), capture=(k == args.steps - 1))
        e1.record(stream)
        barrier()
        wall = time.perf_counter() - w0
    launches = capi.kernel_launches() - launches0
    Pl, nnz_local = last
    stats = Pl.stats()  # kernel times of the last timed step (events recorded inside it)
    tl = capi.timeline(Pl)  # [chunk, 6] ms: analysis, numeric and copy start/end
    info = Pl.info()
    Pl.free()
    ms = e0.elapsed_time(e1)
    t_max = ms
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=cdev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        t_max = float(t.item())
        products_total = pdist.slice_bases(products_local, device=cdev)[1]
        nnz_total = pdist.slice_bases(nnz_local, device=cdev)[1]
        copies_total = pdist.slice_bases(info["num_copies"], device=cdev)[1]
    else:
        products_total, nnz_total, copies_total = products_local, nnz_local, info["num_copies"]
    assert info["products"] == products_local, (info["products"], products_local)
    value = 2.0 * products_total * args.steps / (t_max / 1e3) / 1e9
    # bytes each step moves to the host: C values + columns, and the row offsets (sink mode: one
    # extra offset per output chunk, which restarts at 0)
    d2h_bytes = 12 * nnz_total + 8 * (A.nrows + (copies_total if sink_mode else 0))

    # parity spot check of the last timed step's output (sampled rows vs the oracle)
    parity = None
    if rank == 0:
        import oracle
        rows = sample_rows
        E = oracle.spgemm(A, B, rows=rows)
        if sink_mode:
            got = [out.kept.get(int(r), (np.zeros(0, np.int32), np.zeros(0))) for r in rows]
            gp = np.concatenate([[0], np.cumsum([len(g[0]) for g in got])])
            gc = np.concatenate([g[0] for g in got]) if got else np.zeros(0, np.int32)
            gv = np.concatenate([g[1] for g in got]) if got else np.zeros(0)
            res = oracle.compare(gp, gc, gv, E)
        else:
            hrp, hcol, hval = out.rp.numpy(), out.col.numpy(), out.val.numpy()
            lr = rows - r0
            base = int(hrp[0])
            gp = np.concatenate([[0], np.cumsum(hrp[lr + 1] - hrp[lr])])
            idx = np.concatenate([np.arange(hrp[k] - base, hrp[k + 1] - base) for k in lr])
            res = oracle.compare(gp, hcol[idx], hval[idx], E)
        parity = {"sampled_rows": int(len(rows)), "ok": bool(res["ok"]), "worst_ratio": res["worst_ratio"],
                  "rule": "oracle.compare: row_ptr and col bit-identical, |c - ref| <= 1e-12 sum|a*b|",
                  "nnz_c_total_matches_closed_form": None}
        if args.config == 1:
            from tests import closed_forms as CF
            p, z = CF.c2_totals(args.n)
            parity["nnz_c_total_matches_closed_form"] = bool(z == nnz_total and p == products_total)

    # roofline of the dominant kernel: algorithmic bytes of its launches in the last timed step
    # (per-row figures of DESIGN.md §7, rows assigned to tiers exactly as the kernels do) / its
    # CUDA-event time on the launching stream in that step
    kern = {k: v for k, v in stats.items()
            if k in ("count", "sym_w", "sym_m", "sym_b", "sym_g", "scan", "num_w", "num_m", "num_b", "num_g")}
    dom = max(kern, key=lambda k: kern[k]["ms"]) if kern else None
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:  # noqa: BLE001
        pass
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0))
    peak_src = ("measured: MEASURED_PEAKS.json hbm_gbs (driver-written copy bandwidth)" if "hbm_gbs" in peaks
                else "fallback 6.65 TB/s (B200_PROFILING.md)")
    roof = None
    if dom is not None and out.rownnz is not None:
        tb = {}
        tb.update(tier_bytes(A, u_np, out.rownnz, r0, r1, info, "num"))
        tb.update(tier_bytes(A, u_np, out.rownnz, r0, r1, info, "sym"))
        per_kernel = {}
        for k, v in kern.items():
            b = tb.get(k, {}).get("bytes")
            per_kernel[k] = {"ms": round(v["ms"], 3), "launches": v["launches"],
                             "alg_bytes": b, "GBps": (b / (v["ms"] / 1e3) / 1e9) if (b and v["ms"] > 0) else None,
                             "rows": tb.get(k, {}).get("rows"), "products": tb.get(k, {}).get("products")}
        byts = tb.get(dom, {}).get("bytes", 0.0)
        ms_dom = kern[dom]["ms"]
        ach = byts / (ms_dom / 1e3) / 1e9 if ms_dom > 0 else 0.0
        nl = max(1, kern[dom]["launches"])
        roof = {"bound": "hbm", "kernel": dom, "achieved": ach, "peak": hbm_peak, "unit": "GB/s",
                "frac": ach / hbm_peak, "traffic": None, "peak_source": peak_src,
                "bytes_per_launch": byts / nl, "launches": nl,
                "avg_launch_ms": ms_dom / nl,
                "bytes_rule": "algorithmic, per row of the tier: 16 B row offsets + 28 B per A entry (col, val, "
                              "B row_ptr pair) + 12 B per intermediate product (B col + val) + 12 B per C "
                              "nonzero (numeric); symbolic: 20 + 20 per A entry + 4 per product (DESIGN.md §7)",
                "share_of_step": ms_dom / (t_max / args.steps) if t_max else None,
                "kernel_times_from": "CUDA events on the launching stream, last timed step (read after the timed "
                                     "region); kernels of different streams overlap",
                "per_kernel": per_kernel}
        tf = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tf):
            try:
                tr = json.load(open(tf)).get(f"{dom}@config{args.config}")
                if tr and tr.get("source_digest") == source_digest():
                    roof["traffic"] = tr["dram_bytes_per_launch"]
                    roof["traffic_alg_bytes_per_launch"] = tr.get("alg_bytes_per_launch")
                    roof["traffic_source"] = tr.get("source")
                    roof["binding_unit"] = tr.get("binding_unit")
                elif tr:
                    roof["traffic_note"] = "profiles/traffic.json entry measured on other kernel sources: not reported"
            except Exception:  # noqa: BLE001
                pass

    # e2e: host operands through the public API (H2D of A=B + D2H of C inside the timed region)
    e2e = None
    e2e_steps = args.e2e_steps or args.steps
    if not args.no_e2e:
        hA = W.CSR(A.nrows, A.ncols, torch.from_numpy(A.row_ptr).pin_memory(), torch.from_numpy(A.col).pin_memory(),
                   torch.from_numpy(A.val).pin_memory())
        hB = hA if same else W.CSR(B.nrows, B.ncols, torch.from_numpy(B.row_ptr).pin_memory(),
                                   torch.from_numpy(B.col).pin_memory(), torch.from_numpy(B.val).pin_memory())
        h2d = 8 * (B.nrows + 1) + 12 * B.nnz + (0 if same else 8 * (A.nrows + 1) + 12 * A.nnz)

        # host operands at N = 1: the library copies them into its arena, so the arena is the whole
        # budget (C2: 2 GiB = operands + the arena of the device-operand runs)
        ws_e2e = torch.empty(wbytes + in_bytes, dtype=torch.uint8, device=dev) if (budget and world == 1) else ws

        def e2e_step():
            if world == 1:
                P = capi.Plan(hA, hB, ws_e2e.numel(), mk_opts(workspace=ws_e2e))
            else:
                # B from pinned host memory: every rank uploads 1/world of each array over its own
                # host link, an all-gather over NVLink (NCCL) assembles B on every GPU
                hb = [hB.row_ptr, hB.col, hB.val]
                if cdev is not None:
                    pdist.scatter_allgather_csr(hb, dB.store)
                else:  # gloo control-flow test (several ranks on one GPU): stage through host tensors
                    st = [x.cpu() for x in dB.store]
                    pdist.scatter_allgather_csr(hb, st)
                    for x, y in zip(dB.store, st):
                        x.copy_(y)
                if not same:  # A: only this rank's row panel goes up
                    p0, p1 = int(A.row_ptr[r0]), int(A.row_ptr[r1])
                    dA.row_ptr[r0:r1 + 1].copy_(hA.row_ptr[r0:r1 + 1], non_blocking=True)
                    dA.col[p0:p1].copy_(hA.col[p0:p1], non_blocking=True)
                    dA.val[p0:p1].copy_(hA.val[p0:p1], non_blocking=True)
                P = capi.Plan(dA, dB, wbytes, mk_opts())
            z = out.run(P)
            if world > 1 and not sink_mode:
                b, _ = pdist.slice_bases(z, device=cdev)
                capi.rebase_host(out.rp, b)
            P.free()

        for _ in range(max(1, min(args.warmup, 2))):
            e2e_step()
        barrier()
        f0 = torch.cuda.Event(enable_timing=True)
        f1 = torch.cuda.Event(enable_timing=True)
        f0.record(stream)
        for _ in range(e2e_steps):
            e2e_step()
        f1.record(stream)
        barrier()
        ems = f0.elapsed_time(f1)
        if world > 1:
            t = torch.tensor([ems], dtype=torch.float64, device=cdev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ems = float(t.item())
        e2e = {"value": 2.0 * products_total * e2e_steps / (ems / 1e3) / 1e9, "unit": "GFLOP/s",
               "h2d_bytes_per_step": int(h2d),  # over all ranks (each rank uploads 1/world of B)
               "d2h_bytes_per_step": int(d2h_bytes), "ms_per_step": ems / e2e_steps, "steps": e2e_steps,
               "api": "spgemm_plan(host A, B) + spgemm_execute_stream (sink) + spgemm_free" if sink_mode
               else "spgemm_plan(host A, B) + spgemm_execute_capacity + spgemm_free"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        c = cpu_sample(A, B, args.cpu_seconds)
        cpu = {k: c[k] for k in ("value", "unit", "cores", "kind", "sample")}

    if rank == 0:
        link = json.load(open(os.path.join(ROOT, "profiles", "hostlink.json"))) if os.path.exists(
            os.path.join(ROOT, "profiles", "hostlink.json")) else {}
        link_gbs = float(link_live) if link_live else float(link.get("d2h_GBps", 57.2))
        link_src = ("measured live in this run: copy-engine D2H of one output chunk's size into pinned memory, "
                    "best of 2" if link_live else "profiles/hostlink.json (another box)")
        bound_ms = d2h_bytes / (link_gbs * world) / 1e6
        in_l2 = "inputs ({:.2f} GB) and output ({:.1f} GB) larger than the 126 MB L2: no flush needed".format(
            in_bytes / 1e9, d2h_bytes / 1e9)
        line = {
            "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t_max / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic (seeded generator of BASELINE.json's configuration; DESIGN.md §5)",
            "config": {"workload": name, "config_index": args.config, "budget_bytes": budget or wbytes,
                       "m": A.nrows, "n": B.ncols, "nnz_A": A.nnz, "nnz_B": B.nnz,
                       "products": products_total, "nnz_C": nnz_total, "C_host_bytes": d2h_bytes,
                       "output": "sink (pinned staging ring, chunks dropped: C exceeds host memory)" if sink_mode
                       else "pinned host CSR", "chunks": info["num_chunks"], "output_copies": info["num_copies"],
                       "ring": args.ring, "chunk_nnz": chunk_nnz or None,
                       "plan": "fused (per-chunk symbolic overlapped with D2H)" if fused else "two-phase",
                       "l2": in_l2, "parallelism": f"row panels x{world} (flop-balanced)",
                       "generator_s": round(gen_s, 2)},
            "gpu_launches": int(launches),
            "clocks": clk.summary(),
            "roofline": roof,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "d2h": {"bytes_per_step": d2h_bytes, "achieved_GBps": d2h_bytes / (t_max / args.steps / 1e3) / 1e9,
                    "host_link_GBps": link_gbs, "host_link_source": link_src, "host_link_bound_ms": bound_ms,
                    "frac_of_link_bound": bound_ms / (t_max / args.steps)},
            "d2h_detail": d2h_detail(tl, 12 * nnz_local + 8 * (r1 - r0)),
            "tiers": {"rows_warp": info["rows_warp"], "rows_block": info["rows_block"],
                      "rows_global": info["rows_global"], "max_row_nnz": info["max_row_nnz"]},
            "wall_s_timed": wall,
            "host_ms_per_step": {k: round(float(np.median(v)), 3) for k, v in host_ms.items() if v},
            "pinned_output_alloc_s": pin_s,
            "parity": parity,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
