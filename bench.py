"""bench.py -- C = A*A GFLOP/s (2 x intermediate products) including the D2H of all of C.

Default workload (N = 1): BASELINE.json configs[1] = 3-D 27-point stencil 128^3, device budget
forced to 2 GiB, so C (3.07 GB) is produced out-of-core in chunks and streamed to pinned host
memory.  One step = the whole hot path (DESIGN.md §8 rows S0-S10): plan (count, symbolic,
scan, chunk cut) + execute (numeric + sort per chunk, D2H overlapped) through the C ABI.

  value  inputs resident in HBM when the timed region starts (device operands, where=DEVICE);
  e2e    the same through the public API with HOST operands: the H2D of A (= B) from pinned
         memory and the D2H of C are inside the timed region.

Multi-GPU (torchrun, one rank per GPU): rows of A are dealt as contiguous panels; in the e2e
step every rank uploads 1/world of B over its own host link and an NCCL all-gather over NVLink
assembles B on every GPU; each rank's nnz is all-gathered for the global row_ptr base; every rank
drains its own rows of C.  Total work is fixed -> scaling "strong".

--impl reference runs the CPU oracle (the reference arm of this tier) on bounded samples.
"""
from __future__ import annotations

import argparse
import json
import os
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
    ap.add_argument("--config", type=int, default=1, help="BASELINE.json configs index (1 = 27-pt 128^3, 2 GiB)")
    ap.add_argument("--n", type=int, default=128, help="stencil edge for config 1")
    ap.add_argument("--ring", type=int, default=2)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--two-phase", action="store_true", help="time the two-phase plan/execute path at N = 1")
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
                                       "--format=csv,noheader,nounits", "-lms", "100"],
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
        sm = [float(r[1]) for r in self.rows if len(r) > 8 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) > 8 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            if len(r) > 8:
                for k, nm in enumerate(names):
                    if r[5 + k].lower().startswith("active"):
                        reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows)}


def probe_d2h(h_dsts, dev, reps=2):
    """This box's pinned D2H rate (GB/s) for exactly this step's output, measured in this process
    just before the timed region: plain copy-engine copies from HBM into the bench's own pinned
    output buffers (all of them, whole), best of `reps`, CUDA events on a side stream.  The link
    bound of the step is judged against it (a 1 GiB copy into one buffer reads up to ~10 % faster
    than the sustained rate into all of the step's host memory on some boxes)."""
    import torch
    hbs = [h.view(torch.uint8) for h in h_dsts if h.numel() > 0]
    total = sum(h.numel() for h in hbs)
    if total < (1 << 20):
        return None
    src = torch.empty(max(h.numel() for h in hbs), dtype=torch.uint8, device=dev)
    src.fill_(7)
    s = torch.cuda.Stream(device=dev)
    best = None
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record(s)
            for h in hbs:
                h.copy_(src[:h.numel()], non_blocking=True)
            e1.record(s)
        s.synchronize()
        t = e0.elapsed_time(e1) / 1e3
        best = t if best is None else min(best, t)
    del src
    return total / best / 1e9


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


def load_config(args):
    if args.config == 1:
        A = W.stencil_3d27(args.n)
        return A, A, BUDGET_C2, f"C2: 3-D 27-point stencil {args.n}^3, C=A*A, device budget 2 GiB (out-of-core)"
    A, B, budget, name = W.config(args.config)
    return A, B, budget or 0, name


def launch_bytes(A, B, rows, offs, r0, kind):
    """Bytes of each numeric ("num") or symbolic ("sym") launch (one per analysis unit), two ways
    (DESIGN.md §7 "Roofline"):
      algorithmic  SURVEY §8(a) S4/S6's per-unit figures, i.e. what Gustavson's row-by-row
                   formulation (Alg. 1) reads and writes: the A panel (row_ptr + col
                   [+ val]), one B entry per intermediate product (col [+ val]: 4 or 12 B), the
                   B row_ptr pair per A entry, and the unit's output (C col + val, or nnz per row);
      compulsory   every byte touched once: the A panel, each B row the panel touches read ONCE,
                   the output once -- the floor the L2 (126 MB) makes reachable.
    Returns (algorithmic list, compulsory list)."""
    bl = np.diff(B.row_ptr)
    vb = 12.0 if kind == "num" else 4.0
    alg, comp = [], []
    for c in range(len(rows) - 1):
        a0, a1 = r0 + rows[c], r0 + rows[c + 1]
        p0, p1 = int(A.row_ptr[a0]), int(A.row_ptr[a1])
        cols = A.col[p0:p1]
        touched = np.unique(cols)
        nr, na = a1 - a0, p1 - p0
        prods = float(bl[cols].sum())
        out = 12.0 * float(offs[c + 1] - offs[c]) if kind == "num" else 4.0 * nr
        a_b = 8.0 * (nr + 1) + (12.0 if kind == "num" else 4.0) * na + 8.0 * nr  # + C row offsets / bounds
        alg.append(a_b + 16.0 * na + vb * prods + out)
        comp.append(a_b + 16.0 * len(touched) + vb * float(bl[touched].sum()) + out)
    return alg, comp


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
    A, B, budget, name = load_config(args)
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
    A, B, budget, name = load_config(args)
    same = A is B
    panels = pdist.row_panels(A.row_ptr, world)
    r0, r1 = panels[rank]

    class Dev:
        pass

    def to_dev(M):
        # storage padded to a multiple of the world size: the e2e step refills these arrays with a
        # scatter (each rank uploads 1/world) + all-gather over NVLink (dist.scatter_allgather_csr)
        d = Dev()
        d.nrows, d.ncols = M.nrows, M.ncols
        d.store = []
        for name, x in (("row_ptr", M.row_ptr), ("col", M.col), ("val", M.val)):
            t = torch.from_numpy(x)
            buf = torch.zeros(pdist.padded_len(t.numel(), world), dtype=t.dtype, device=dev)
            buf[:t.numel()].copy_(t)
            d.store.append(buf)
            setattr(d, name, buf[:t.numel()])
        return d

    dB = to_dev(B)
    dA = dB if same else to_dev(A)
    # the budget covers every device byte of the multiply (reading R15): with resident
    # operands the arena gets the budget minus the operands' bytes
    in_bytes = 8 * (B.nrows + 1) + 12 * B.nnz + (0 if same else 8 * (A.nrows + 1) + 12 * A.nnz)
    ws = torch.empty((budget - in_bytes) if budget else int(torch.cuda.mem_get_info()[0] * 0.85),
                     dtype=torch.uint8, device=dev)
    wbytes = ws.numel()
    stream = torch.cuda.current_stream()

    # Fused plans (per-chunk symbolic overlapped with the previous chunk's D2H, the call
    # spgemm_multiply makes).  With N > 1 ranks each rank's global row_ptr base is the sum of the
    # earlier ranks' nnz, known after execution: an 8-byte all_gather, then spgemm_rebase_host on
    # the rank's row_ptr slice.  --two-phase: plans whose symbolic pass runs in spgemm_plan.
    fused = not args.two_phase

    def mk_opts(profile=False, base=0):
        return capi.opts(device=local, ring=args.ring, profile=profile, row_begin=r0, row_end=r1, workspace=ws,
                         stream=stream.cuda_stream, row_ptr_base=base, fused=fused)

    ws_e2e = None

    def mk_opts_e2e():
        # host operands: the library copies them into the arena, so the arena is the whole budget
        nonlocal ws_e2e
        if ws_e2e is None:
            ws_e2e = torch.empty(wbytes + in_bytes, dtype=torch.uint8, device=dev)
        return capi.opts(device=local, ring=args.ring, row_begin=r0, row_end=r1, workspace=ws_e2e,
                         stream=stream.cuda_stream, fused=fused)

    # untimed: sizes, global base, pinned outputs (pinning is a one-time cost, reported separately)
    with capi.Plan(dA, dB, wbytes, capi.opts(device=local, ring=args.ring, row_begin=r0, row_end=r1, workspace=ws,
                                             stream=stream.cuda_stream)) as P:
        info = P.info()
    nnz_local = info["nnz"]
    base = 0
    if world > 1:
        base, nnz_total = pdist.slice_bases(nnz_local, device=cdev)
    else:
        nnz_total = nnz_local
    t0 = time.perf_counter()
    h_rp = torch.empty(r1 - r0 + 1, dtype=torch.int64, pin_memory=True)
    h_col = torch.empty(nnz_local, dtype=torch.int32, pin_memory=True)
    h_val = torch.empty(nnz_local, dtype=torch.float64, pin_memory=True)
    pin_s = time.perf_counter() - t0

    chunk_table = {}

    host_ms = {"plan": [], "execute": [], "free": []}

    def step(profile=False, keep=False):
        """One multiply (plan + execute + free).  keep: return the plan unfreed, so that its
        kernel times (CUDA events recorded inside the step) are read after the timed region."""
        h0 = time.perf_counter()
        P = capi.Plan(dA, dB, wbytes, mk_opts(profile))
        h1 = time.perf_counter()
        if fused:
            z = P.execute_capacity(h_rp, h_col, h_val, nnz_local)
            if world > 1:
                b, _ = pdist.slice_bases(z, device=cdev)
                capi.rebase_host(h_rp, b)
        else:
            if world > 1:
                b, _ = pdist.slice_bases(P.info()["nnz"], device=cdev)
                P.set_row_ptr_base(b)
            P.execute_into(h_rp, h_col, h_val)
        h2 = time.perf_counter()
        host_ms["plan"].append(1e3 * (h1 - h0))
        host_ms["execute"].append(1e3 * (h2 - h1))
        if keep:
            return P
        P.free()
        host_ms["free"].append(1e3 * (time.perf_counter() - h2))
        return None

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        step(profile=True)
    barrier()
    for v in host_ms.values():
        v.clear()
    link_live = probe_d2h([h_col, h_val], dev)
    launches0 = capi.kernel_launches()
    stats = []
    with Clocks(local) as clk:
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        w0 = time.perf_counter()
        e0.record(stream)
        for k in range(args.steps):
            last = step(profile=True, keep=(k == args.steps - 1))
        e1.record(stream)
        barrier()
        wall = time.perf_counter() - w0
    # kernel times of the last timed step (its events were recorded inside the timed region)
    stats.append(last.stats())
    tl = capi.timeline(last)  # [chunk, 6] ms: analysis, numeric and copy start/end
    chunk_table["rows"], chunk_table["offs"] = last.chunks()
    chunk_table["info"] = last.info()
    last.free()
    nstat = len(stats)
    launches = capi.kernel_launches() - launches0
    ms = e0.elapsed_time(e1)
    t_max = ms
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=cdev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        t_max = float(t.item())
    products_total = info["products"]
    if world > 1:
        products_total = pdist.slice_bases(info["products"], device=cdev)[1]
    value = 2.0 * products_total * args.steps / (t_max / 1e3) / 1e9

    # parity spot check of the last step's output (sampled rows vs the oracle)
    parity = None
    if rank == 0:
        import oracle
        rng = np.random.default_rng(1)
        nloc = r1 - r0
        rows = np.unique(np.concatenate([[0, nloc - 1], rng.integers(0, max(nloc, 1), 64)])) if nloc else np.zeros(0, int)
        E = oracle.spgemm(A, B, rows=rows + r0)
        hrp, hcol, hval = h_rp.numpy(), h_col.numpy(), h_val.numpy()
        gp = np.concatenate([[0], np.cumsum(hrp[rows + 1] - hrp[rows])])
        idx = np.concatenate([np.arange(hrp[r] - base, hrp[r + 1] - base) for r in rows]) if len(rows) else []
        res = oracle.compare(gp, hcol[idx], hval[idx], E)
        parity = {"sampled_rows": int(len(rows)), "ok": bool(res["ok"]), "worst_ratio": res["worst_ratio"],
                  "nnz_c_total_matches_closed_form": None}
        if args.config == 1:
            from tests import closed_forms as CF
            p, z = CF.c2_totals(args.n)
            parity["nnz_c_total_matches_closed_form"] = bool(z == nnz_total and p == products_total)

    # roofline of the dominant kernel, from the library's CUDA events on the launching stream
    agg = {}
    for st in stats:
        for k, v in st.items():
            a = agg.setdefault(k, {"launches": 0, "ms": 0.0})
            a["launches"] += v["launches"]
            a["ms"] += v["ms"]
    kern = {k: v for k, v in agg.items() if k in ("count", "sym_w", "sym_b", "sym_g", "scan", "num_w", "num_b", "num_g")}
    dom = max(kern, key=lambda k: kern[k]["ms"]) if kern else None
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:  # noqa: BLE001
        pass
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0))
    peak_src = "measured (MEASURED_PEAKS.json hbm_gbs)" if "hbm_gbs" in peaks else "fallback 6.65 TB/s"
    roof = None
    if dom is not None:
        byts = byts_c = 0.0
        if dom[:3] in ("num", "sym"):
            alg, comp = launch_bytes(A, B, chunk_table["rows"], chunk_table["offs"], r0, dom[:3])
            byts, byts_c = float(np.sum(alg)) * nstat, float(np.sum(comp)) * nstat
        ms_dom = kern[dom]["ms"]
        ach = byts / (ms_dom / 1e3) / 1e9 if ms_dom > 0 else 0.0
        ach_c = byts_c / (ms_dom / 1e3) / 1e9 if ms_dom > 0 else 0.0
        nl = max(1, kern[dom]["launches"])
        roof = {"bound": "hbm", "kernel": dom, "achieved": ach, "peak": hbm_peak, "unit": "GB/s",
                "frac": ach / hbm_peak, "traffic": None, "peak_source": peak_src,
                "bytes_per_launch": byts / nl,
                "bytes_rule": "algorithmic: SURVEY S6/S4 per-unit figures (A panel, 12 B (num) / 4 B (sym) of B "
                              "per intermediate product, B row_ptr pair per A entry, C out) -- DESIGN.md §7",
                "achieved_compulsory": ach_c, "frac_compulsory": ach_c / hbm_peak,
                "bytes_per_launch_compulsory": byts_c / nl,
                "avg_launch_ms": ms_dom / max(1, kern[dom]["launches"]),
                "share_of_step": (ms_dom / nstat) / (t_max / args.steps) if t_max else None,
                "per_kernel_ms_per_step": {k: v["ms"] / nstat for k, v in agg.items()},
                "kernel_times_from": "CUDA events of the last timed step (read after the timed region)"}
        tf = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tf):
            try:
                tr = json.load(open(tf)).get(dom)
                if tr:
                    roof["traffic"] = tr["bytes_per_launch"]
                    roof["traffic_source"] = tr.get("source")
                    if "lsu_pipe_frac_of_peak" in tr:  # the unit that actually binds the hash kernels
                        roof["binding_unit"] = {"unit": "LSU data pipe (shared memory + L1)",
                                                "frac_of_peak": tr["lsu_pipe_frac_of_peak"],
                                                "sm_throughput_frac": tr.get("sm_throughput_frac"),
                                                "source": tr.get("source")}
            except Exception:  # noqa: BLE001
                pass

    # e2e: host operands through the public API (H2D of A=B + D2H of C inside the timed region)
    e2e = None
    if not args.no_e2e:
        hA = W.CSR(A.nrows, A.ncols, torch.from_numpy(A.row_ptr).pin_memory(), torch.from_numpy(A.col).pin_memory(),
                   torch.from_numpy(A.val).pin_memory())
        hB = hA if same else W.CSR(B.nrows, B.ncols, torch.from_numpy(B.row_ptr).pin_memory(),
                                   torch.from_numpy(B.col).pin_memory(), torch.from_numpy(B.val).pin_memory())
        h2d = 8 * (B.nrows + 1) + 12 * B.nnz + (0 if same else 8 * (A.nrows + 1) + 12 * A.nnz)

        def e2e_step():
            if world == 1:
                P = capi.Plan(hA, hB, wbytes + in_bytes, mk_opts_e2e())
                if fused:
                    P.execute_capacity(h_rp, h_col, h_val, nnz_local)
                    P.free()
                    return
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
                if fused:
                    z = P.execute_capacity(h_rp, h_col, h_val, nnz_local)
                    b, _ = pdist.slice_bases(z, device=cdev)
                    capi.rebase_host(h_rp, b)
                    P.free()
                    return
                b, _ = pdist.slice_bases(P.info()["nnz"], device=cdev)
                P.set_row_ptr_base(b)
            P.execute_into(h_rp, h_col, h_val)
            P.free()

        for _ in range(max(1, args.warmup)):
            e2e_step()
        barrier()
        f0 = torch.cuda.Event(enable_timing=True)
        f1 = torch.cuda.Event(enable_timing=True)
        f0.record(stream)
        for _ in range(args.steps):
            e2e_step()
        f1.record(stream)
        barrier()
        ems = f0.elapsed_time(f1)
        if world > 1:
            t = torch.tensor([ems], dtype=torch.float64, device=cdev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ems = float(t.item())
        e2e = {"value": 2.0 * products_total * args.steps / (ems / 1e3) / 1e9, "unit": "GFLOP/s",
               "h2d_bytes_per_step": int(h2d),  # over all ranks (each rank uploads 1/world of B)
               "d2h_bytes_per_step": int(12 * nnz_total + 8 * (A.nrows + 1)), "ms_per_step": ems / args.steps}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        c = cpu_sample(A, B, args.cpu_seconds)
        cpu = {k: c[k] for k in ("value", "unit", "cores", "kind", "sample")}

    if rank == 0:
        d2h_bytes = 12 * nnz_total + 8 * (A.nrows + 1)
        link = json.load(open(os.path.join(ROOT, "profiles", "hostlink.json"))) if os.path.exists(
            os.path.join(ROOT, "profiles", "hostlink.json")) else {}
        link_gbs = float(link_live) if link_live else float(link.get("d2h_GBps", 57.2))
        link_src = ("measured live in this run: copy-engine D2H of the step's output size into the step's own "
                    "pinned buffers, best of 2" if link_live
                    else "profiles/hostlink.json (another box)")
        bound_ms = d2h_bytes / (link_gbs * world) / 1e6
        line = {
            "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t_max / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": name, "budget_bytes": budget, "m": A.nrows, "nnz_A": A.nnz,
                       "products": products_total, "nnz_C": nnz_total, "C_host_bytes": d2h_bytes,
                       "chunks": chunk_table["info"]["num_chunks"], "output_copies": chunk_table["info"]["num_copies"],
                       "ring": args.ring,
                       "plan": "fused (per-chunk symbolic overlapped with D2H)" if fused else "two-phase",
                       "l2": "inputs (686 MB) and output (3.07 GB) larger than L2; no flush needed",
                       "parallelism": f"row panels x{world}"},
            "gpu_launches": int(launches),
            "clocks": clk.summary(),
            "roofline": roof,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "d2h": {"bytes_per_step": d2h_bytes, "achieved_GBps": d2h_bytes / (t_max / args.steps / 1e3) / 1e9,
                    "host_link_GBps": link_gbs, "host_link_source": link_src, "host_link_bound_ms": bound_ms,
                    "frac_of_link_bound": bound_ms / (t_max / args.steps)},
            "d2h_detail": d2h_detail(tl, d2h_bytes),
            "wall_s_timed": wall,
            "host_ms_per_step": {k: round(float(np.median(v)), 3) for k, v in host_ms.items() if v}, "pinned_output_alloc_s": pin_s,
            "parity": parity,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
