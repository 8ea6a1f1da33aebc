"""Pipeline ablations on C2 (27-pt 128^3, 2 GiB budget, device operands) -- the analogue of the
paper's synchronous-vs-asynchronous comparison (Fig. 8, §IV).  Each variant is run
through the same C ABI call as the bench step (plan + execute into pinned host C); best of 3.

  async (default)      ring 2, fused plan, analysis stream, output chunks grown online
  sync                 ring 1: the numeric pass of the next unit waits for the copy of the last
                       (the paper's synchronous partitioned baseline, its Fig. 4 / Fig. 8 'sync')
  serial_analysis      ring 2, symbolic passes on the compute stream (no analysis/numeric overlap)
  one_copy_per_unit    ring 2, every analysis unit leaves as its own copies (no output chunks)
  two_phase            ring 2, symbolic for all rows inside spgemm_plan, then execute
  two_phase_flops_order  two_phase with the paper's chunk schedule: decreasing flops (§IV-C)
  ring3                ring 3
WL=c2 (default) or WL=rmatNN (R-MAT scale NN, C = A*A).  Writes gpurun_out/ablation_<WL>.json and prints it."""
import json, os, subprocess, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

VARIANTS = {
    "async": ({}, dict(ring=2, fused=True)),
    "sync": ({}, dict(ring=1, fused=True)),
    "serial_analysis": ({"SPGEMM_SERIAL_ANALYSIS": "1"}, dict(ring=2, fused=True)),
    "one_copy_per_unit": ({"SPGEMM_NO_GROUPS": "1"}, dict(ring=2, fused=True)),
    "two_phase": ({}, dict(ring=2, fused=False)),
    "two_phase_flops_order": ({}, dict(ring=2, fused=False, order=1)),
    "ring3": ({}, dict(ring=3, fused=True)),
}

if len(sys.argv) > 1:  # child: one variant
    import numpy as np
    import torch
    import workloads as W
    from paper_conf_ipps_xia0ar21_b200 import capi
    kw = json.loads(sys.argv[1])
    wl = os.environ.get("WL", "c2")
    A = W.stencil_3d27(128) if wl == "c2" else W.rmat_torch(int(wl[4:]))
    dev = torch.device("cuda", 0)
    class D: pass
    d = D(); d.nrows, d.ncols = A.nrows, A.ncols
    d.row_ptr = torch.from_numpy(A.row_ptr).to(dev); d.col = torch.from_numpy(A.col).to(dev); d.val = torch.from_numpy(A.val).to(dev)
    ws = torch.empty((2 << 30) - (8 * (A.nrows + 1) + 12 * A.nnz), dtype=torch.uint8, device=dev)
    s = torch.cuda.current_stream()
    with capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream)) as P:
        z = P.info()["nnz"]; prods = P.info()["products"]
    rp = torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True)
    col = torch.empty(z, dtype=torch.int32, pin_memory=True)
    val = torch.empty(z, dtype=torch.float64, pin_memory=True)
    best = 1e9
    for rep in range(4):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        P = capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream, **kw))
        if kw["fused"]:
            P.execute_capacity(rp, col, val, z)
        else:
            P.execute_into(rp, col, val)
        copies = P.info()["num_copies"]; units = P.info()["num_chunks"]
        P.free(); torch.cuda.synchronize()
        if rep:
            best = min(best, time.perf_counter() - t0)
    print(json.dumps({"ms": 1e3 * best, "gflops": 2 * prods / best / 1e9, "units": units, "copies": copies}))
else:
    out = {}
    for name, (env, kw) in VARIANTS.items():
        r = subprocess.run([sys.executable, __file__, json.dumps(kw)], env={**os.environ, **env},
                           capture_output=True, text=True)
        out[name] = json.loads(r.stdout.strip().splitlines()[-1]) if r.returncode == 0 else {"error": r.stderr[-400:]}
    out["async_vs_sync_speedup"] = out["sync"]["ms"] / out["async"]["ms"] if "ms" in out.get("sync", {}) else None
    os.makedirs("gpurun_out", exist_ok=True)
    out["workload"] = os.environ.get("WL", "c2")
    json.dump(out, open(f"gpurun_out/ablation_{out['workload']}.json", "w"), indent=1)
    print(json.dumps(out, indent=1))
