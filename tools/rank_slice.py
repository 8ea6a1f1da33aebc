"""One rank's share of a strong-scaled C2 step on one GPU (diagnostic): rows [0, R/N) of the
27-pt 128^3 C = A*A with device operands, fused plan, for several min_chunks; prints ms, the
link-bound ms of the slice and the fraction.  N from env (default 8)."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import workloads as W
from paper_conf_ipps_xia0ar21_b200 import capi

N = int(os.environ.get("N", "8"))
A = W.stencil_3d27(128)
dev = torch.device("cuda", 0)
class D: pass
d = D(); d.nrows, d.ncols = A.nrows, A.ncols
d.row_ptr = torch.from_numpy(A.row_ptr).to(dev); d.col = torch.from_numpy(A.col).to(dev); d.val = torch.from_numpy(A.val).to(dev)
ws = torch.empty((2 << 30) - (8 * (A.nrows + 1) + 12 * A.nnz), dtype=torch.uint8, device=dev)
s = torch.cuda.current_stream()
r1 = A.nrows // N
with capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream, row_end=r1)) as P:
    z = P.info()["nnz"]
rp = torch.empty(r1 + 1, dtype=torch.int64, pin_memory=True)
col = torch.empty(z, dtype=torch.int32, pin_memory=True)
val = torch.empty(z, dtype=torch.float64, pin_memory=True)
src = torch.empty(z * 8, dtype=torch.uint8, device=dev)
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
best_link = 1e9
for _ in range(3):
    e0.record(s); col.view(torch.uint8).copy_(src[:z * 4], non_blocking=True); val.view(torch.uint8).copy_(src, non_blocking=True); e1.record(s)
    torch.cuda.synchronize(); best_link = min(best_link, e0.elapsed_time(e1))
out = {"N": N, "rows": r1, "nnz": z, "link_bound_ms": best_link}
for minc in [int(x) for x in os.environ.get("MINC", "0,8,16,32").split(",")]:
    best, units = 1e9, 0
    for rep in range(5):
        torch.cuda.synchronize()
        e0.record(s)
        P = capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream, fused=True, row_end=r1, min_chunks=minc))
        P.execute_capacity(rp, col, val, z)
        e1.record(s)
        units = P.info()["num_chunks"]
        P.free()
        torch.cuda.synchronize()
        if rep:
            best = min(best, e0.elapsed_time(e1))
    out[f"minc{minc}"] = {"ms": best, "units": units, "frac": best_link / best}
print(json.dumps(out))
