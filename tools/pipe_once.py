"""Run the C2 fused multiply a few times (for nsys / ncu captures; prints nothing else)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import workloads as W
from paper_conf_ipps_xia0ar21_b200 import capi

n = int(os.environ.get("N", "128")); reps = int(os.environ.get("REPS", "3"))
fused = os.environ.get("FUSED", "1") == "1"
A = W.stencil_3d27(n)
dev = torch.device("cuda", 0)
class D: pass
d = D(); d.nrows, d.ncols = A.nrows, A.ncols
d.row_ptr = torch.from_numpy(A.row_ptr).to(dev); d.col = torch.from_numpy(A.col).to(dev); d.val = torch.from_numpy(A.val).to(dev)
inb = 8 * (A.nrows + 1) + 12 * A.nnz
ws = torch.empty((2 << 30) - inb, dtype=torch.uint8, device=dev)
s = torch.cuda.current_stream()
with capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream)) as P:
    z = P.info()["nnz"]
rp = torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True)
col = torch.empty(z, dtype=torch.int32, pin_memory=True)
val = torch.empty(z, dtype=torch.float64, pin_memory=True)
for r in range(reps):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    P = capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream, fused=fused, ring=int(os.environ.get("RING", "2"))))
    if fused:
        P.execute_capacity(rp, col, val, z)
    else:
        P.execute_into(rp, col, val)
    P.free(); torch.cuda.synchronize()
    print(f"rep {r}: {1e3 * (time.perf_counter() - t0):.2f} ms", flush=True)
