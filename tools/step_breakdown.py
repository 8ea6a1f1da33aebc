"""Host-wall breakdown of one bench step (C2, device operands): Plan(), execute_capacity(),
stats(), free(), with profile mode on and off.  Diagnostic for the gap between the bench's
ms_per_step and the pipeline's execute_total."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import workloads as W
from paper_conf_ipps_xia0ar21_b200 import capi

n = int(os.environ.get("N", "128"))
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
out = {}
for profile in (False, True):
    rows = []
    for rep in range(6):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        P = capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream, fused=True, profile=profile))
        t1 = time.perf_counter()
        P.execute_capacity(rp, col, val, z)
        t2 = time.perf_counter()
        st = P.stats() if profile else {}
        t3 = time.perf_counter()
        P.free()
        t4 = time.perf_counter()
        torch.cuda.synchronize()
        t5 = time.perf_counter()
        rows.append([1e3 * (t1 - t0), 1e3 * (t2 - t1), 1e3 * (t3 - t2), 1e3 * (t4 - t3), 1e3 * (t5 - t0),
                     st.get("execute_total", {}).get("ms", 0.0), st.get("plan_device_span", {}).get("ms", 0.0)])
    r = np.median(np.array(rows[1:]), axis=0)
    out["profile" if profile else "plain"] = dict(zip(
        ["plan_ms", "execute_ms", "stats_ms", "free_ms", "step_ms", "execute_total_ev_ms", "plan_device_span_ms"],
        [round(float(x), 3) for x in r]))
print(json.dumps(out, indent=1))
