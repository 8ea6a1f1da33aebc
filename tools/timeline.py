"""Per-chunk pipeline timeline of the C2 multiply (profile mode events; diagnostic)."""
import json, os, sys
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
for label, kw in [("fused_ring2", dict(fused=True, ring=2)), ("fused_ring3", dict(fused=True, ring=3)),
                  ("twophase_ring2", dict(fused=False, ring=2))]:
    import time
    for rep in range(3):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        P = capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream, profile=True, **kw))
        t_plan = time.perf_counter() - t0
        if kw["fused"]:
            P.execute_capacity(rp, col, val, z)
        else:
            P.execute_into(rp, col, val)
        tl = capi.timeline(P)
        st = P.stats()
        P.free()
    out[label] = {"timeline": np.round(tl, 3).tolist(), "stats": st}
    t = tl
    print(label, "execute_total", st["execute_total"]["ms"], "plan_wall_ms", 1e3 * t_plan)
    for c in range(len(t)):
        print(f"  c{c:02d} sym {t[c,0]:7.3f}-{t[c,1]:7.3f}  num {t[c,2]:7.3f}-{t[c,3]:7.3f}  d2h {t[c,4]:7.3f}-{t[c,5]:7.3f}  gap {t[c,4]-(t[c-1,5] if c else 0):6.3f}")
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/timeline.json", "w"))
for label, v in out.items():
    st = v["stats"]
    print(label, {k: round(st[k]["ms"], 3) for k in ("sym_w", "num_w", "scan", "d2h_span", "execute_total") if k in st})
