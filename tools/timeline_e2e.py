"""Per-chunk timeline of the C2 multiply with HOST operands (the e2e path: H2D of A = B inside
the step).  Diagnostic: prints plan host time, execute host time and the chunk timeline."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import workloads as W
from paper_conf_ipps_xia0ar21_b200 import capi

n = int(os.environ.get("N", "128"))
A = W.stencil_3d27(n)
hA = W.CSR(A.nrows, A.ncols, torch.from_numpy(A.row_ptr).pin_memory(), torch.from_numpy(A.col).pin_memory(),
           torch.from_numpy(A.val).pin_memory())
ws = torch.empty(2 << 30, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream()
with capi.Plan(hA, hA, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream)) as P:
    z = P.info()["nnz"]
rp = torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True)
col = torch.empty(z, dtype=torch.int32, pin_memory=True)
val = torch.empty(z, dtype=torch.float64, pin_memory=True)
for rep in range(4):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    P = capi.Plan(hA, hA, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream, fused=True, profile=True))
    t1 = time.perf_counter()
    P.execute_capacity(rp, col, val, z)
    t2 = time.perf_counter()
    tl = capi.timeline(P)
    rows_, offs_ = P.chunks()
    st = P.stats()
    P.free()
    torch.cuda.synchronize()
    print(f"rep {rep}: plan {1e3 * (t1 - t0):.2f} ms, execute {1e3 * (t2 - t1):.2f} ms, total {1e3 * (t2 - t0):.2f} ms;",
          {k: round(v["ms"], 3) for k, v in st.items()})
t = tl
for c in range(len(t)):
    print(f"  c{c:02d} sym {t[c,0]:7.3f}-{t[c,1]:7.3f}  num {t[c,2]:7.3f}-{t[c,3]:7.3f}  d2h {t[c,4]:7.3f}-{t[c,5]:7.3f}  gap {t[c,4]-(t[c-1,5] if c else 0):6.3f}")

# copy-engine view: busy time, idle gaps and rate while busy (copies recorded on each group's last unit)
g = [c for c in range(len(t)) if t[c, 4] >= 0]
busy = sum(t[c, 5] - t[c, 4] for c in g)
span = t[g[-1], 5] - t[g[0], 4]
nbytes = 12 * int(offs_[-1] - offs_[0])
print(f"copies {len(g)}: first start {t[g[0], 4]:.3f} ms, span {span:.3f}, busy {busy:.3f}, idle {span - busy:.3f} ms, "
      f"rate while busy {nbytes / busy / 1e6:.2f} GB/s")
