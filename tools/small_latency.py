"""Latency of small in-core multiplies (configs[0]: 2-D 5-pt 64x64, C = A*A) through the C ABI:
plan + execute with host and with device operands, fused and two-phase (diagnostic)."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import workloads as W
from paper_conf_ipps_xia0ar21_b200 import capi

A = W.stencil_2d5(64)
dev = torch.device("cuda", 0)
class D: pass
d = D(); d.nrows, d.ncols = A.nrows, A.ncols
d.row_ptr = torch.from_numpy(A.row_ptr).to(dev); d.col = torch.from_numpy(A.col).to(dev); d.val = torch.from_numpy(A.val).to(dev)
ws = torch.empty(64 << 20, dtype=torch.uint8, device=dev)
s = torch.cuda.current_stream()
z = 51972
rp = torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True)
col = torch.empty(z, dtype=torch.int32, pin_memory=True)
val = torch.empty(z, dtype=torch.float64, pin_memory=True)
out = {}
for name, M, fused in (("device_fused", d, True), ("device_two_phase", d, False), ("host_fused", A, True), ("host_two_phase", A, False)):
    ts = []
    for rep in range(30):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        P = capi.Plan(M, M, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream, fused=fused))
        t1 = time.perf_counter()
        P.execute_capacity(rp, col, val, z)
        t2 = time.perf_counter()
        P.free()
        ts.append((t1 - t0, t2 - t1))
    ts = np.array(ts[5:]) * 1e3
    out[name] = {"plan_ms": float(np.median(ts[:, 0])), "execute_ms": float(np.median(ts[:, 1])),
                 "total_ms": float(np.median(ts.sum(1)))}
    # repeated execute of one plan (two-phase only: sizes known)
with capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream)) as P:
    ts = []
    for rep in range(30):
        t0 = time.perf_counter(); P.execute_into(rp, col, val); ts.append(time.perf_counter() - t0)
    out["re_execute_ms"] = float(np.median(ts[5:]) * 1e3)
print(json.dumps(out))
