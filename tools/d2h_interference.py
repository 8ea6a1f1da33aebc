"""Copy-engine rate of the C2 pipeline vs plain chunked copies on the same box (diagnostic).

Prints, per variant, the D2H rate while the copy stream is busy (from the chunk timeline):
  pipeline          the fused multiply as the bench runs it
  pipeline_serial   SPGEMM_SERIAL_ANALYSIS=1 set by the caller (analysis on the compute stream)
and the rate of the same copies (same sizes, same destinations) with no kernels running.
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import workloads as W
from paper_conf_ipps_xia0ar21_b200 import capi

A = W.stencil_3d27(128)
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
for rep in range(4):
    P = capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream, fused=True, profile=True))
    P.execute_capacity(rp, col, val, z)
    tl = capi.timeline(P); rows, offs = P.chunks(); P.free()
busy = float(np.sum(tl[:, 5] - tl[:, 4]))
out["pipeline_rate_while_busy_GBps"] = (12 * z + 8 * A.nrows) / busy / 1e6
out["pipeline_busy_ms"] = busy
# the same copies with no kernels: chunk c -> col[offs[c]:offs[c+1]], val[...], rp[rows[c]+1 : rows[c+1]+1]
dcol = torch.empty(int(np.max(np.diff(offs))), dtype=torch.int32, device=dev)
dval = torch.empty(dcol.numel(), dtype=torch.float64, device=dev)
drp = torch.empty(int(np.max(np.diff(rows))) + 1, dtype=torch.int64, device=dev)
cs = torch.cuda.Stream()
best = 1e9
for rep in range(3):
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(cs):
        e0.record(cs)
        for c in range(len(rows) - 1):
            o0, o1 = int(offs[c]), int(offs[c + 1]); r0, r1 = int(rows[c]), int(rows[c + 1])
            col[o0:o1].copy_(dcol[:o1 - o0], non_blocking=True)
            val[o0:o1].copy_(dval[:o1 - o0], non_blocking=True)
            rp[r0 + 1:r1 + 1].copy_(drp[:r1 - r0], non_blocking=True)
        e1.record(cs)
    cs.synchronize()
    best = min(best, e0.elapsed_time(e1))
out["same_copies_no_kernels_GBps"] = (12 * z + 8 * A.nrows) / best / 1e6
def copies(with_col=True, with_val=True, with_rp=True, align=1, src_shift=0):
    best = 1e9
    nbytes = 0
    for rep in range(3):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        nbytes = 0
        with torch.cuda.stream(cs):
            e0.record(cs)
            for c in range(len(rows) - 1):
                o0, o1 = int(offs[c]) // align * align, int(offs[c + 1]) // align * align
                r0, r1 = int(rows[c]), int(rows[c + 1])
                if with_col:
                    col[o0:o1].copy_(dcol[src_shift:src_shift + o1 - o0], non_blocking=True); nbytes += 4 * (o1 - o0)
                if with_val:
                    val[o0:o1].copy_(dval[src_shift:src_shift + o1 - o0], non_blocking=True); nbytes += 8 * (o1 - o0)
                if with_rp:
                    rp[r0 + 1:r1 + 1].copy_(drp[:r1 - r0], non_blocking=True); nbytes += 8 * (r1 - r0)
            e1.record(cs)
        cs.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return nbytes / best / 1e6
dcol = torch.empty(dcol.numel() + 64, dtype=torch.int32, device=dev)
dval = torch.empty(dcol.numel(), dtype=torch.float64, device=dev)
out["no_rp_GBps"] = copies(with_rp=False)
out["val_only_GBps"] = copies(with_col=False, with_rp=False)
out["col_only_GBps"] = copies(with_val=False, with_rp=False)
out["aligned32_no_rp_GBps"] = copies(with_rp=False, align=32)
out["col_only_aligned32_GBps"] = copies(with_val=False, with_rp=False, align=32)
out["col_only_src_shift1_GBps"] = copies(with_val=False, with_rp=False, src_shift=1)
hv = val.view(torch.uint8)[: 1 << 30]; src = torch.empty(1 << 30, dtype=torch.uint8, device=dev)
e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
with torch.cuda.stream(cs):
    e0.record(cs); hv.copy_(src, non_blocking=True); e1.record(cs)
cs.synchronize()
out["single_1GiB_GBps"] = (1 << 30) / e0.elapsed_time(e1) / 1e6
print(json.dumps({k: round(v, 2) for k, v in out.items()}))
