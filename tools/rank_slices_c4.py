"""All N rank slices of a multi-GPU configuration, emulated one after the other on ONE GPU
(VERDICT r1 item 6): the flop-balanced row panels bench.py deals (per-row products from the
library's count kernel, dist.row_panels with those weights), and for every panel the time of
plan + execute_stream (sink, fused plan, ring 3) with device operands -- what that rank would
spend on its own GPU and host link.  Prints one JSON line: per-rank ms, products, nnz, the
spread of the times, and each slice's D2H link bound from a live probe.

  CONFIG=3 N=8 python tools/rank_slices_c4.py     # configs[3] = R-MAT s24 over 8 ranks
  CONFIG=4 N=8 python tools/rank_slices_c4.py     # configs[4] = rectangular power-law
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_ipps_xia0ar21_b200 import capi  # noqa: E402
from paper_conf_ipps_xia0ar21_b200 import dist as pdist  # noqa: E402

cfg = int(os.environ.get("CONFIG", "3"))
N = int(os.environ.get("N", "8"))
chunk = int(os.environ.get("CHUNK", "200000000"))
t0 = time.perf_counter()
if cfg == 3:
    A = B = W.rmat_torch(int(os.environ.get("SCALE", "24")), 16, seed=20210518)
else:
    A = W.rmat_torch(24, col_scale=22, nedges=1 << 28, seed=11, symmetric=False)
    B = W.rmat_torch(22, col_scale=24, nedges=1 << 28, seed=12, symmetric=False)
gen_s = time.perf_counter() - t0
dev = torch.device("cuda", 0)


class D:
    pass


def to_dev(M):
    d = D()
    d.nrows, d.ncols = M.nrows, M.ncols
    d.row_ptr = torch.from_numpy(M.row_ptr).to(dev)
    d.col = torch.from_numpy(M.col).to(dev)
    d.val = torch.from_numpy(M.val).to(dev)
    return d


dA = to_dev(A)
dB = dA if B is A else to_dev(B)
u, tot = capi.row_products(dA, dB)
panels = pdist.row_panels(A.row_ptr, N, weights=u)
ws = torch.empty(int(torch.cuda.mem_get_info()[0] * 0.85), dtype=torch.uint8, device=dev)
s = torch.cuda.current_stream()

# link probe: one chunk-sized D2H into pinned memory
nb = 12 * chunk
h = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
src = torch.empty(nb, dtype=torch.uint8, device=dev)
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
link = 0.0
for _ in range(2):
    e0.record(s)
    h.copy_(src, non_blocking=True)
    e1.record(s)
    torch.cuda.synchronize()
    link = max(link, nb / (e0.elapsed_time(e1) / 1e3) / 1e9)
del h, src

out = {"config": cfg, "N": N, "gen_s": gen_s, "products": int(tot), "link_GBps": link, "ranks": []}
for r, (r0, r1) in enumerate(panels):
    got = {"nnz": 0}

    def sink(a, b, rp, col, val):
        got["nnz"] += int(rp[-1])

    best = None
    for rep in range(int(os.environ.get("REPS", "2"))):
        got["nnz"] = 0
        torch.cuda.synchronize()
        e0.record(s)
        P = capi.Plan(dA, dB, ws.numel(), capi.opts(workspace=ws, stream=s.cuda_stream, fused=True, ring=3,
                                                    chunk_nnz=chunk, row_begin=r0, row_end=r1))
        P.execute_stream(sink)
        e1.record(s)
        info = P.info()
        P.free()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        best = ms if best is None else min(best, ms)
    d2h = 12 * got["nnz"] + 8 * (r1 - r0 + info["num_copies"])
    out["ranks"].append({"rank": r, "rows": [r0, r1], "products": int(u[r0:r1].sum()), "nnz": got["nnz"],
                         "ms": round(best, 2), "link_bound_ms": round(d2h / link / 1e6, 2),
                         "frac_of_link_bound": round(d2h / link / 1e6 / best, 4)})
ms = [x["ms"] for x in out["ranks"]]
out["ms_max"], out["ms_min"], out["spread"] = max(ms), min(ms), (max(ms) - min(ms)) / max(ms)
out["gflops_if_parallel"] = 2 * out["products"] / (max(ms) / 1e3) / 1e9
print(json.dumps(out), flush=True)
