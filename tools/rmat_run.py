"""Time C = A*A on an R-MAT graph through the sink (C larger than host RAM); prints a JSON line.

SCALE (default 22) picks configs[2] (s22) / configs[3]-like (s24) sizes; ROWS_FRAC (default 1)
takes the first fraction of rows (one rank's panel of a multi-GPU run).
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import workloads as W
from paper_conf_ipps_xia0ar21_b200 import capi

scale = int(os.environ.get("SCALE", "22"))
frac = float(os.environ.get("ROWS_FRAC", "1"))
t0 = time.perf_counter()
if os.environ.get("GEN", "numpy") == "torch":
    A = W.rmat_torch(scale, 16)
else:
    A = W.rmat(scale, 16)
gen_s = time.perf_counter() - t0
dev = torch.device("cuda", 0)


class D:
    pass


d = D()
d.nrows, d.ncols = A.nrows, A.ncols
d.row_ptr = torch.from_numpy(A.row_ptr).to(dev)
d.col = torch.from_numpy(A.col).to(dev)
d.val = torch.from_numpy(A.val).to(dev)
r1 = int(A.nrows * frac)
# one arena for every repetition (cudaMalloc/cudaFree of ~150 GB per plan is not part of a multiply)
ws = torch.empty(int(torch.cuda.mem_get_info()[0] * 0.85), dtype=torch.uint8, device=dev)
res = {"scale": scale, "nnz_A": int(A.nnz), "rows": r1, "gen_s": gen_s}
for rep in range(int(os.environ.get("REPS", "2"))):
    got = {"nnz": 0, "chunks": 0}

    rownnz = np.zeros(r1, dtype=np.int64) if os.environ.get("TIERS") else None

    def sink(r0_, r1_, rp, col, val):
        got["nnz"] += int(rp[-1])
        got["chunks"] += 1
        if rownnz is not None:
            rownnz[r0_:r1_] = np.diff(rp)

    torch.cuda.synchronize()
    t0 = time.perf_counter()
    P = capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, fused=True, ring=3, chunk_nnz=int(os.environ.get("CHUNK", "200000000")),
                                     row_end=r1, profile=True))
    tp = time.perf_counter() - t0
    P.execute_stream(sink)
    torch.cuda.synchronize()
    t = time.perf_counter() - t0
    info = P.info()
    st = P.stats()
    P.free()
    res.update({"rep": rep, "seconds": t, "plan_s": tp, "products": info["products"], "nnz_C": info["nnz"],
                "chunks": info["num_chunks"], "gflops": 2 * info["products"] / t / 1e9,
                "d2h_GBps": 12 * info["nnz"] / t / 1e9, "rows_warp": info["rows_warp"],
                "rows_block": info["rows_block"], "rows_global": info["rows_global"],
                "max_row_nnz": info["max_row_nnz"], "max_row_products": info["max_row_products"],
                "stats_ms": {k: round(v["ms"], 2) for k, v in st.items()}})
if rownnz is not None:
    # products and nnz per accumulator tier (numeric thresholds of internal.h: W <= 384, B <= 12288,
    # H <= 393216, G beyond)
    deg = np.diff(A.row_ptr)
    prod = np.add.reduceat(deg[A.col].astype(np.int64), A.row_ptr[:-1].clip(max=max(A.nnz - 1, 0)))
    prod[deg == 0] = 0
    prod = prod[:r1]
    tiers = {}
    for name, lo, hi in (("W", 1, 384), ("B", 385, 12288), ("H", 12289, 393216), ("G", 393217, 1 << 62)):
        m = (rownnz >= lo) & (rownnz <= hi)
        tiers[name] = {"rows": int(m.sum()), "products": int(prod[m].sum()), "nnz": int(rownnz[m].sum()),
                       "max_products": int(prod[m].max()) if m.any() else 0}
    res["tiers"] = tiers
print(json.dumps(res), flush=True)
