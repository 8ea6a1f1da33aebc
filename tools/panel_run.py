"""Time a row panel of configs[2..4] through the sink (C larger than host RAM); prints JSON lines.

CONFIG=2: R-MAT s22 ef16 (C3), 3: R-MAT s24 ef16 (C4), 4: rectangular 2^24x2^22 * 2^22x2^24 (C5).
ROWS_FRAC: the fraction of rows timed (0.125 = the panel one rank owns in an 8-GPU deal).
Inputs are generated on the GPU (workloads.rmat_torch) and resident in HBM before timing.
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import workloads as W
from paper_conf_ipps_xia0ar21_b200 import capi

cfg = int(os.environ.get("CONFIG", "3"))
frac = float(os.environ.get("ROWS_FRAC", "0.125"))
t0 = time.perf_counter()
if cfg == 2:
    A = W.rmat_torch(22, 16)
    B = A
elif cfg == 3:
    A = W.rmat_torch(24, 16, seed=20210518)
    B = A
else:
    A = W.rmat_torch(24, col_scale=22, nedges=1 << 28, seed=11, symmetric=False)
    B = W.rmat_torch(22, col_scale=24, nedges=1 << 28, seed=12, symmetric=False)
gen_s = time.perf_counter() - t0
dev = torch.device("cuda", 0)


class D:
    pass


def dcsr(M):
    d = D()
    d.nrows, d.ncols = M.nrows, M.ncols
    d.row_ptr = torch.from_numpy(M.row_ptr).to(dev)
    d.col = torch.from_numpy(M.col).to(dev)
    d.val = torch.from_numpy(M.val).to(dev)
    return d


dA = dcsr(A)
dB = dA if B is A else dcsr(B)
r1 = int(A.nrows * frac)
# one arena for every repetition (cudaMalloc/cudaFree of ~150 GB per plan is not part of a multiply)
ws = torch.empty(int(torch.cuda.mem_get_info()[0] * 0.85), dtype=torch.uint8, device=dev)
for rep in range(2):
    got = {"nnz": 0}

    def sink(r0_, r1_, rp, col, val):
        got["nnz"] += int(rp[-1])

    torch.cuda.synchronize()
    t0 = time.perf_counter()
    P = capi.Plan(dA, dB, ws.numel(), capi.opts(workspace=ws, fused=True, ring=3, chunk_nnz=200_000_000, row_end=r1, profile=True))
    P.execute_stream(sink)
    torch.cuda.synchronize()
    t = time.perf_counter() - t0
    info = P.info()
    st = P.stats()
    P.free()
print(json.dumps({"config": cfg, "rows": r1, "of_rows": A.nrows, "nnz_A": int(A.nnz), "nnz_B": int(B.nnz),
                  "gen_s": gen_s, "seconds": t, "products": info["products"], "nnz_C": info["nnz"],
                  "C_host_bytes": 12 * info["nnz"] + 8 * (r1 + 1), "chunks": info["num_chunks"],
                  "gflops": 2 * info["products"] / t / 1e9, "d2h_GBps_effective": 12 * info["nnz"] / t / 1e9,
                  "rows_warp": info["rows_warp"], "rows_block": info["rows_block"],
                  "rows_arena_tiers": info["rows_global"], "max_row_nnz": info["max_row_nnz"],
                  "stats_ms_overlapping": {k: round(v["ms"], 1) for k, v in st.items()}}), flush=True)
