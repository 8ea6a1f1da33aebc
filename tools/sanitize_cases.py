"""Small multiplies through every path for compute-sanitizer (memcheck / racecheck / synccheck):
in-core two-phase and fused plans (host cut included), forced chunking, long-row tiers (medium, CTA whole / pieced,
dense), column panels.  Run under every compute-sanitizer tool (memcheck, racecheck, synccheck, initcheck)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle
import workloads as W
from paper_conf_ipps_xia0ar21_b200 import capi


def run(A, B, **kw):
    with capi.Plan(A, B, 0, capi.opts(**kw)) as P:
        info = P.info()
        n = info["nnz"] if info["nnz"] >= 0 else int(oracle.spgemm(A, B)["row_ptr"][-1])
        rp = torch.empty(info["nrows"] + 1, dtype=torch.int64, pin_memory=True)
        col = torch.empty(max(n, 1), dtype=torch.int32, pin_memory=True)
        val = torch.empty(max(n, 1), dtype=torch.float64, pin_memory=True)
        P.execute_capacity(rp, col, val, n)
    res = oracle.compare(rp.numpy(), col.numpy()[:n], val.numpy()[:n], oracle.spgemm(A, B))
    assert res["ok"], (kw, res)


S = W.stencil_3d27(10)
R = W.rmat(10, 8, seed=3)
rng = np.random.default_rng(5)
brows = [np.sort(rng.choice(200_000, 1500, replace=False)) for _ in range(40)] + \
        [np.sort(rng.choice(200_000, 3, replace=False)) for _ in range(100)]
rp = np.zeros(len(brows) + 1, np.int64); np.cumsum([len(b) for b in brows], out=rp[1:])
LB = W.CSR(len(brows), 200_000, rp, np.concatenate(brows).astype(np.int32), rng.uniform(-1, 1, rp[-1]))
LA = W.CSR(2, len(brows), np.array([0, 40, 45], np.int64), np.concatenate([np.arange(40), np.arange(40, 45)]).astype(np.int32),
           rng.uniform(-1, 1, 45))
for kw in ({}, {"fused": True}, {"chunk_nnz": 3000, "ring": 3}, {"fused": True, "chunk_nnz": 3000}, {"col_panels": 3}):
    run(S, S, **kw)
    run(R, R, **kw)
    run(LA, LB, **kw)
# host cut (fused C = A*A from host arrays) with many small interleaved operand pieces
os.environ["SPGEMM_PIECE_NNZ"] = "500"
for kw in ({"fused": True}, {"fused": True, "chunk_nnz": 3000, "ring": 1}):
    run(S, S, **kw)
    run(R, R, **kw)
del os.environ["SPGEMM_PIECE_NNZ"]
# power-law rows through the medium, CTA (whole and pieced) and dense tiers: R-MAT s12 with a small
# dense-slot count and pieces forced by a wide column span
R2 = W.rmat(12, 16, seed=7)
run(R2, R2, fused=True)
run(R2, R2, chunk_nnz=200_000, ring=2)
print("sanitize cases ok")
