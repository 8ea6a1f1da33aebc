"""Column-panel mode at full size (diagnostic + evidence): C2 (27-pt 128^3, C = A*A) with host
operands and a device budget smaller than B, so the plan cuts B into column panels
(Alg. 3 line 4, §III-D).  Prints one JSON line: panels, plan/execute ms, GFLOP/s, output rate,
and a sampled parity check against the closed form + the oracle."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle
import workloads as W
from tests import closed_forms as CF
from paper_conf_ipps_xia0ar21_b200 import capi

n = int(os.environ.get("N", "128"))
budget = int(float(os.environ.get("BUDGET_MB", "512")) * (1 << 20))
A = W.stencil_3d27(n)
hA = W.CSR(A.nrows, A.ncols, torch.from_numpy(A.row_ptr).pin_memory(), torch.from_numpy(A.col).pin_memory(),
           torch.from_numpy(A.val).pin_memory())
p_tot, z_tot = CF.c2_totals(n)
rp = torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True)
col = torch.empty(z_tot, dtype=torch.int32, pin_memory=True)
val = torch.empty(z_tot, dtype=torch.float64, pin_memory=True)
ws = torch.empty(budget, dtype=torch.uint8, device="cuda")
res = []
for rep in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    P = capi.Plan(hA, hA, budget, capi.opts(workspace=ws))
    t1 = time.perf_counter()
    P.execute_into(rp, col, val)
    t2 = time.perf_counter()
    info = P.info()
    P.free()
    res.append((t1 - t0, t2 - t1))
plan_s, exec_s = min(r[0] for r in res), min(r[1] for r in res)
tot = min(r[0] + r[1] for r in res)
rng = np.random.default_rng(3)
rows = np.unique(np.concatenate([[0, A.nrows - 1], rng.integers(0, A.nrows, 200)]))
E = oracle.spgemm(A, A, rows=rows)
hrp, hcol, hval = rp.numpy(), col.numpy(), val.numpy()
gp = np.concatenate([[0], np.cumsum(hrp[rows + 1] - hrp[rows])])
idx = np.concatenate([np.arange(hrp[r], hrp[r + 1]) for r in rows])
cmp = oracle.compare(gp, hcol[idx], hval[idx], E)
exact = bool(np.array_equal(hval[idx], E["val"]))
out = {"workload": f"C2 27-pt {n}^3, host operands, budget {budget >> 20} MiB (B = {(8 * (A.nrows + 1) + 12 * A.nnz) / 1e6:.0f} MB)",
       "col_panels": info["col_panels"], "chunks": info["num_chunks"], "nnz": info["nnz"], "nnz_ok": info["nnz"] == z_tot,
       "products_ok": info["products"] == p_tot, "plan_ms": 1e3 * plan_s, "execute_ms": 1e3 * exec_s,
       "total_ms": 1e3 * tot, "GFLOPs": 2 * p_tot / tot / 1e9, "C_GBps": (12 * z_tot + 8 * (A.nrows + 1)) / tot / 1e9,
       "arena_used": info["arena_used"], "sampled_rows": int(len(rows)), "parity_ok": bool(cmp["ok"]), "bit_exact": exact,
       "row_ptr_ok": bool(np.array_equal(np.diff(hrp), CF.c2_row_nnz(n, np.arange(A.nrows)))),
       "sum_ok": bool(float(hval.sum()) == CF.c2_sum(n))}
print(json.dumps(out))
