"""Per-tier kernel times of C = A*A on an R-MAT graph WITHOUT cross-stream contention: a two-phase
plan runs the symbolic pass of all rows alone on one stream (plan stats), and the execution runs
only the numeric passes (plus copies on the copy engine).  A/B tool for kernel changes (the fused
bench overlaps symbolic, numeric and copies, so its per-kernel event times include contention).

  SCALE=22 python tools/tier_times.py            # configs[2]
  SPGEMM_NO_MEDIUM=1 SCALE=20 python tools/tier_times.py
Prints one JSON line.
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_ipps_xia0ar21_b200 import capi  # noqa: E402

scale = int(os.environ.get("SCALE", "22"))
reps = int(os.environ.get("REPS", "2"))
A = W.rmat_torch(scale, 16, seed=20210517)
dev = torch.device("cuda", 0)


class D:
    pass


d = D()
d.nrows, d.ncols = A.nrows, A.ncols
d.row_ptr = torch.from_numpy(A.row_ptr).to(dev)
d.col = torch.from_numpy(A.col).to(dev)
d.val = torch.from_numpy(A.val).to(dev)
ws = torch.empty(int(torch.cuda.mem_get_info()[0] * 0.85), dtype=torch.uint8, device=dev)
out = {"scale": scale, "nnz_A": A.nnz, "medium": os.environ.get("SPGEMM_NO_MEDIUM", "0") != "1"}
for rep in range(reps):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    P = capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, ring=3, chunk_nnz=200_000_000, profile=True))
    t1 = time.perf_counter()
    plan_stats = P.stats()
    P.execute_stream(lambda *a: 0)
    t2 = time.perf_counter()
    st = P.stats()
    info = P.info()
    P.free()
    keep = ("count", "sym_w", "sym_m", "sym_b", "sym_g", "scan", "num_w", "num_m", "num_b", "num_g")
    out[f"rep{rep}"] = {"plan_s": t1 - t0, "execute_s": t2 - t1,
                        "ms": {k: round(v["ms"], 2) for k, v in {**plan_stats, **st}.items() if k in keep},
                        "rows": {k: info[k] for k in ("rows_warp", "rows_medium", "rows_block", "rows_global")},
                        "products": info["products"], "nnz": info["nnz"]}
print(json.dumps(out), flush=True)
