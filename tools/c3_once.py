"""Run the C3 step (R-MAT s22, C = A*A, fused plan, chunks through a dropping sink) REPS times,
device operands as in bench.py's `value` -- for ncu captures of one unit's kernels; prints the
step times only.  SCALE overrides the R-MAT scale."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import workloads as W  # noqa: E402
from paper_conf_ipps_xia0ar21_b200 import capi  # noqa: E402

scale = int(os.environ.get("SCALE", "22"))
reps = int(os.environ.get("REPS", "1"))
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
s = torch.cuda.current_stream()
for r in range(reps):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    P = capi.Plan(d, d, ws.numel(), capi.opts(workspace=ws, fused=True, ring=3, chunk_nnz=200_000_000, stream=s.cuda_stream))
    P.execute_stream(lambda *a: 0)
    P.free()
    torch.cuda.synchronize()
    print(f"rep {r}: {1e3 * (time.perf_counter() - t0):.1f} ms", flush=True)
