"""The multi-GPU plumbing on a real B200 (`-m gpu`): the NCCL call sites of dist.py execute on
hardware (a world-size-1 NCCL process group -- gpurun gives one GPU), and bench.py's multi-rank
path runs end to end with two ranks on one GPU over gloo (control flow of the deal, the product
all-gather, the per-rank sink and the max-over-ranks timing; NCCL refuses two ranks on one
device).  Row panels of C are independent (§III-A), so every rank's slice is checked
against the oracle rows it owns.
"""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_ipps_xia0ar21_b200 import capi  # noqa: E402
from paper_conf_ipps_xia0ar21_b200 import dist as pdist  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_nccl_world1_collectives_and_panel_multiply():
    """NCCL process group (world 1) on cuda:0: scatter_allgather_csr fills device B from pinned host
    memory, allgather_rows gathers the library's per-row product counts, slice_bases gives the
    global base; the plan on the gathered device operands matches the oracle."""
    import torch.distributed as dist
    dev = torch.device("cuda", 0)
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{_port()}", rank=0, world_size=1, device_id=dev)
    try:
        A = W.rmat(12, 8, seed=4)
        host = [torch.from_numpy(A.row_ptr).pin_memory(), torch.from_numpy(A.col).pin_memory(),
                torch.from_numpy(A.val).pin_memory()]
        store = [torch.full((pdist.padded_len(h.numel(), 1),), -1, dtype=h.dtype, device=dev) for h in host]
        pdist.scatter_allgather_csr(host, store)
        torch.cuda.synchronize()
        assert all(torch.equal(s[:h.numel()].cpu(), h) for h, s in zip(host, store))

        class D:
            pass
        d = D()
        d.nrows, d.ncols = A.nrows, A.ncols
        d.row_ptr, d.col, d.val = (s[:h.numel()] for s, h in zip(store, host))
        u_loc, tot = capi.row_products(d, d)
        u_all = pdist.allgather_rows(u_loc, A.nrows, device=dev)
        u = oracle.products(A, A)
        assert np.array_equal(u_all, u) and tot == int(u.sum())
        (r0, r1), = pdist.row_panels(A.row_ptr, 1, weights=u_all)
        base, total = pdist.slice_bases(12345, device=dev)
        assert (r0, r1) == (0, A.nrows) and base == 0 and total == 12345
        E = oracle.spgemm(A, A)
        z = len(E["col"])
        rp = torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True)
        col = torch.empty(z, dtype=torch.int32, pin_memory=True)
        val = torch.empty(z, dtype=torch.float64, pin_memory=True)
        with capi.Plan(d, d, 0, capi.opts(fused=True)) as P:
            assert P.execute_capacity(rp, col, val, z) == z
        assert oracle.compare(rp.numpy(), col.numpy(), val.numpy(), E)["ok"]
    finally:
        dist.destroy_process_group()


def test_bench_two_ranks_gloo_one_gpu():
    """bench.py under torchrun with 2 ranks (gloo, both on cuda:0): flop-balanced panels from the
    all-gathered product counts, each rank's sink, max-over-ranks timing, one JSON line."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", "2",
           "--dist-backend", "gloo", "--config", "2", "--scale", "14", "--steps", "2", "--warmup", "1",
           "--e2e-steps", "1", "--no-cpu"]
    out = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["parity"]["ok"] and d["e2e"]["value"] > 0
    assert d["config"]["parallelism"].startswith("row panels x2")
