"""Multi-GPU host logic on CPU with gloo, world size 2 (`-m "not gpu"`).

The row-panel deal, the per-rank global row_ptr base (all_gather of nnz), the broadcast of B and
the stitching of per-rank slices must reproduce the single-process result.  Each rank's slice is
computed by the oracle here (the per-rank GPU computation is covered by the GPU parity tests'
row-panel case, tests/test_gpu_parity.py::test_device_inputs_with_base_and_row_panels).
"""
import os
import socket

import numpy as np
import pytest

import oracle
import workloads as W
from paper_conf_ipps_xia0ar21_b200 import dist as pdist


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_row_panels_cover_and_balance():
    A = W.rmat(11, 8, seed=3)
    for world in (1, 2, 3, 4, 8):
        p = pdist.row_panels(A.row_ptr, world)
        assert p[0][0] == 0 and p[-1][1] == A.nrows and len(p) == world
        assert all(p[i][1] == p[i + 1][0] for i in range(world - 1))
        loads = [A.row_ptr[b] - A.row_ptr[a] for a, b in p]
        assert max(loads) <= A.nnz / world + np.diff(A.row_ptr).max() + 1
    # weights (e.g. products per row) and degenerate inputs
    u = oracle.products(A, A)
    p = pdist.row_panels(A.row_ptr, 4, weights=u)
    assert p[-1][1] == A.nrows
    assert pdist.row_panels(np.zeros(1, np.int64), 3) == [(0, 0), (0, 0), (0, 0)]
    e = pdist.row_panels(np.zeros(6, np.int64), 2)
    assert e[0][0] == 0 and e[-1][1] == 5


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = W.rmat(10, 8, seed=5)
        # B staged on rank 0 only; others receive it by broadcast into preallocated tensors
        if rank == 0:
            rp, col, val = torch.from_numpy(A.row_ptr.copy()), torch.from_numpy(A.col.copy()), torch.from_numpy(A.val.copy())
        else:
            rp = torch.zeros(A.nrows + 1, dtype=torch.int64)
            col = torch.zeros(A.nnz, dtype=torch.int32)
            val = torch.zeros(A.nnz, dtype=torch.float64)
        pdist.broadcast_csr([rp, col, val], src=0)
        B = W.CSR(A.nrows, A.ncols, rp.numpy(), col.numpy(), val.numpy())
        r0, r1 = pdist.row_panels(B.row_ptr, world)[rank]
        S = oracle.spgemm(B, B, rows=np.arange(r0, r1), threads=2)
        nnz = int(S["row_ptr"][-1])
        base, total = pdist.slice_bases(nnz)
        q.put((rank, r0, r1, S["row_ptr"] + base, S["col"], S["val"], total))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_slices_stitch_to_whole():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=120) for _ in range(2)], key=lambda t: t[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    A = W.rmat(10, 8, seed=5)
    whole = oracle.spgemm(A, A)
    rp, col, val = pdist.gather_rows_global([(r[3], r[4], r[5]) for r in res])
    assert res[0][2] == res[1][1] and res[1][2] == A.nrows
    assert res[0][6] == res[1][6] == whole["row_ptr"][-1]
    assert np.array_equal(rp, whole["row_ptr"]) and np.array_equal(col, whole["col"])
    assert np.array_equal(val, whole["val"])


def _worker_allgather(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = W.rmat(9, 8, seed=6)
        host = [torch.from_numpy(A.row_ptr), torch.from_numpy(A.col), torch.from_numpy(A.val)]
        dev = [torch.full((pdist.padded_len(h.numel(), world),), -7, dtype=h.dtype) for h in host]
        pdist.scatter_allgather_csr(host, dev)
        ok = all(torch.equal(d[:h.numel()], h) for h, d in zip(host, dev))
        q.put((rank, ok))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_scatter_allgather_b(world):
    """B reaches every rank with each rank uploading 1/world of every array, then an all-gather
    (the multi-GPU e2e upload; uneven lengths are padded to a multiple of the world size)."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_allgather, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(ok for _, ok in res), res


def _worker_flops(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = W.rmat(11, 8, seed=9)
        s0, s1 = pdist.even_slices(A.nrows, world)[rank]
        # each rank counts only its even slice (bench.py: spgemm_row_products on its GPU)
        u_loc = oracle.products(A, A, rows=np.arange(s0, s1))
        u_all = pdist.allgather_rows(u_loc, A.nrows)
        panels = pdist.row_panels(A.row_ptr, world, weights=u_all)
        q.put((rank, u_all, panels))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_flop_balanced_panels(world):
    """every rank counts the products of 1/world of the rows, one all_gather gives
    everybody the whole per-row count, and all ranks cut the SAME row panels, balanced by products
    (within one row's products of the ideal share) -- bench.py's multi-GPU deal."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_flops, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=120) for _ in range(world)], key=lambda t: t[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    A = W.rmat(11, 8, seed=9)
    u = oracle.products(A, A)
    for _, u_all, panels in res:
        assert np.array_equal(u_all, u)
        assert panels == res[0][2]
    panels = res[0][2]
    assert panels[0][0] == 0 and panels[-1][1] == A.nrows
    loads = [int(u[a:b].sum()) for a, b in panels]
    assert max(loads) - u.sum() / world <= u.max() + 1
