"""Multi-GPU row-panel deal (one process per GPU, torch.distributed over NCCL / NVLink).

Rows of C are independent (§III-A: "final values within a chunk of the output
matrix C are independent"), so A is dealt across ranks as contiguous row panels (§III-A,
§III-D) and every rank needs all of B.  The only exchanges on the path are
  * B (and A when A is B) reaching every GPU from host memory: every rank uploads 1/world of each
    CSR array over its OWN host link and an all-gather over NVLink/NVSwitch assembles the whole
    on every GPU (`scatter_allgather_csr`; H2D time / world instead of one rank uploading all of
    it and broadcasting, `broadcast_csr`; NCCL on a B200 box, gloo in the CPU tests);
  * the 8-byte nnz of every rank's slice (`slice_bases`, an all_gather) so that each rank writes
    its C rows with GLOBAL row_ptr values into its part of one logical host CSR.
After that every rank drains its own C chunks over its own host link; nothing else crosses GPUs.
"""
from __future__ import annotations

from typing import List, Sequence, Tuple

import numpy as np


def row_panels(row_ptr: np.ndarray, world: int, weights: np.ndarray | None = None) -> List[Tuple[int, int]]:
    """Contiguous row ranges [r0, r1) per rank, balanced by `weights` per row (default: nnz of A's
    rows, which is what row_ptr gives for free).  Every rank gets a range (possibly empty)."""
    n = len(row_ptr) - 1
    if weights is None:
        cum = np.asarray(row_ptr, dtype=np.int64) - int(row_ptr[0])
    else:
        cum = np.zeros(n + 1, dtype=np.int64)
        np.cumsum(np.asarray(weights, dtype=np.int64), out=cum[1:])
    total = int(cum[-1])
    cuts = [0]
    for r in range(1, world):
        target = (total * r + world - 1) // world if total else 0
        c = int(np.searchsorted(cum, target, side="left")) if total else (n * r) // world
        cuts.append(min(max(c, cuts[-1]), n))
    cuts.append(n)
    return [(cuts[r], cuts[r + 1]) for r in range(world)]


def even_slices(n: int, world: int) -> List[Tuple[int, int]]:
    """n rows split into world near-equal contiguous ranges (who counts which rows' products)."""
    return [((n * r) // world, (n * (r + 1)) // world) for r in range(world)]


def allgather_rows(local, n: int, group=None, device=None) -> np.ndarray:
    """Every rank holds `local` = an int64 value per row of its even_slices(n, world) range (e.g.
    the products per row from the library's count kernel, spgemm_row_products); returns the whole
    length-n array on every rank (one all_gather, NCCL over NVLink on GPUs).  Used to deal
    flop-balanced row panels (all_gather(products), then identical cuts)."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    sl = even_slices(n, world)
    m = max(b - a for a, b in sl) if world else 0
    t = torch.zeros(max(m, 1), dtype=torch.int64, device=device)
    loc = torch.as_tensor(np.asarray(local, dtype=np.int64))
    t[:len(loc)].copy_(loc.to(t.device))
    out = [torch.zeros_like(t) for _ in range(world)]
    dist.all_gather(out, t, group=group)
    return np.concatenate([out[r][:b - a].cpu().numpy() for r, (a, b) in enumerate(sl)])


def slice_bases(local_nnz: int, group=None, device=None) -> Tuple[int, int]:
    """All-gather every rank's nnz; returns (global row_ptr base of this rank, total nnz)."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    t = torch.tensor([int(local_nnz)], dtype=torch.int64, device=device)
    out = [torch.zeros(1, dtype=torch.int64, device=device) for _ in range(world)]
    dist.all_gather(out, t, group=group)
    vals = [int(x.item()) for x in out]
    return sum(vals[:rank]), sum(vals)


def broadcast_csr(arrays: Sequence, src: int = 0, group=None) -> None:
    """In-place broadcast of the CSR arrays (row_ptr, col, val tensors, already allocated with the
    right shapes on every rank) from `src` -- NCCL over NVLink on GPUs."""
    import torch.distributed as dist
    for a in arrays:
        dist.broadcast(a, src=src, group=group)


def padded_len(n: int, world: int) -> int:
    """Length of a device array that `scatter_allgather_csr` can fill: n rounded up to a multiple
    of the world size (the all-gather moves equal chunks)."""
    return ((int(n) + world - 1) // world) * world


def scatter_allgather_csr(host_arrays: Sequence, dev_arrays: Sequence, group=None) -> None:
    """Every rank copies its 1/world chunk of each host array (pinned, true length n) into the same
    place of the matching device array (length padded_len(n, world)) over its own host link, then
    an in-place all-gather (NCCL over NVLink on GPUs) gives every rank the whole array in
    dev_array[:n]."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    for h, d in zip(host_arrays, dev_arrays):
        n = int(h.numel())
        chunk = int(d.numel()) // world
        assert chunk * world == int(d.numel()) and chunk * world >= n
        lo, hi = min(rank * chunk, n), min((rank + 1) * chunk, n)
        mine = d[rank * chunk:(rank + 1) * chunk]
        if hi > lo:
            mine[:hi - lo].copy_(h[lo:hi], non_blocking=True)
        dist.all_gather_into_tensor(d, mine, group=group)


def gather_rows_global(parts: Sequence[Tuple[np.ndarray, np.ndarray, np.ndarray]]):
    """Stitch per-rank slices (row_ptr with global values, col, val) into one CSR (tests)."""
    rp = [parts[0][0][:1]]
    for p in parts:
        rp.append(p[0][1:])
    return (np.concatenate(rp), np.concatenate([p[1] for p in parts]), np.concatenate([p[2] for p in parts]))
