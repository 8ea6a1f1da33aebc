"""B200-native out-of-core chunked SpGEMM C = A x B on CSR (Xia et al., IPDPS'21 hot path).

The product path is the sm_100a library libspgemm_b200.so behind the C ABI in
include/spgemm.h; `capi` is its ctypes binding (same names), `matmul` a convenience wrapper
and `dist` the multi-GPU row-panel deal.  There is no CPU fallback: importing this package
without the built library raises ImportError.
"""
from __future__ import annotations

from . import capi
from .capi import (Plan, SpgemmError, opts, release_cache, spgemm_multiply, spgemm_plan)

__all__ = ["capi", "Plan", "SpgemmError", "opts", "spgemm_plan", "spgemm_multiply", "matmul", "release_cache"]


class HostCSR:
    """Host CSR result: row_ptr int64, col int32, val fp64 (torch pinned tensors or numpy)."""

    def __init__(self, nrows, ncols, row_ptr, col, val):
        self.nrows, self.ncols, self.row_ptr, self.col, self.val = nrows, ncols, row_ptr, col, val

    @property
    def nnz(self):
        return int(self.col.shape[0])


def matmul(A, B, budget: int = 0, *, ring: int = 2, validate: bool = False, chunk_nnz: int = 0,
           device: int = -1, stream=None, pinned: bool = True) -> HostCSR:
    """C = A x B through spgemm_plan + spgemm_execute_into; C lands in (pinned) host memory.

    A, B: objects with nrows, ncols, row_ptr (int64), col (int32), val (fp64) as numpy arrays
    (host inputs, H2D-copied into the arena) or CUDA tensors (device inputs, used in place).
    """
    import torch
    o = opts(device=device, validate=validate, ring=ring, chunk_nnz=chunk_nnz, stream=stream)
    with Plan(A, B, budget, o) as P:
        info = P.info()
        n, z = info["nrows"], info["nnz"]
        rp = torch.empty(n + 1, dtype=torch.int64, pin_memory=pinned)
        col = torch.empty(z, dtype=torch.int32, pin_memory=pinned)
        val = torch.empty(z, dtype=torch.float64, pin_memory=pinned)
        P.execute_into(rp, col, val)
    return HostCSR(n, info["ncols"], rp, col, val)
