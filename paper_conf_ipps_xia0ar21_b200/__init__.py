"""B200-native out-of-core chunked SpGEMM C = A x B on CSR (Xia et al., IPDPS'21 hot path).

The product path is the sm_100a library libspgemm_b200.so behind the C ABI in
include/spgemm.h; `capi` is its ctypes binding (same names), `matmul` a convenience wrapper
and `dist` the multi-GPU row-panel deal.  There is no CPU fallback: importing this package
without the built library raises ImportError.
"""
from __future__ import annotations

from . import capi
from .capi import (Plan, SpgemmError, opts, release_cache, spgemm_multiply, spgemm_plan)

__all__ = ["capi", "Plan", "SpgemmError", "opts", "spgemm_plan", "spgemm_multiply", "matmul", "as_csr", "release_cache"]


class HostCSR:
    """Host CSR result: row_ptr int64, col int32, val fp64 (torch pinned tensors or numpy)."""

    def __init__(self, nrows, ncols, row_ptr, col, val):
        self.nrows, self.ncols, self.row_ptr, self.col, self.val = nrows, ncols, row_ptr, col, val

    @property
    def nnz(self):
        return int(self.col.shape[0])


class _CSRView:
    def __init__(self, nrows, ncols, row_ptr, col, val):
        self.nrows, self.ncols, self.row_ptr, self.col, self.val = nrows, ncols, row_ptr, col, val


def as_csr(M):
    """A CSR operand for the C ABI: objects with nrows/ncols/row_ptr/col/val (numpy or CUDA tensors)
    pass through; a scipy.sparse matrix is converted (int64 row_ptr, int32 sorted columns, fp64)."""
    if hasattr(M, "row_ptr"):
        return M
    import numpy as np
    if hasattr(M, "tocsr"):  # scipy.sparse
        C = M.tocsr()
        if not C.has_sorted_indices:
            C = C.sorted_indices()
        return _CSRView(C.shape[0], C.shape[1], np.ascontiguousarray(C.indptr, dtype=np.int64),
                        np.ascontiguousarray(C.indices, dtype=np.int32), np.ascontiguousarray(C.data, dtype=np.float64))
    raise TypeError("A/B must be a CSR object (nrows, ncols, row_ptr, col, val) or a scipy.sparse matrix")


def matmul(A, B, budget: int = 0, *, ring: int = 2, validate: bool = False, chunk_nnz: int = 0,
           device: int = -1, stream=None, pinned: bool = True, col_panels: int = 0, order: int = 0) -> HostCSR:
    """C = A x B through spgemm_plan + spgemm_execute_into; C lands in (pinned) host memory.

    A, B: objects with nrows, ncols, row_ptr (int64), col (int32), val (fp64) as numpy arrays
    (host inputs, H2D-copied into the arena) or CUDA tensors (device inputs, used in place), or
    scipy.sparse matrices.  budget: device bytes (0 = 90 % of free memory); a B larger than the
    budget is cut into column panels automatically (col_panels: 0 auto, 1 never, >= 2 forced).
    order = 1: the paper's decreasing-flops chunk schedule.
    """
    import torch
    A, B = as_csr(A), as_csr(B)
    o = opts(device=device, validate=validate, ring=ring, chunk_nnz=chunk_nnz, stream=stream,
             col_panels=col_panels, order=order)
    with Plan(A, B, budget, o) as P:
        info = P.info()
        n, z = info["nrows"], info["nnz"]
        rp = torch.empty(n + 1, dtype=torch.int64, pin_memory=pinned)
        col = torch.empty(z, dtype=torch.int32, pin_memory=pinned)
        val = torch.empty(z, dtype=torch.float64, pin_memory=pinned)
        P.execute_into(rp, col, val)
    return HostCSR(n, info["ncols"], rp, col, val)
