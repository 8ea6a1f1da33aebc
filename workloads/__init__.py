"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NONE of the method's arithmetic: it only builds input
matrices A and B in CSR form (int64 row_ptr, int32 col, fp64 val; see
DESIGN.md "Readings" #3).  Both sides of every parity test consume the same
arrays; neither the oracle (`oracle/`) nor the CUDA path
(`paper_conf_ipps_xia0ar21_b200/`) is imported here.

Workload shapes follow BASELINE.json `configs` and the paper's inputs
(§V-B, Table II: square SuiteSparse matrices,
C = A x A, fp64 data; graphs with com-LiveJournal-like skew, FEM/stencil
matrices such as stokes/nlpkkt200).  Recipes are stated in DESIGN.md §"Input
recipe".
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

__all__ = [
    "CSR", "stencil_2d5", "stencil_3d27", "rmat", "rmat_rect", "random_csr",
    "identity", "permutation", "fig2_instance", "config",
]


@dataclass
class CSR:
    """CSR matrix: row_ptr int64 [nrows+1], col int32 [nnz] (sorted, unique per row), val fp64 [nnz].

    The CSR layout is the paper's (§II-A: row_offsets,
    col_ids sorted per row, data).
    """
    nrows: int
    ncols: int
    row_ptr: np.ndarray
    col: np.ndarray
    val: np.ndarray

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1]) if self.nrows >= 0 and len(self.row_ptr) else 0

    def check(self) -> None:
        rp, c = self.row_ptr, self.col
        assert rp.dtype == np.int64 and c.dtype == np.int32 and self.val.dtype == np.float64
        assert len(rp) == self.nrows + 1 and rp[0] == 0 and np.all(np.diff(rp) >= 0)
        assert len(c) == rp[-1] == len(self.val)
        if len(c):
            assert c.min() >= 0 and c.max() < self.ncols
            d = np.diff(c.astype(np.int64))
            # strictly increasing inside a row: a non-positive step is only allowed at row starts
            starts = np.zeros(len(c), dtype=bool)
            starts[rp[:-1][rp[:-1] < len(c)]] = True
            assert np.all((d > 0) | starts[1:])

    def to_scipy(self):
        import scipy.sparse as sp
        return sp.csr_matrix((self.val, self.col, self.row_ptr), shape=(self.nrows, self.ncols))

    def dense(self) -> np.ndarray:
        out = np.zeros((self.nrows, self.ncols))
        for i in range(self.nrows):
            for p in range(self.row_ptr[i], self.row_ptr[i + 1]):
                out[i, self.col[p]] += self.val[p]
        return out


def _assemble(nrows, ncols, counts, cols_by_offset):
    """Build CSR from per-offset (valid_mask, col) arrays listed in increasing column order."""
    rp = np.zeros(nrows + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    col = np.empty(int(rp[-1]), dtype=np.int32)
    val = np.empty(int(rp[-1]), dtype=np.float64)
    cursor = rp[:-1].copy()
    for mask, cvals, v in cols_by_offset:
        rows = np.nonzero(mask)[0]
        pos = cursor[rows]
        col[pos] = cvals[rows]
        val[pos] = v
        cursor[rows] += 1
    return CSR(nrows, ncols, rp, col, val)


def stencil_2d5(n: int, diag: float = 4.0, off: float = -1.0) -> CSR:
    """2-D 5-point Laplacian on an n x n grid, row i = n*y + x (BASELINE config 0, n = 64)."""
    m = n * n
    idx = np.arange(m, dtype=np.int64)
    x, y = idx % n, idx // n
    offs = [(0, -1), (-1, 0), (0, 0), (1, 0), (0, 1)]  # increasing linear delta: -n, -1, 0, 1, n
    parts, counts = [], np.zeros(m, dtype=np.int64)
    for dx, dy in offs:
        mask = (x + dx >= 0) & (x + dx < n) & (y + dy >= 0) & (y + dy < n)
        counts += mask
        parts.append((mask, (idx + dx + dy * n).astype(np.int32), diag if (dx, dy) == (0, 0) else off))
    return _assemble(m, m, counts, parts)


def stencil_3d27(n: int, diag: float = 26.0, off: float = -1.0) -> CSR:
    """3-D 27-point stencil on n^3, row i = (n*z + y)*n + x, A = 27 I - S (BASELINE config 1, n = 128)."""
    m = n ** 3
    idx = np.arange(m, dtype=np.int64)
    x, y, z = idx % n, (idx // n) % n, idx // (n * n)
    parts, counts = [], np.zeros(m, dtype=np.int64)
    for dz in (-1, 0, 1):
        mz = (z + dz >= 0) & (z + dz < n)
        for dy in (-1, 0, 1):
            my = mz & (y + dy >= 0) & (y + dy < n)
            for dx in (-1, 0, 1):
                mask = my & (x + dx >= 0) & (x + dx < n)
                counts += mask
                c = (idx + dx + dy * n + dz * n * n).astype(np.int32)
                parts.append((mask, c, diag if (dx, dy, dz) == (0, 0, 0) else off))
    return _assemble(m, m, counts, parts)


def _coo_to_csr(nrows, ncols, r, c, rng, values="uniform"):
    key = r.astype(np.int64) * ncols + c.astype(np.int64)
    key = np.unique(key)
    r = (key // ncols).astype(np.int64)
    c = (key % ncols).astype(np.int32)
    rp = np.zeros(nrows + 1, dtype=np.int64)
    np.cumsum(np.bincount(r, minlength=nrows), out=rp[1:])
    if values == "uniform":
        v = rng.uniform(-1.0, 1.0, size=len(c))
    elif values == "positive":
        v = rng.uniform(0.5, 1.5, size=len(c))
    elif values == "ones":
        v = np.ones(len(c))
    else:
        raise ValueError(values)
    return CSR(nrows, ncols, rp, c, v.astype(np.float64))


def _rmat_bits(rng, nedges, row_scale, col_scale, a, b, c):
    """R-MAT edge endpoints: each level picks a quadrant with probabilities (a, b, c, d)."""
    r = np.zeros(nedges, dtype=np.int64)
    q = np.zeros(nedges, dtype=np.int64)
    levels = max(row_scale, col_scale)
    for lvl in range(levels):
        u = rng.random(nedges, dtype=np.float32)
        if lvl < row_scale and lvl < col_scale:
            rbit = u >= (a + b)
            cbit = np.where(rbit, u >= (a + b + c), u >= a)
        elif lvl < row_scale:
            rbit, cbit = u >= (a + b), None
        else:
            rbit, cbit = None, u >= (a + c)
        if rbit is not None:
            r = (r << 1) | rbit
        if cbit is not None:
            q = (q << 1) | cbit
    return r, q


def rmat(scale: int, edge_factor: int = 16, a=0.45, b=0.20, c=0.20, seed: int = 20210517,
         symmetric: bool = True, values: str = "uniform") -> CSR:
    """R-MAT graph, 2^scale vertices, edge_factor*2^scale generated edges, ids scrambled,
    symmetrised, deduplicated, no self-loops (BASELINE configs 2/3; reading R17)."""
    rng = np.random.default_rng(seed)
    n = 1 << scale
    ne = edge_factor * n
    r, q = _rmat_bits(rng, ne, scale, scale, a, b, c)
    perm = rng.permutation(n)
    r, q = perm[r], perm[q]
    keep = r != q
    r, q = r[keep], q[keep]
    if symmetric:
        r, q = np.concatenate([r, q]), np.concatenate([q, r])
    return _coo_to_csr(n, n, r, q, rng, values)


def rmat_torch(scale: int, edge_factor: int = 16, a=0.45, b=0.20, c=0.20, seed: int = 20210517,
               device="cuda", col_scale: int | None = None, nedges: int | None = None, symmetric: bool = True):
    """The R-MAT recipe of `rmat` / `rmat_rect` drawn with torch's Philox generator on a GPU (seconds
    instead of minutes at scale 22-24; a different stream of random numbers than the numpy
    version, so a different -- equally distributed -- matrix).  Returns a CSR of numpy arrays.
    Square and symmetrised by default; col_scale/nedges give the rectangular variant."""
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    rs = scale
    cs = scale if col_scale is None else col_scale
    ne = edge_factor * (1 << rs) if nedges is None else nedges
    r = torch.zeros(ne, dtype=torch.int64, device=device)
    q = torch.zeros(ne, dtype=torch.int64, device=device)
    for lvl in range(max(rs, cs)):
        u = torch.rand(ne, generator=g, device=device)
        if lvl < rs and lvl < cs:
            rbit = u >= (a + b)
            cbit = torch.where(rbit, u >= (a + b + c), u >= a)
        elif lvl < rs:
            rbit, cbit = u >= (a + b), None
        else:
            rbit, cbit = None, u >= (a + c)
        if rbit is not None:
            r = (r << 1) | rbit.to(torch.int64)
        if cbit is not None:
            q = (q << 1) | cbit.to(torch.int64)
        del u
    nr, nc = 1 << rs, 1 << cs
    pr = torch.randperm(nr, generator=g, device=device)
    pc = pr if rs == cs else torch.randperm(nc, generator=g, device=device)  # square: relabel vertices
    r, q = pr[r], pc[q]
    if symmetric and rs == cs:
        keep = r != q
        r, q = r[keep], q[keep]
        r, q = torch.cat([r, q]), torch.cat([q, r])
    key = torch.unique(r * nc + q)
    del r, q
    rows = key // nc
    cols = (key % nc).to(torch.int32)
    rp = torch.zeros(nr + 1, dtype=torch.int64, device=device)
    rp[1:] = torch.cumsum(torch.bincount(rows, minlength=nr), 0)
    vals = torch.rand(len(key), generator=g, device=device, dtype=torch.float64) * 2.0 - 1.0
    return CSR(nr, nc, rp.cpu().numpy(), cols.cpu().numpy(), vals.cpu().numpy())


def rmat_rect(row_scale: int, col_scale: int, nedges: int, a=0.45, b=0.20, c=0.20,
              seed: int = 7, values: str = "uniform") -> CSR:
    """Rectangular power-law matrix 2^row_scale x 2^col_scale (BASELINE config 4)."""
    rng = np.random.default_rng(seed)
    r, q = _rmat_bits(rng, nedges, row_scale, col_scale, a, b, c)
    r = rng.permutation(1 << row_scale)[r]
    q = rng.permutation(1 << col_scale)[q]
    return _coo_to_csr(1 << row_scale, 1 << col_scale, r, q, rng, values)


def random_csr(nrows: int, ncols: int, density: float, seed: int, values: str = "uniform",
               empty_rows: float = 0.0) -> CSR:
    """Uniform random sparsity pattern (tiny brute-force cases and ragged tails)."""
    rng = np.random.default_rng(seed)
    if nrows == 0 or ncols == 0:
        return CSR(nrows, ncols, np.zeros(nrows + 1, dtype=np.int64), np.zeros(0, np.int32), np.zeros(0))
    mask = rng.random((nrows, ncols)) < density
    if empty_rows > 0:
        mask[rng.random(nrows) < empty_rows, :] = False
    r, c = np.nonzero(mask)
    return _coo_to_csr(nrows, ncols, r, c, rng, values)


def random_csr_sparse(nrows: int, ncols: int, nnz_per_row: float, seed: int, values: str = "uniform") -> CSR:
    """Random pattern without a dense mask (large sizes); nnz per row ~ Poisson(nnz_per_row)."""
    rng = np.random.default_rng(seed)
    counts = rng.poisson(nnz_per_row, size=nrows)
    r = np.repeat(np.arange(nrows, dtype=np.int64), counts)
    c = rng.integers(0, ncols, size=len(r))
    return _coo_to_csr(nrows, ncols, r, c, rng, values)


def identity(n: int, scale: float = 1.0) -> CSR:
    return CSR(n, n, np.arange(n + 1, dtype=np.int64), np.arange(n, dtype=np.int32), np.full(n, scale))


def permutation(perm: np.ndarray) -> CSR:
    """Permutation matrix P with P[i, perm[i]] = 1."""
    n = len(perm)
    return CSR(n, n, np.arange(n + 1, dtype=np.int64), np.asarray(perm, dtype=np.int32), np.ones(n))


def fig2_instance():
    """The text-recoverable part of PAPER.md Fig. 2 (§II-B): row 0 of A has nonzeros in
    columns 0 and 2; rows 0 and 2 of B hold only column ids {0, 3}, both containing column 0.
    Values are ours (the figure's pixels are not in the text); see tests/golden/fig2_row0.txt."""
    A = CSR(1, 4, np.array([0, 2], dtype=np.int64), np.array([0, 2], dtype=np.int32), np.array([2.0, 3.0]))
    B = CSR(4, 4, np.array([0, 2, 2, 3, 3], dtype=np.int64), np.array([0, 3, 0], dtype=np.int32),
            np.array([5.0, 7.0, 11.0]))
    return A, B


def config(idx: int, small: bool = False):
    """(A, B, budget_bytes, name) for BASELINE.json configs[idx] (full size unless small=True).

    config 0: 2-D 5-pt 64x64, in-core.   config 1: 3-D 27-pt 128^3, budget 2 GiB.
    config 2: R-MAT s22 ef16.            config 3: R-MAT s24 ef16.   config 4: rect 2^24 x 2^22 times 2^22 x 2^24.
    """
    if idx == 0:
        A = stencil_2d5(64)
        return A, A, None, "C1: 2D 5-pt Laplacian 64x64, C=A*A, in-core"
    if idx == 1:
        A = stencil_3d27(32 if small else 128)
        return A, A, 2 << 30, f"C2: 3D 27-pt stencil {A.nrows}, C=A*A, budget 2 GiB"
    if idx == 2:
        A = rmat(12 if small else 22)
        return A, A, None, f"C3: R-MAT s{12 if small else 22} ef16 sym, C=A*A"
    if idx == 3:
        A = rmat(13 if small else 24)
        return A, A, None, f"C4: R-MAT s{13 if small else 24} ef16 sym, C=A*A"
    if idx == 4:
        if small:
            A = rmat_rect(14, 12, 60000, seed=11)
            B = rmat_rect(12, 14, 60000, seed=12)
        else:
            A = rmat_rect(24, 22, 1 << 28, seed=11)
            B = rmat_rect(22, 24, 1 << 28, seed=12)
        return A, B, None, "C5: rect power-law A (m x k) times B (k x n)"
    raise ValueError(idx)
