"""Closed forms for C = A*A on the two stencil workloads (BASELINE configs 0 and 1).

These are derived by hand from the stencil definitions (reading R16), not
from any implementation, and pin both the oracle and the CUDA path:

C1: A = 2-D 5-point Laplacian on n x n (diag 4, off-diagonal -1, row i = n*y + x).
    C = A^2 has the 13-offset pattern |dx|+|dy| <= 2 with values
      diagonal      16 + (#grid neighbours of the point)   (20 interior / 19 edge / 18 corner)
      |d| = 1       -8      (A_ii*A_ij + A_ij*A_jj = 2 * 4 * (-1))
      straight 2    +1      (one path through the middle point)
      diagonal 1,1  +2      (two paths)
C2: A = 27 I - S on n^3, S = K (x) K (x) K, K = tridiag(1, 1, 1) (n x n, truncated at the boundary).
    A^2 = 729 I - 54 S + K^2 (x) K^2 (x) K^2, with (K^2)_{x,x'} = deg1(x) if x == x', 2 if |x-x'| = 1,
    1 if |x-x'| = 2 (deg1 = 2 at the ends, 3 inside).
    products of row (x,y,z) = s(x) s(y) s(z), s = [5, 8, 9, ..., 9, 8, 5];
    nnz of row (x,y,z)      = w(x) w(y) w(z), w = [3, 4, 5, ..., 5, 4, 3];
    totals (n = 128): products 1142^3 = 1,489,355,288, nnz 634^3 = 254,840,104.
Sum identity (any A, B): sum_ij C_ij = sum_k colsum_A(k) * rowsum_B(k).
"""
from __future__ import annotations

import numpy as np


def c1_entry(n: int, i: np.ndarray, j: np.ndarray) -> np.ndarray:
    """Exact value of (A^2)_{ij} for the 2-D 5-point Laplacian (vectorised)."""
    xi, yi = i % n, i // n
    xj, yj = j % n, j // n
    dx, dy = np.abs(xi - xj), np.abs(yi - yj)
    nb = (xi > 0).astype(int) + (xi < n - 1) + (yi > 0) + (yi < n - 1)
    out = np.zeros(len(i), dtype=np.float64)
    out[(dx == 0) & (dy == 0)] = (16 + nb)[(dx == 0) & (dy == 0)]
    out[(dx + dy) == 1] = -8.0
    out[((dx == 2) & (dy == 0)) | ((dx == 0) & (dy == 2))] = 1.0
    out[(dx == 1) & (dy == 1)] = 2.0
    return out


def c1_pattern_count(n: int) -> int:
    tot = 0
    for dx in range(-2, 3):
        for dy in range(-2, 3):
            if abs(dx) + abs(dy) <= 2:
                tot += (n - abs(dx)) * (n - abs(dy))
    return tot


def c1_products_total(n: int) -> int:
    # sum_k nnz(A_*k) * nnz(A_k*) = sum_k deg(k)^2, deg = 1 + #grid neighbours
    x = np.arange(n)
    nb1 = (x > 0).astype(np.int64) + (x < n - 1)
    deg = 1 + nb1[:, None] + nb1[None, :]
    return int((deg ** 2).sum())


def _deg1(n):
    x = np.arange(n)
    return 1 + (x > 0).astype(np.int64) + (x < n - 1)


def c2_s(n: int) -> np.ndarray:
    d = _deg1(n)
    s = d.copy()
    s[1:] += d[:-1]
    s[:-1] += d[1:]
    return s


def c2_w(n: int) -> np.ndarray:
    x = np.arange(n)
    return np.minimum(x, 2) + np.minimum(n - 1 - x, 2) + 1


def c2_row_products(n: int, rows: np.ndarray) -> np.ndarray:
    s = c2_s(n)
    return s[rows % n] * s[(rows // n) % n] * s[rows // (n * n)]


def c2_row_nnz(n: int, rows: np.ndarray) -> np.ndarray:
    w = c2_w(n)
    return w[rows % n] * w[(rows // n) % n] * w[rows // (n * n)]


def c2_totals(n: int):
    return int(c2_s(n).sum()) ** 3, int(c2_w(n).sum()) ** 3


def _k2(n, a, b):
    d1 = _deg1(n)
    dd = np.abs(a - b)
    return np.where(dd == 0, d1[a], np.where(dd == 1, 2, np.where(dd == 2, 1, 0)))


def c2_entry(n: int, i: np.ndarray, j: np.ndarray) -> np.ndarray:
    xi, yi, zi = i % n, (i // n) % n, i // (n * n)
    xj, yj, zj = j % n, (j // n) % n, j // (n * n)
    cheb = np.maximum(np.maximum(np.abs(xi - xj), np.abs(yi - yj)), np.abs(zi - zj))
    return (729.0 * (i == j) - 54.0 * (cheb <= 1)
            + _k2(n, xi, xj) * _k2(n, yi, yj) * _k2(n, zi, zj)).astype(np.float64)


def c2_sum(n: int) -> float:
    d = _deg1(n)
    rowsum = 27 - (d[:, None, None] * d[None, :, None] * d[None, None, :])
    return float((rowsum.astype(np.int64) ** 2).sum())


def c2_row_cols(n: int, i: int) -> np.ndarray:
    """Sorted column set of C2 row i: all points within Chebyshev distance 2."""
    x, y, z = i % n, (i // n) % n, i // (n * n)
    cols = []
    for dz in range(-2, 3):
        for dy in range(-2, 3):
            for dx in range(-2, 3):
                if 0 <= x + dx < n and 0 <= y + dy < n and 0 <= z + dz < n:
                    cols.append(i + dx + dy * n + dz * n * n)
    return np.array(sorted(cols), dtype=np.int64)
