"""CPU oracle for C = A x B on CSR -- TEST INFRASTRUCTURE ONLY.

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s `cpu_baseline` /
`--impl reference` legs may import this package.  The product path
(`paper_conf_ipps_xia0ar21_b200/`) never imports it and shares no code with it.

The arithmetic lives in `oracle/oracle.c` (plain C, fp64 in Alg. 1 order plus a
long-double reference sum, see its header); this module only marshals numpy
arrays through ctypes.  `oracle.pyref` is a third, pure-Python implementation
of Alg. 1 for tiny inputs.

Pins (tests/test_oracle.py, `-m "not gpu"`): dense brute force, A*I = I*A = A,
permutation matrices, stencil closed forms (C1, C2), sum and Freivalds
identities, scipy on all-positive inputs, the paper's Fig. 2 (tests/golden/),
degenerate shapes, and ESC-vs-SPA agreement.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None

CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-pthread", "-Wall"]


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (the checker is built here; building it is not using it)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _SO)
    return _SO


class _OCSR(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int64), ("ncols", ctypes.c_int64),
                ("rp", ctypes.c_void_p), ("col", ctypes.c_void_p), ("val", ctypes.c_void_p)]


def _load():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        P, I64, I = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
        _lib.oracle_products.argtypes = [P, P, P, I64, P, I]
        _lib.oracle_row_nnz.argtypes = [P, P, P, I64, P, I]
        _lib.oracle_numeric.argtypes = [P, P, P, I64, P, P, P, P, P, I]
        _lib.oracle_numeric_esc.argtypes = [P, P, P, I64, P, P, P, I]
        for f in (_lib.oracle_products, _lib.oracle_row_nnz, _lib.oracle_numeric, _lib.oracle_numeric_esc):
            f.restype = ctypes.c_int
    return _lib


def _ptr(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _mk(M):
    rp = np.ascontiguousarray(M.row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(M.col, dtype=np.int32)
    val = np.ascontiguousarray(M.val, dtype=np.float64)
    s = _OCSR(int(M.nrows), int(M.ncols), rp.ctypes.data, col.ctypes.data, val.ctypes.data)
    return s, (rp, col, val)


def default_threads() -> int:
    try:
        return max(1, len(os.sched_getaffinity(0)))
    except Exception:
        return os.cpu_count() or 1


def _sel(A, rows):
    if rows is None:
        return None, int(A.nrows)
    r = np.ascontiguousarray(rows, dtype=np.int64)
    if len(r) and (r.min() < 0 or r.max() >= A.nrows):
        raise IndexError("row selection out of range")
    return r, len(r)


def _check_shapes(A, B):
    if int(A.ncols) != int(B.nrows):
        raise ValueError(f"shape mismatch: A is {A.nrows}x{A.ncols}, B is {B.nrows}x{B.ncols}")


def products(A, B, rows=None, threads: Optional[int] = None) -> np.ndarray:
    """u_i = number of intermediate products of row i (Alg. 1 line-4 trip count; §III-B)."""
    _check_shapes(A, B)
    r, n = _sel(A, rows)
    sa, ka = _mk(A)
    sb, kb = _mk(B)
    u = np.empty(n, dtype=np.int64)
    rc = _load().oracle_products(ctypes.byref(sa), ctypes.byref(sb), _ptr(r), n, _ptr(u), threads or default_threads())
    if rc:
        raise RuntimeError(f"oracle_products failed ({rc})")
    return u


def row_nnz(A, B, rows=None, threads: Optional[int] = None) -> np.ndarray:
    """nnz of each C row (the symbolic count, §II-B)."""
    _check_shapes(A, B)
    r, n = _sel(A, rows)
    sa, ka = _mk(A)
    sb, kb = _mk(B)
    out = np.empty(n, dtype=np.int64)
    rc = _load().oracle_row_nnz(ctypes.byref(sa), ctypes.byref(sb), _ptr(r), n, _ptr(out), threads or default_threads())
    if rc:
        raise RuntimeError(f"oracle_row_nnz failed ({rc})")
    return out


def spgemm(A, B, rows=None, threads: Optional[int] = None, with_ref: bool = True, method: str = "spa") -> dict:
    """C = A x B restricted to the selected rows (all rows if None).

    Returns dict(row_ptr int64 [nsel+1] (starting at 0), col int32, val fp64 (Alg. 1 order),
    ref fp64 (long-double sum), tol fp64 (1e-12 * sum |a*b|), products int64 [nsel]).
    method = "spa" (Alg. 1 + marker array) or "esc" (expand/sort/compress; val only).
    """
    _check_shapes(A, B)
    r, n = _sel(A, rows)
    th = threads or default_threads()
    nnz = row_nnz(A, B, rows, th)
    rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(nnz, out=rp[1:])
    tot = int(rp[-1])
    col = np.empty(tot, dtype=np.int32)
    val = np.empty(tot, dtype=np.float64)
    ref = np.empty(tot, dtype=np.float64) if (with_ref and method == "spa") else None
    tol = np.empty(tot, dtype=np.float64) if (with_ref and method == "spa") else None
    sa, ka = _mk(A)
    sb, kb = _mk(B)
    lib = _load()
    if method == "spa":
        rc = lib.oracle_numeric(ctypes.byref(sa), ctypes.byref(sb), _ptr(r), n, _ptr(rp), _ptr(col), _ptr(val),
                                _ptr(ref), _ptr(tol), th)
    elif method == "esc":
        rc = lib.oracle_numeric_esc(ctypes.byref(sa), ctypes.byref(sb), _ptr(r), n, _ptr(rp), _ptr(col), _ptr(val), th)
    else:
        raise ValueError(method)
    if rc:
        raise RuntimeError(f"oracle numeric failed ({rc})")
    return {"row_ptr": rp, "col": col, "val": val, "ref": ref, "tol": tol}


def compare(rp, col, val, expect: dict, rows_offset: int = 0) -> dict:
    """Parity rule: row_ptr and col bit-identical, |val - ref| <= tol.

    `rp/col/val` are the candidate's arrays for the same row selection, with rp rebased to 0.
    Returns dict(ok, worst_ratio, n, first_bad).
    """
    rp = np.asarray(rp, dtype=np.int64) - int(rows_offset)
    res = {"ok": True, "worst_ratio": 0.0, "n": int(len(expect["col"])), "first_bad": None}
    if not np.array_equal(rp, expect["row_ptr"]):
        bad = int(np.nonzero(rp != expect["row_ptr"])[0][0]) if len(rp) == len(expect["row_ptr"]) else -1
        res.update(ok=False, first_bad=("row_ptr", bad))
        return res
    if not np.array_equal(np.asarray(col), expect["col"]):
        bad = int(np.nonzero(np.asarray(col) != expect["col"])[0][0])
        res.update(ok=False, first_bad=("col", bad))
        return res
    val = np.asarray(val, dtype=np.float64)
    ref, tol = expect["ref"], expect["tol"]
    err = np.abs(val - ref)
    nan_ok = np.isnan(val) == np.isnan(ref)
    with np.errstate(invalid="ignore", divide="ignore"):
        ratio = np.where(tol > 0, err / np.where(tol > 0, tol, 1), np.where(err == 0, 0.0, np.inf))
    ratio = np.where(np.isnan(ref) & np.isnan(val), 0.0, ratio)
    good = (ratio <= 1.0) & nan_ok
    if len(ratio):
        res["worst_ratio"] = float(np.nanmax(ratio))
    if not np.all(good):
        res.update(ok=False, first_bad=("val", int(np.nonzero(~good)[0][0])))
    return res
