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
degenerate shapes, and ESC-vs-SPA agreement.  The checkers `compare()` (against a stored
oracle result) and `verify()` (rows checked while the oracle computes them, for C larger
than host memory) are pinned by mutation tests: every kind of wrong candidate -- a row_ptr
entry, a column, a value just outside the bound, an infinity of the wrong sign, a NaN --
must be rejected, and correct candidates (including equal infinities and NaNs) accepted.
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
        _lib.oracle_verify.argtypes = [P, P, I64, I64, P, P, P, P, I, P, P]
        _lib.oracle_verify_ctx_new.argtypes = [I64, I]
        _lib.oracle_verify_ctx_new.restype = P
        _lib.oracle_verify_ctx_free.argtypes = [P]
        _lib.oracle_verify_ctx_free.restype = None
        for f in (_lib.oracle_products, _lib.oracle_row_nnz, _lib.oracle_numeric, _lib.oracle_numeric_esc,
                  _lib.oracle_verify):
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


def _value_good(val, ref, tol):
    """The value rule (SURVEY.md §8(c) "Comparison rule", oracle.c header): NaN on either side ->
    good iff both NaN; Inf on either side -> good iff equal; else |val - ref| <= tol (tol = 0 ->
    val must equal ref exactly).  Returns (good mask, ratio |val - ref| / tol for finite entries)."""
    nan = np.isnan(val) | np.isnan(ref)
    inf = ~nan & (np.isinf(val) | np.isinf(ref))
    fin = ~nan & ~inf
    with np.errstate(invalid="ignore", divide="ignore", over="ignore"):
        err = np.where(fin, np.abs(val - ref), 0.0)
        ratio = np.where(err == 0, 0.0, np.where(tol > 0, err / np.where(tol > 0, tol, 1.0), np.inf))
    good = np.where(nan, np.isnan(val) & np.isnan(ref), np.where(inf, val == ref, err <= tol))
    return good, np.where(fin, ratio, 0.0)


def compare(rp, col, val, expect: dict, rows_offset: int = 0) -> dict:
    """Parity rule: row_ptr and col bit-identical to the oracle's,
    every value good by `_value_good` against the oracle's long-double `ref` and `tol`.

    `rp/col/val` are the candidate's arrays for the same row selection; rp minus `rows_offset`
    must start at 0.  col / val must hold exactly rp[-1] entries.
    Returns dict(ok, worst_ratio, n, first_bad) with first_bad = (kind, index) or None.
    Pinned by tests/test_oracle.py::test_compare_* (mutations of every part must be rejected).
    """
    rp = np.asarray(rp, dtype=np.int64) - int(rows_offset)
    col = np.asarray(col)
    val = np.asarray(val, dtype=np.float64)
    res = {"ok": True, "worst_ratio": 0.0, "n": int(len(expect["col"])), "first_bad": None}
    erp = expect["row_ptr"]
    if len(rp) != len(erp) or not np.array_equal(rp, erp):
        bad = int(np.nonzero(rp != erp)[0][0]) if len(rp) == len(erp) else -1
        res.update(ok=False, first_bad=("row_ptr", bad))
        return res
    if len(col) != len(expect["col"]) or len(val) != len(expect["col"]):
        res.update(ok=False, first_bad=("length", -1))
        return res
    if not np.array_equal(col, expect["col"]):
        bad = int(np.nonzero(col != expect["col"])[0][0])
        res.update(ok=False, first_bad=("col", bad))
        return res
    good, ratio = _value_good(val, expect["ref"], expect["tol"])
    if len(ratio):
        res["worst_ratio"] = float(np.max(np.where(good, ratio, 0.0)))
    if not np.all(good):
        res.update(ok=False, first_bad=("val", int(np.nonzero(~good)[0][0])))
    return res


class _VStat(ctypes.Structure):
    _fields_ = [("rows", ctypes.c_int64), ("entries", ctypes.c_int64), ("products", ctypes.c_int64),
                ("bad_rows", ctypes.c_int64), ("bad_row_ptr", ctypes.c_int64), ("bad_col", ctypes.c_int64),
                ("bad_val", ctypes.c_int64), ("bad_products", ctypes.c_int64), ("first_bad_row", ctypes.c_int64),
                ("first_bad_kind", ctypes.c_int32), ("pad", ctypes.c_int32), ("worst_ratio", ctypes.c_double)]


_KINDS = {0: None, 1: "row_ptr", 2: "col", 3: "val", 4: "products"}


class Operands:
    """A, B marshalled once, plus persistent per-thread verify scratch, for repeated verify()
    calls (a sink checks chunk after chunk)."""

    def __init__(self, A, B, threads: Optional[int] = None):
        _check_shapes(A, B)
        self.sa, self.ka = _mk(A)
        self.sb, self.kb = _mk(B)
        self.nrows = int(A.nrows)
        self.threads = threads or default_threads()
        self.ctx = _load().oracle_verify_ctx_new(int(B.ncols), self.threads)
        if not self.ctx:
            raise MemoryError("oracle_verify_ctx_new failed")

    def __del__(self):
        if getattr(self, "ctx", None):
            _load().oracle_verify_ctx_free(self.ctx)
            self.ctx = None


def verify(A, B, row0: int, rp, col, val, products=None, threads: Optional[int] = None,
           ops: Optional[Operands] = None) -> dict:
    """Check candidate rows row0 .. row0 + len(rp) - 2 of C = A x B against Alg. 1 without storing
    the oracle's output (oracle.c oracle_verify; the same rule as compare()).  rp: the rows'
    offsets (any base), col / val: their entries, products: optional per-row product counts.
    Returns dict(ok, rows, entries, products, bad_*, first_bad_row, first_bad_kind, worst_ratio)."""
    ops = ops or Operands(A, B)
    rp = np.ascontiguousarray(rp, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    val = np.ascontiguousarray(val, dtype=np.float64)
    n = len(rp) - 1
    if n < 0 or len(col) < rp[-1] - rp[0] or len(val) < rp[-1] - rp[0]:
        raise ValueError("candidate arrays shorter than their row_ptr says")
    pr = None if products is None else np.ascontiguousarray(products, dtype=np.int64)
    if pr is not None and len(pr) != n:
        raise ValueError("products must have one entry per row")
    st = _VStat()
    rc = _load().oracle_verify(ctypes.byref(ops.sa), ctypes.byref(ops.sb), int(row0), n, _ptr(rp), _ptr(col),
                               _ptr(val), _ptr(pr), threads or ops.threads, ctypes.byref(st), ops.ctx)
    if rc:
        raise RuntimeError(f"oracle_verify failed ({rc})")
    out = {k: getattr(st, k) for k, _ in _VStat._fields_ if k != "pad"}
    out["first_bad_kind"] = _KINDS[st.first_bad_kind]
    out["ok"] = st.bad_rows == 0 and st.bad_products == 0 and st.rows == n
    return out
