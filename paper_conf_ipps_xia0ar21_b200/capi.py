"""Thin ctypes binding of the C ABI in include/spgemm.h (argument marshalling only).

Every step of the hot path runs in libspgemm_b200.so (sm_100a kernels + the chunk pipeline);
this module only converts numpy arrays / torch tensors to pointers and status codes to
exceptions.  There is no fallback: if the shared library is missing, importing this module
raises, loudly.  PyTorch is used only for device memory (workspace, device-resident inputs)
and streams.
"""
from __future__ import annotations

import ctypes
import os
from typing import Callable, Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# SPGEMM_CHECKED=1 loads the checked build (device-side bounds checks that trap; build.py), for tests
LIB_PATH = os.path.join(_HERE, "libspgemm_b200_checked.so" if os.environ.get("SPGEMM_CHECKED") == "1"
                        else "libspgemm_b200.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build the CUDA library first (python -c 'import __graft_entry__ as g; g.build()')")

_lib = ctypes.CDLL(LIB_PATH)

# status codes (include/spgemm.h)
OK, ERR_INVALID_ARGUMENT, ERR_SHAPE, ERR_INDEX_OVERFLOW, ERR_BUDGET, ERR_HOST_ALLOC, ERR_CUDA, ERR_STATE, \
    ERR_CAPACITY, ERR_CALLBACK = range(10)
HOST, DEVICE = 0, 1


class spgemm_csr(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int64), ("ncols", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("col_idx", ctypes.c_void_p), ("values", ctypes.c_void_p),
                ("where", ctypes.c_int32), ("reserved", ctypes.c_int32)]


class spgemm_csr_out(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int64), ("ncols", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("col_idx", ctypes.c_void_p), ("values", ctypes.c_void_p)]


class spgemm_opts(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("validate", ctypes.c_int32), ("ring", ctypes.c_int32),
                ("profile", ctypes.c_int32), ("row_begin", ctypes.c_int64), ("row_end", ctypes.c_int64),
                ("workspace", ctypes.c_void_p), ("stream", ctypes.c_void_p), ("chunk_nnz", ctypes.c_int64),
                ("row_ptr_base", ctypes.c_int64), ("min_chunks", ctypes.c_int64), ("fused", ctypes.c_int32),
                ("col_panels", ctypes.c_int32), ("order", ctypes.c_int32), ("reserved", ctypes.c_int32)]


class spgemm_info(ctypes.Structure):
    _fields_ = [("nrows", ctypes.c_int64), ("ncols", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("products", ctypes.c_int64), ("max_row_nnz", ctypes.c_int64), ("max_row_products", ctypes.c_int64),
                ("num_chunks", ctypes.c_int32), ("ring", ctypes.c_int32), ("chunk_capacity", ctypes.c_int64),
                ("arena_bytes", ctypes.c_int64), ("arena_used", ctypes.c_int64), ("ring_bytes", ctypes.c_int64),
                ("rows_warp", ctypes.c_int64), ("rows_block", ctypes.c_int64), ("rows_global", ctypes.c_int64),
                ("fused", ctypes.c_int32), ("num_copies", ctypes.c_int32),
                ("col_panels", ctypes.c_int32), ("reserved", ctypes.c_int32), ("rows_medium", ctypes.c_int64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class spgemm_kernel_stat(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char * 24), ("launches", ctypes.c_int32), ("ms", ctypes.c_double),
                ("bytes", ctypes.c_double)]


CHUNK_CB = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p,
                            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64)

_P, _I64, _SZ = ctypes.c_void_p, ctypes.c_int64, ctypes.c_size_t
_sig = {
    "spgemm_opts_default": (None, [ctypes.POINTER(spgemm_opts)]),
    "spgemm_plan": (ctypes.c_int, [ctypes.POINTER(spgemm_csr), ctypes.POINTER(spgemm_csr), _SZ,
                                   ctypes.POINTER(spgemm_opts), ctypes.POINTER(ctypes.c_void_p)]),
    "spgemm_plan_info": (ctypes.c_int, [_P, ctypes.POINTER(spgemm_info)]),
    "spgemm_plan_chunks": (ctypes.c_int, [_P, _P, _P]),
    "spgemm_execute_into": (ctypes.c_int, [_P, _P, _P, _P]),
    "spgemm_execute_capacity": (ctypes.c_int, [_P, _P, _P, _P, _I64, ctypes.POINTER(ctypes.c_int64)]),
    "spgemm_execute": (ctypes.c_int, [_P, ctypes.POINTER(spgemm_csr_out)]),
    "spgemm_execute_stream": (ctypes.c_int, [_P, CHUNK_CB, _P]),
    "spgemm_set_row_ptr_base": (ctypes.c_int, [_P, _I64]),
    "spgemm_multiply": (ctypes.c_int, [ctypes.POINTER(spgemm_csr), ctypes.POINTER(spgemm_csr), _SZ,
                                       ctypes.POINTER(spgemm_opts), _P, _P, _P, _I64, ctypes.POINTER(ctypes.c_int64)]),
    "spgemm_stats": (ctypes.c_int, [_P, ctypes.POINTER(spgemm_kernel_stat), ctypes.c_int32,
                                    ctypes.POINTER(ctypes.c_int32)]),
    "spgemm_free": (None, [_P]),
    "spgemm_release_cache": (None, []),
    "spgemm_status_string": (ctypes.c_char_p, [ctypes.c_int]),
    "spgemm_last_error": (ctypes.c_char_p, []),
    "spgemm_abi_version": (ctypes.c_int32, []),
    "spgemm_kernel_launches": (ctypes.c_int64, []),
}
for _name, (_res, _args) in _sig.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED = tuple(_sig)


class SpgemmError(RuntimeError):
    def __init__(self, status: int, msg: str):
        self.status = status
        super().__init__(f"{_lib.spgemm_status_string(status).decode()}: {msg}")


def _check(st: int):
    if st != OK:
        raise SpgemmError(st, (_lib.spgemm_last_error() or b"").decode())


def status_string(st: int) -> str:
    return _lib.spgemm_status_string(st).decode()


def abi_version() -> int:
    return _lib.spgemm_abi_version()


# ----------------------------------------------------------------------------------- marshalling

def _ptr(x) -> Optional[int]:
    if x is None:
        return None
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    return x.data_ptr()  # torch tensor


def _is_cuda(x) -> bool:
    return not isinstance(x, np.ndarray) and getattr(x, "is_cuda", False)


def make_csr(M) -> tuple:
    """M has nrows, ncols, row_ptr (int64), col (int32), val (fp64) as numpy arrays or torch tensors
    (all on the host, or all on one CUDA device).  Returns (spgemm_csr, keepalive)."""
    rp, col, val = M.row_ptr, M.col, M.val
    dev = _is_cuda(rp)
    if dev:
        import torch
        assert rp.dtype == torch.int64 and col.dtype == torch.int32 and val.dtype == torch.float64
        assert rp.is_contiguous() and col.is_contiguous() and val.is_contiguous()
        assert col.is_cuda and val.is_cuda
        nnz = int(col.numel())
    else:
        if isinstance(rp, np.ndarray):
            rp = np.ascontiguousarray(rp, dtype=np.int64)
            col = np.ascontiguousarray(col, dtype=np.int32)
            val = np.ascontiguousarray(val, dtype=np.float64)
        nnz = int(rp[-1]) if len(rp) else 0
    c = spgemm_csr(int(M.nrows), int(M.ncols), nnz, _ptr(rp), _ptr(col),
                   _ptr(val), DEVICE if dev else HOST, 0)
    return c, (rp, col, val)


def opts(device: int = -1, validate: bool = False, ring: int = 2, profile: bool = False, row_begin: int = 0,
         row_end: int = -1, workspace=None, stream=None, chunk_nnz: int = 0, row_ptr_base: int = 0,
         min_chunks: int = 0, fused: bool = False, col_panels: int = 0, order: int = 0) -> spgemm_opts:
    o = spgemm_opts()
    _lib.spgemm_opts_default(ctypes.byref(o))
    o.device, o.validate, o.ring, o.profile = device, int(validate), ring, int(profile)
    o.row_begin, o.row_end = row_begin, row_end
    o.workspace = _ptr(workspace) if workspace is not None else None
    o.stream = stream
    o.chunk_nnz, o.row_ptr_base, o.min_chunks = chunk_nnz, row_ptr_base, min_chunks
    o.fused = int(fused)
    o.col_panels = int(col_panels)
    o.order = int(order)
    o._keep = workspace  # the caller's workspace tensor must outlive the plan
    return o


class Plan:
    """Owns a spgemm_plan_t.  Methods mirror the C entry points."""

    def __init__(self, A, B, budget: int = 0, o: Optional[spgemm_opts] = None):
        ca, self._ka = make_csr(A)
        cb, self._kb = make_csr(B)
        self._opts = o if o is not None else opts()
        self._ws = getattr(self._opts, "_keep", None)
        h = ctypes.c_void_p()
        _check(_lib.spgemm_plan(ctypes.byref(ca), ctypes.byref(cb), budget, ctypes.byref(self._opts), ctypes.byref(h)))
        self.h = h

    def info(self) -> dict:
        i = spgemm_info()
        _check(_lib.spgemm_plan_info(self.h, ctypes.byref(i)))
        return i.as_dict()

    def chunks(self):
        n = self.info()["num_chunks"]
        rows = np.zeros(n + 1, dtype=np.int64)
        offs = np.zeros(n + 1, dtype=np.int64)
        _check(_lib.spgemm_plan_chunks(self.h, rows.ctypes.data, offs.ctypes.data))
        return rows, offs

    def execute_into(self, row_ptr, col, val):
        _check(_lib.spgemm_execute_into(self.h, _ptr(row_ptr), _ptr(col), _ptr(val)))

    def execute_capacity(self, row_ptr, col, val, capacity: int) -> int:
        """Returns nnz(C); raises SpgemmError(ERR_CAPACITY) (with .nnz) if it exceeds capacity."""
        nnz = ctypes.c_int64(-1)
        st = _lib.spgemm_execute_capacity(self.h, _ptr(row_ptr), _ptr(col), _ptr(val), int(capacity),
                                          ctypes.byref(nnz))
        if st == ERR_CAPACITY:
            e = SpgemmError(st, (_lib.spgemm_last_error() or b"").decode())
            e.nnz = nnz.value
            raise e
        _check(st)
        return nnz.value

    def execute(self):
        """Plan-owned pinned output; returns numpy views valid until free()."""
        out = spgemm_csr_out()
        _check(_lib.spgemm_execute(self.h, ctypes.byref(out)))
        n, z = out.nrows, out.nnz
        rp = np.ctypeslib.as_array((ctypes.c_int64 * (n + 1)).from_address(out.row_ptr))
        col = np.ctypeslib.as_array((ctypes.c_int32 * max(z, 1)).from_address(out.col_idx))[:z]
        val = np.ctypeslib.as_array((ctypes.c_double * max(z, 1)).from_address(out.values))[:z]
        return rp, col, val

    def execute_stream(self, fn: Callable):
        """fn(row0, row1, row_ptr, col, val) gets numpy views of each chunk (valid during the call)."""
        err = []

        def cb(user, r0, r1, rp, col, val, nnz):
            try:
                a_rp = np.ctypeslib.as_array((ctypes.c_int64 * (r1 - r0 + 1)).from_address(rp))
                a_col = np.ctypeslib.as_array((ctypes.c_int32 * max(nnz, 1)).from_address(col))[:nnz] if nnz else \
                    np.zeros(0, np.int32)
                a_val = np.ctypeslib.as_array((ctypes.c_double * max(nnz, 1)).from_address(val))[:nnz] if nnz else \
                    np.zeros(0)
                r = fn(r0, r1, a_rp, a_col, a_val)
                return int(r or 0)
            except Exception as e:  # noqa: BLE001
                err.append(e)
                return 1

        cfun = CHUNK_CB(cb)
        st = _lib.spgemm_execute_stream(self.h, cfun, None)
        if err:
            raise err[0]
        _check(st)

    def row_bounds(self) -> np.ndarray:
        """The plan's per-row bounds min(products, ncols) (spgemm_plan_row_bounds)."""
        out = np.zeros(max(self.info()["nrows"], 1), dtype=np.int64)
        _check(_lib.spgemm_plan_row_bounds(self.h, out.ctypes.data))
        return out[:self.info()["nrows"]]

    def set_row_ptr_base(self, base: int):
        _check(_lib.spgemm_set_row_ptr_base(self.h, int(base)))

    def stats(self) -> dict:
        n = ctypes.c_int32()
        arr = (spgemm_kernel_stat * 64)()
        _check(_lib.spgemm_stats(self.h, arr, 64, ctypes.byref(n)))
        return {arr[k].name.decode(): {"launches": arr[k].launches, "ms": arr[k].ms, "bytes": arr[k].bytes}
                for k in range(min(n.value, 64))}

    def free(self):
        if getattr(self, "h", None):
            _lib.spgemm_free(self.h)
            self.h = None

    def __del__(self):
        try:
            self.free()
        except Exception:  # noqa: BLE001
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.free()


def spgemm_plan(A, B, budget: int = 0, o: Optional[spgemm_opts] = None) -> Plan:
    return Plan(A, B, budget, o)


def spgemm_multiply(A, B, budget: int, o: Optional[spgemm_opts], row_ptr, col, val, capacity: int) -> int:
    ca, ka = make_csr(A)
    cb, kb = make_csr(B)
    o = o if o is not None else opts()
    nnz = ctypes.c_int64(0)
    st = _lib.spgemm_multiply(ctypes.byref(ca), ctypes.byref(cb), budget, ctypes.byref(o), _ptr(row_ptr), _ptr(col),
                              _ptr(val), int(capacity), ctypes.byref(nnz))
    if st == ERR_CAPACITY:
        raise SpgemmError(st, f"need capacity {nnz.value}")
    _check(st)
    return nnz.value


def kernel_launches() -> int:
    return int(_lib.spgemm_kernel_launches())


def release_cache():
    _lib.spgemm_release_cache()


_lib.spgemm_timeline.restype = ctypes.c_int
_lib.spgemm_timeline.argtypes = [_P, _P, _I64, ctypes.POINTER(ctypes.c_int64)]
EXPORTED = EXPORTED + ("spgemm_timeline",)


def timeline(plan: "Plan") -> np.ndarray:
    """[chunks, 6] ms: symbolic start/end, numeric start/end, copy start/end (profile plans)."""
    n = ctypes.c_int64()
    _check(_lib.spgemm_timeline(plan.h, None, 0, ctypes.byref(n)))
    out = np.zeros(max(n.value, 1), dtype=np.float64)
    _check(_lib.spgemm_timeline(plan.h, out.ctypes.data, n.value, ctypes.byref(n)))
    return out[:n.value].reshape(-1, 6)


_lib.spgemm_rebase_host.restype = ctypes.c_int
_lib.spgemm_rebase_host.argtypes = [_P, _I64, _I64]
EXPORTED = EXPORTED + ("spgemm_rebase_host",)


def rebase_host(row_ptr, delta: int) -> None:
    """row_ptr[:] += delta in place (host int64 array / tensor), in the library."""
    n = row_ptr.shape[0]
    _check(_lib.spgemm_rebase_host(_ptr(row_ptr), int(n), int(delta)))


_lib.spgemm_row_products.restype = ctypes.c_int
_lib.spgemm_row_products.argtypes = [ctypes.POINTER(spgemm_csr), ctypes.POINTER(spgemm_csr),
                                     ctypes.POINTER(spgemm_opts), _P, ctypes.POINTER(ctypes.c_int64)]
_lib.spgemm_plan_row_bounds.restype = ctypes.c_int
_lib.spgemm_plan_row_bounds.argtypes = [_P, _P]
EXPORTED = EXPORTED + ("spgemm_row_products", "spgemm_plan_row_bounds")


def row_products(A, B, o: Optional[spgemm_opts] = None):
    """(u, total): intermediate products of every row of A x B in the plan's row range, by the
    library's count kernel (spgemm_row_products)."""
    ca, ka = make_csr(A)
    cb, kb = make_csr(B)
    o = o if o is not None else opts()
    r1 = int(A.nrows) if o.row_end < 0 else int(o.row_end)
    u = np.zeros(max(r1 - int(o.row_begin), 1), dtype=np.int64)
    tot = ctypes.c_int64(0)
    _check(_lib.spgemm_row_products(ctypes.byref(ca), ctypes.byref(cb), ctypes.byref(o), u.ctypes.data,
                                    ctypes.byref(tot)))
    return u[:r1 - int(o.row_begin)], tot.value
