"""CPU-side checks of the C ABI library (`-m "not gpu"`): it loads, exports every symbol
include/spgemm.h declares, and its host-only entry points (defaults, status strings, argument
and shape validation that precedes any CUDA call) behave as documented.  No compute call."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

import workloads as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "spgemm.h")


@pytest.fixture(scope="module")
def capi():
    from paper_conf_ipps_xia0ar21_b200 import build
    build.build()
    from paper_conf_ipps_xia0ar21_b200 import capi as c
    return c


def declared():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(spgemm_[a-z_]+)\s*\(", txt)) - {"spgemm_chunk_cb"})


def test_header_symbols_exported(capi):
    names = declared()
    assert len(names) >= 15
    out = subprocess.run(["nm", "-D", "--defined-only", capi.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (spgemm_\w+)", out))
    missing = [n for n in names if n not in exported]
    assert not missing, missing
    # and the binding wraps every one of them
    assert set(names) <= set(capi.EXPORTED)


def test_library_is_sm100a(capi):
    out = subprocess.run(["cuobjdump", "--list-elf", capi.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_defaults_and_strings(capi):
    o = capi.spgemm_opts()
    capi._lib.spgemm_opts_default(ctypes.byref(o))
    assert (o.device, o.ring, o.row_begin, o.row_end, o.validate) == (-1, 2, 0, -1, 0)
    assert capi.abi_version() == 3
    for st in range(10):
        assert capi.status_string(st).startswith("SPGEMM_")
    assert capi.status_string(4) == "SPGEMM_ERR_BUDGET"


def test_host_side_argument_errors(capi):
    """Errors detected before any CUDA call: NULL out-param, shape mismatch, bad row range,
    int32 column overflow, bad row_ptr."""
    A = W.random_csr(4, 5, 0.5, seed=1)
    B = W.random_csr(6, 3, 0.5, seed=2)
    ca, ka = capi.make_csr(A)
    cb, kb = capi.make_csr(B)
    assert capi._lib.spgemm_plan(ctypes.byref(ca), ctypes.byref(cb), 0, None, None) == capi.ERR_INVALID_ARGUMENT
    h = ctypes.c_void_p(123)
    st = capi._lib.spgemm_plan(ctypes.byref(ca), ctypes.byref(cb), 0, None, ctypes.byref(h))
    assert st == capi.ERR_SHAPE and h.value is None
    assert b"A.ncols" in capi._lib.spgemm_last_error()
    B2 = W.random_csr(5, 3, 0.5, seed=2)
    cb2, kb2 = capi.make_csr(B2)
    o = capi.opts(row_begin=2, row_end=7)
    assert capi._lib.spgemm_plan(ctypes.byref(ca), ctypes.byref(cb2), 0, ctypes.byref(o), ctypes.byref(h)) == capi.ERR_SHAPE
    big = capi.spgemm_csr(5, 1 << 31, 0, kb2[0].ctypes.data, kb2[1].ctypes.data, kb2[2].ctypes.data, 0, 0)
    rp = np.zeros(6, np.int64)
    big.row_ptr = rp.ctypes.data
    assert capi._lib.spgemm_plan(ctypes.byref(ca), ctypes.byref(big), 0, None, ctypes.byref(h)) == capi.ERR_INDEX_OVERFLOW
    badrp = A.row_ptr.copy()
    badrp[0] = 1
    cbad = capi.spgemm_csr(4, 5, A.nnz, badrp.ctypes.data, A.col.ctypes.data, A.val.ctypes.data, 0, 0)
    assert capi._lib.spgemm_plan(ctypes.byref(cbad), ctypes.byref(cb2), 0, None, ctypes.byref(h)) == capi.ERR_INVALID_ARGUMENT
    capi._lib.spgemm_free(None)  # NULL-safe


def test_binding_raises_without_library(tmp_path):
    """The product path fails loudly when the CUDA library is missing (no CPU fallback)."""
    code = ("import sys, importlib.util, os\n"
            f"spec = importlib.util.spec_from_file_location('capi_copy', r'{tmp_path}/capi.py')\n"
            "m = importlib.util.module_from_spec(spec)\n"
            "try:\n    spec.loader.exec_module(m)\nexcept ImportError as e:\n    print('IMPORTERROR', e)\n")
    src = open(os.path.join(ROOT, "paper_conf_ipps_xia0ar21_b200", "capi.py")).read()
    (tmp_path / "capi.py").write_text(src)
    out = subprocess.run(["python", "-c", code], capture_output=True, text=True).stdout
    assert "IMPORTERROR" in out and "libspgemm_b200.so is missing" in out


def test_product_package_does_not_import_oracle():
    """The product path never imports, links or executes the oracle."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_xia0ar21_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".h", ".cpp", ".cuh")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "liboracle" not in txt, f
    out = subprocess.run(["nm", "-D", os.path.join(pkg, "libspgemm_b200.so")], capture_output=True, text=True).stdout
    assert "oracle_" not in out


def test_struct_layouts_match_header(capi, tmp_path):
    """The ctypes mirrors have the C structs' sizes and field offsets (gcc on include/spgemm.h)."""
    import ctypes as ct
    src = tmp_path / "lay.c"
    fields = {"spgemm_opts": ["ring", "row_begin", "workspace", "stream", "chunk_nnz", "row_ptr_base", "min_chunks",
                              "fused", "col_panels", "order"],
              "spgemm_info": ["num_chunks", "chunk_capacity", "rows_global", "fused", "num_copies", "col_panels",
                              "rows_medium"],
              "spgemm_csr": ["row_ptr", "values", "where"], "spgemm_kernel_stat": ["launches", "ms", "bytes"]}
    lines = ["#include <stdio.h>", "#include <stddef.h>", f'#include "{HEADER}"', "int main(void) {"]
    for s, fs in fields.items():
        lines.append(f'printf("{s} %zu\\n", sizeof({s}));')
        for f in fs:
            lines.append(f'printf("{s}.{f} %zu\\n", offsetof({s}, {f}));')
    lines.append("return 0; }")
    src.write_text("\n".join(lines))
    exe = tmp_path / "lay"
    subprocess.run(["gcc", "-O0", "-o", str(exe), str(src)], check=True)
    got = dict(l.split() for l in subprocess.run([str(exe)], capture_output=True, text=True).stdout.splitlines())
    for s, fs in fields.items():
        cls = getattr(capi, s)
        assert int(got[s]) == ct.sizeof(cls), s
        for f in fs:
            assert int(got[f"{s}.{f}"]) == getattr(cls, f).offset, (s, f)


def test_order_needs_two_phase_plan(capi):
    """opts.order = 1 (the paper's decreasing-flops chunk schedule) is rejected on a fused plan
    before any CUDA call."""
    A = W.random_csr(4, 4, 0.5, seed=1)
    ca, ka = capi.make_csr(A)
    h = ctypes.c_void_p()
    o = capi.opts(order=1, fused=True)
    assert capi._lib.spgemm_plan(ctypes.byref(ca), ctypes.byref(ca), 0, ctypes.byref(o), ctypes.byref(h)) == \
        capi.ERR_INVALID_ARGUMENT
    assert b"two-phase" in capi._lib.spgemm_last_error()
    o = capi.opts(order=2)
    assert capi._lib.spgemm_plan(ctypes.byref(ca), ctypes.byref(ca), 0, ctypes.byref(o), ctypes.byref(h)) == \
        capi.ERR_INVALID_ARGUMENT


def test_checked_library_exports_the_same_abi_and_product_has_no_checks():
    """libspgemm_b200_checked.so (SPG_CHECK bounds checks, tests only) exports exactly the product
    library's C ABI; the product library carries none of the checks."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_xia0ar21_b200")

    def syms(name):
        out = subprocess.run(["nm", "-D", "--defined-only", os.path.join(pkg, name)], capture_output=True,
                             text=True).stdout
        return {ln.split()[-1] for ln in out.splitlines() if " T spgemm_" in ln}

    prod, chk = syms("libspgemm_b200.so"), syms("libspgemm_b200_checked.so")
    assert prod and prod == chk
    blob = open(os.path.join(pkg, "libspgemm_b200.so"), "rb").read()
    assert b"SPG_CHECK failed" not in blob
    assert b"SPG_CHECK failed" in open(os.path.join(pkg, "libspgemm_b200_checked.so"), "rb").read()
