"""GPU parity of the column-panel mode (B cut into column panels: Alg. 3 line 4, §III-D
of PAPER.md; DESIGN.md §2 row (f) NEXT-1) against the CPU oracle, through the C ABI.

Same bar as tests/test_gpu_parity.py: row_ptr and col_idx bit-identical, values within
1e-12 * sum_k |a_ik b_kj|, bit-exact on the integer-valued stencils.  The panel count, the
budget, the ring and the operand residency must not change the result (reading R11).
"""
import numpy as np
import pytest

import oracle
import workloads as W
from tests import closed_forms as CF

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_ipps_xia0ar21_b200 import capi  # noqa: E402


def run(A, B, budget=0, pinned=True, **kw):
    with capi.Plan(A, B, budget, capi.opts(**kw)) as P:
        info = P.info()
        if pinned:
            rp = torch.empty(info["nrows"] + 1, dtype=torch.int64, pin_memory=True)
            col = torch.empty(info["nnz"], dtype=torch.int32, pin_memory=True)
            val = torch.empty(info["nnz"], dtype=torch.float64, pin_memory=True)
            P.execute_into(rp, col, val)
            return rp.numpy(), col.numpy(), val.numpy(), info
        rp = np.empty(info["nrows"] + 1, np.int64)
        col = np.empty(info["nnz"], np.int32)
        val = np.empty(info["nnz"], np.float64)
        P.execute_into(rp, col, val)
        return rp, col, val, info


def check(A, B, r, exact=False, base=0):
    E = oracle.spgemm(A, B)
    res = oracle.compare(r[0], r[1], r[2], E, rows_offset=base) if base else oracle.compare(r[0], r[1], r[2], E)
    assert res["ok"], res
    if exact:
        assert np.array_equal(r[2], E["val"])


@pytest.mark.parametrize("panels", [2, 3, 7])
def test_stencil_forced_panels_bit_exact(panels):
    A = W.stencil_3d27(24)
    r = run(A, A, col_panels=panels)
    assert r[3]["col_panels"] == panels
    p, z = CF.c2_totals(24)
    assert r[3]["nnz"] == z and r[3]["products"] == p
    check(A, A, r, exact=True)


@pytest.mark.parametrize("panels", [2, 5])
def test_rmat_forced_panels(panels):
    """Skewed rows (CTA tier) split across panels; products sum over the panels."""
    A = W.rmat(13, 16, seed=11)
    r = run(A, A, col_panels=panels)
    assert r[3]["products"] == int(oracle.products(A, A).sum())
    check(A, A, r)


def test_long_rows_dense_and_pieced_tiers_in_panels():
    """Rows long enough for the pieced CTA tier and the dense tier inside a panel."""
    rng = np.random.default_rng(5)
    ncols = 400_000
    brows = [np.sort(rng.choice(ncols, 1500, replace=False)) for _ in range(400)]
    brows += [np.sort(rng.choice(ncols, 3, replace=False)) for _ in range(2000)]
    rp = np.zeros(len(brows) + 1, np.int64)
    np.cumsum([len(b) for b in brows], out=rp[1:])
    B = W.CSR(len(brows), ncols, rp, np.concatenate(brows).astype(np.int32), rng.uniform(-1, 1, rp[-1]))
    arows = [np.arange(0, 400), np.arange(0, 60), np.sort(rng.choice(2400, 30, replace=False)), np.array([], int)]
    ap = np.zeros(len(arows) + 1, np.int64)
    np.cumsum([len(a) for a in arows], out=ap[1:])
    A = W.CSR(len(arows), B.nrows, ap, np.concatenate(arows).astype(np.int32), rng.uniform(-1, 1, ap[-1]))
    for panels in (2, 3):
        r = run(A, B, col_panels=panels)
        check(A, B, r)


def test_auto_fallback_when_b_exceeds_budget():
    """Host A = B (C = A*A) larger than the budget: the plan retries with column panels."""
    A = W.stencil_3d27(40)            # 64,000 rows, 1.6M nnz: ~19.7 MB of CSR
    budget = 16 << 20                  # < B's bytes: the in-core plan cannot hold B
    with pytest.raises(capi.SpgemmError) as e:
        capi.Plan(A, A, budget, capi.opts(col_panels=1))
    assert e.value.status == capi.ERR_BUDGET
    r = run(A, A, budget=budget)
    assert r[3]["col_panels"] >= 2 and r[3]["arena_used"] <= budget
    check(A, A, r, exact=True)


def test_rectangular_device_operands_and_row_panels():
    """A on the device with a row_ptr base, B on the host; row panels with a global base."""
    A = W.rmat_rect(11, 10, 30_000, seed=3)
    B = W.rmat_rect(10, 12, 20_000, seed=4)
    full = run(A, B, col_panels=3)
    check(A, B, full)
    E = oracle.spgemm(A, B)
    dA = type("D", (), {})()
    dA.nrows, dA.ncols = A.nrows, A.ncols
    dA.row_ptr = torch.from_numpy(A.row_ptr + 9).cuda()
    dA.col = torch.from_numpy(np.concatenate([np.zeros(9, np.int32), A.col])).cuda()
    dA.val = torch.from_numpy(np.concatenate([np.zeros(9), A.val])).cuda()
    cuts = [0, 500, 501, A.nrows]
    for r0, r1 in zip(cuts[:-1], cuts[1:]):
        base = int(E["row_ptr"][r0])
        prp, pcol, pval, info = run(dA, B, col_panels=2, row_begin=r0, row_end=r1, row_ptr_base=base)
        assert prp[0] == base
        res = oracle.compare(prp, pcol, pval, oracle.spgemm(A, B, rows=np.arange(r0, r1)), rows_offset=base)
        assert res["ok"], res


def test_panel_invariance_ring_chunks_pageable():
    """Any panel count, ring, chunk cap, or pageable (registered on the fly) output: same C."""
    A = W.random_csr_sparse(3000, 2000, 7.0, seed=12)
    B = W.random_csr_sparse(2000, 5000, 9.0, seed=13)
    for kw in ({"col_panels": 1}, {"col_panels": 2}, {"col_panels": 4, "ring": 1},
               {"col_panels": 3, "chunk_nnz": 3000, "ring": 3}, {"col_panels": 6, "pinned": False}):
        check(A, B, run(A, B, **kw))


def test_degenerate_and_empty_panels():
    """Panels that hold no column of B, empty rows, an empty product."""
    A = W.random_csr(50, 40, 0.1, seed=1, empty_rows=0.3)
    B = W.random_csr(40, 30, 0.1, seed=2, empty_rows=0.3)
    r = run(A, B, col_panels=9)
    check(A, B, r)
    Z = W.random_csr(40, 30, 0.0, seed=3)
    r = run(A, Z, col_panels=2)
    assert r[3]["nnz"] == 0 and np.all(r[0] == 0)


def test_repeat_multiply_and_errors():
    A = W.stencil_3d27(12)
    with capi.Plan(A, A, 0, capi.opts(col_panels=3)) as P:
        info = P.info()
        outs = []
        for _ in range(2):
            rp = torch.empty(info["nrows"] + 1, dtype=torch.int64, pin_memory=True)
            col = torch.empty(info["nnz"], dtype=torch.int32, pin_memory=True)
            val = torch.empty(info["nnz"], dtype=torch.float64, pin_memory=True)
            P.execute_into(rp, col, val)
            outs.append((rp.numpy(), col.numpy(), val.numpy()))
        for o in outs:
            check(A, A, o, exact=True)
        with pytest.raises(capi.SpgemmError) as e:
            P.execute_stream(lambda *a: 0)
        assert e.value.status == capi.ERR_INVALID_ARGUMENT
        with pytest.raises(capi.SpgemmError):
            P.chunks()
    # the one-shot API (fused is ignored in column-panel mode)
    n = CF.c2_totals(12)[1]
    out = [torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True),
           torch.empty(n, dtype=torch.int32, pin_memory=True), torch.empty(n, dtype=torch.float64, pin_memory=True)]
    z = capi.spgemm_multiply(A, A, 0, capi.opts(col_panels=2), *out, capacity=n)
    assert z == n
    check(A, A, (out[0].numpy(), out[1].numpy(), out[2].numpy()), exact=True)


def test_c2_full_size_budget_below_b():
    """BASELINE config 1 at full size (128^3, C = 3.07 GB) with host operands and a device budget
    of 256 MiB, well below B's 686 MB: the plan falls back to column panels.  Every row's nnz by
    closed form, the sum of C, and 200 sampled rows against the oracle (bit-exact)."""
    n = 128
    A = W.stencil_3d27(n)
    p, z = CF.c2_totals(n)
    budget = 256 << 20
    ws = torch.empty(budget, dtype=torch.uint8, device="cuda")
    hA = W.CSR(A.nrows, A.ncols, torch.from_numpy(A.row_ptr).pin_memory(), torch.from_numpy(A.col).pin_memory(),
               torch.from_numpy(A.val).pin_memory())
    with capi.Plan(hA, hA, budget, capi.opts(workspace=ws)) as P:
        info = P.info()
        assert info["col_panels"] >= 2 and info["nnz"] == z and info["products"] == p
        assert info["arena_used"] <= budget
        rp = torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True)
        col = torch.empty(z, dtype=torch.int32, pin_memory=True)
        val = torch.empty(z, dtype=torch.float64, pin_memory=True)
        P.execute_into(rp, col, val)
    rp, col, val = rp.numpy(), col.numpy(), val.numpy()
    assert np.array_equal(np.diff(rp), CF.c2_row_nnz(n, np.arange(A.nrows)))
    assert float(val.sum()) == CF.c2_sum(n)
    rng = np.random.default_rng(8)
    rows = np.unique(np.concatenate([[0, A.nrows - 1], rng.integers(0, A.nrows, 200)]))
    E = oracle.spgemm(A, A, rows=rows)
    gp = np.concatenate([[0], np.cumsum(rp[rows + 1] - rp[rows])])
    idx = np.concatenate([np.arange(rp[r], rp[r + 1]) for r in rows])
    res = oracle.compare(gp, col[idx], val[idx], E)
    assert res["ok"], res
    assert np.array_equal(val[idx], E["val"])
