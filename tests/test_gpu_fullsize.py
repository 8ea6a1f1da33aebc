"""Full-size parity at BASELINE.json's sizes, in the launch configuration bench.py times.

C2 (configs[1]): 3-D 27-point 128^3, device budget 2 GiB, fused plan, ring 2 -- the bench
workload.  Every row_ptr entry is checked against the closed form (nnz per row = product of
per-axis widths), every column and value of a contiguous block of rows and of sampled rows against
the closed form A^2 = 729 I - 54 S + K^2 (x) K^2 (x) K^2 and against the oracle, and sum(C) against
its closed form.  C3 (configs[2], R-MAT s22) streams its ~0.3 TB of C through the sink and every
row is checked against the oracle as it arrives (oracle.verify); likewise every row of the C4 / C5
row panels one rank of an 8-GPU deal owns.
"""
import os

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


class _Dev:
    pass


def _device_csr(M, dev):
    d = _Dev()
    d.nrows, d.ncols = M.nrows, M.ncols
    d.row_ptr = torch.from_numpy(M.row_ptr).to(dev)
    d.col = torch.from_numpy(M.col).to(dev)
    d.val = torch.from_numpy(M.val).to(dev)
    return d


def test_c2_full_size_budget_2gib():
    n = 128
    A = W.stencil_3d27(n)
    dev = torch.device("cuda", 0)
    dA = _device_csr(A, dev)
    in_bytes = 8 * (A.nrows + 1) + 12 * A.nnz
    ws = torch.empty((2 << 30) - in_bytes, dtype=torch.uint8, device=dev)   # operands + arena = 2 GiB
    p_tot, z_tot = CF.c2_totals(n)
    rp = torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True)
    col = torch.empty(z_tot, dtype=torch.int32, pin_memory=True)
    val = torch.empty(z_tot, dtype=torch.float64, pin_memory=True)
    o = capi.opts(workspace=ws, stream=torch.cuda.current_stream().cuda_stream, fused=True, ring=2)
    with capi.Plan(dA, dA, ws.numel(), o) as P:
        nnz = P.execute_capacity(rp, col, val, z_tot)
        info = P.info()
    assert nnz == z_tot and info["products"] == p_tot and info["num_chunks"] > 8
    assert info["arena_used"] <= ws.numel()
    rp, col, val = rp.numpy(), col.numpy(), val.numpy()
    rows = np.arange(A.nrows, dtype=np.int64)
    assert rp[0] == 0 and np.array_equal(np.diff(rp), CF.c2_row_nnz(n, rows))     # every row_ptr entry
    assert float(val.sum()) == CF.c2_sum(n)
    # a contiguous block spanning chunk boundaries + random rows, entrywise vs the closed form
    rng = np.random.default_rng(2)
    blocks = [np.arange(0, 40000), np.arange(A.nrows // 2 - 20000, A.nrows // 2 + 20000),
              np.arange(A.nrows - 40000, A.nrows), rng.integers(0, A.nrows, 5000)]
    for rs in blocks:
        idx = np.concatenate([np.arange(rp[r], rp[r + 1]) for r in rs])
        i = np.repeat(rs, rp[rs + 1] - rp[rs])
        c = col[idx].astype(np.int64)
        assert np.all(np.diff(c)[np.diff(i) == 0] > 0)  # sorted, unique per row
        # column sets: Chebyshev distance <= 2 (the count per row is already exact above)
        xi, yi, zi = i % n, (i // n) % n, i // (n * n)
        xc, yc, zc = c % n, (c // n) % n, c // (n * n)
        assert np.all(np.maximum(np.maximum(np.abs(xi - xc), np.abs(yi - yc)), np.abs(zi - zc)) <= 2)
        for r in rs[:100]:
            assert np.array_equal(col[rp[r]:rp[r + 1]], CF.c2_row_cols(n, r))
        assert np.array_equal(val[idx], CF.c2_entry(n, i, c))
    # and sampled rows against the oracle
    sel = rng.integers(0, A.nrows, 300)
    E = oracle.spgemm(A, A, rows=sel)
    gp = np.concatenate([[0], np.cumsum(rp[sel + 1] - rp[sel])])
    idx = np.concatenate([np.arange(rp[r], rp[r + 1]) for r in sel])
    assert oracle.compare(gp, col[idx], val[idx], E)["ok"]


def _streamed_verify(A, B, r0, r1, chunk_nnz=400_000_000):
    """Stream rows [r0, r1) of C = A*B through the sink (fused plan, ring 3, device operands) and
    check EVERY row of every output chunk against the oracle while it is delivered (oracle.verify:
    Alg. 1 per row on all host cores, structure bit-exact, values within the bound; nothing of C
    is stored).  Also checks the plan's per-row bounds against the oracle's product counts."""
    dev = torch.device("cuda", 0)
    dA = _device_csr(A, dev)
    dB = dA if B is A else _device_csr(B, dev)
    ops = oracle.Operands(A, B)
    tot = {"rows": 0, "entries": 0, "products": 0, "chunks": 0, "worst_ratio": 0.0, "bad": []}

    def sink(ra, rb, rp, col, val):
        res = oracle.verify(A, B, ra, rp, col, val, ops=ops)
        tot["chunks"] += 1
        for k in ("rows", "entries", "products"):
            tot[k] += res[k]
        tot["worst_ratio"] = max(tot["worst_ratio"], res["worst_ratio"])
        if not res["ok"]:
            tot["bad"].append((ra, rb, res["first_bad_row"], res["first_bad_kind"]))

    o = capi.opts(fused=True, ring=3, chunk_nnz=chunk_nnz, row_begin=r0, row_end=r1)
    with capi.Plan(dA, dB, 0, o) as P:
        bnd = P.row_bounds()
        P.execute_stream(sink)
        info = P.info()
    assert not tot["bad"], tot["bad"][:5]
    assert tot["rows"] == r1 - r0 and tot["entries"] == info["nnz"] and tot["products"] == info["products"]
    assert tot["chunks"] == info["num_copies"]
    u = oracle.products(A, B, rows=np.arange(r0, r1))
    assert np.array_equal(bnd, np.minimum(u, B.ncols)) and int(u.sum()) == info["products"]
    print(f"rows {r0}..{r1}: {tot['rows']} rows, {tot['entries']} entries, {tot['products']} products checked "
          f"in {tot['chunks']} chunks, worst |c - ref| / tol = {tot['worst_ratio']:.3g}")
    return info, tot


@pytest.mark.skipif(os.environ.get("SPGEMM_SKIP_C45") == "1", reason="C4/C5 panel runs disabled")
def test_c4_rmat_s24_rank_panel():
    """configs[3] (R-MAT s24 ef16, C several TB): EVERY row of the row panel one rank of an 8-GPU
    deal owns (1/8 of the rows, ~2e11 bytes of C), checked against the oracle."""
    A = W.rmat_torch(24, 16, seed=20210518)
    info, tot = _streamed_verify(A, A, 0, A.nrows // 8)
    assert info["rows_block"] + info["rows_global"] > 0


@pytest.mark.skipif(os.environ.get("SPGEMM_SKIP_C45") == "1", reason="C4/C5 panel runs disabled")
def test_c5_rectangular_rank_panel():
    """configs[4]: A = 2^24 x 2^22 power-law, B = 2^22 x 2^24 (2^28 generated edges each): every row
    of rank 0's panel and of the LAST rank's panel of an 8-GPU deal (the two ends of the skew)."""
    A = W.rmat_torch(24, col_scale=22, nedges=1 << 28, seed=11, symmetric=False)
    B = W.rmat_torch(22, col_scale=24, nedges=1 << 28, seed=12, symmetric=False)
    assert A.nnz + B.nnz > 4e8
    _streamed_verify(A, B, 0, A.nrows // 8)
    _streamed_verify(A, B, A.nrows - A.nrows // 8, A.nrows)


@pytest.mark.skipif(os.environ.get("SPGEMM_SKIP_C3") == "1", reason="C3 full-size run disabled")
def test_c3_rmat_s22_streamed():
    """configs[2] at full size: ~2.9e10 products, C of ~0.3 TB streamed through the sink; EVERY row
    of C is compared with the oracle as its chunk arrives."""
    A = W.rmat(22, 16)
    info, tot = _streamed_verify(A, A, 0, A.nrows)
    assert tot["rows"] == A.nrows == 1 << 22
    assert info["rows_global"] + info["rows_block"] > 0  # the skewed tiers were exercised
