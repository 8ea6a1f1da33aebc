"""Property-based GPU parity (hypothesis, derandomized): random CSR shapes, sparsity patterns with hub
rows and hub columns, value kinds (uniform reals, small integers, explicit zeros), and random
execution options (two-phase / fused plans, ring depth, forced chunk caps, column panels of B, the
decreasing-flops chunk order, device-resident operands with a row_ptr base, row panels with a
global base) -- every result against the CPU oracle: row_ptr and col bit-identical, values within
1e-12 * sum_k |a_ik b_kj| (bit-exact when all values are integers).  The options must never change
the result (reading R11)."""
import os

import numpy as np
import pytest

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
hyp = pytest.importorskip("hypothesis")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

from hypothesis import HealthCheck, given, settings  # noqa: E402
from hypothesis import strategies as st  # noqa: E402

from paper_conf_ipps_xia0ar21_b200 import capi  # noqa: E402


def make(rng, m, n, deg, hubs, kind):
    """m x n CSR: Poisson(deg) entries per row, `hubs` rows ~ n/3 long, a few hot columns."""
    rows = []
    hot = rng.choice(n, size=min(n, 3), replace=False) if n else np.zeros(0, int)
    for i in range(m):
        k = int(rng.poisson(deg))
        if i < hubs:
            k = max(k, n // 3)
        c = rng.choice(n, size=min(k, n), replace=False) if n and k else np.zeros(0, int)
        if n and rng.random() < 0.3:
            c = np.union1d(c, hot)
        rows.append(np.sort(c))
    rp = np.zeros(m + 1, np.int64)
    np.cumsum([len(r) for r in rows], out=rp[1:])
    col = np.concatenate(rows).astype(np.int32) if m else np.zeros(0, np.int32)
    z = int(rp[-1])
    if kind == "int":
        val = rng.integers(-3, 4, z).astype(np.float64)
    elif kind == "zeros":
        val = np.where(rng.random(z) < 0.3, 0.0, rng.uniform(-1, 1, z))
    else:
        val = rng.uniform(-1, 1, z)
    return W.CSR(m, n, rp, col, val)


def to_dev(M, base):
    d = type("D", (), {})()
    d.nrows, d.ncols = M.nrows, M.ncols
    d.row_ptr = torch.from_numpy(M.row_ptr + base).cuda()
    d.col = torch.from_numpy(np.concatenate([np.zeros(base, np.int32), M.col])).cuda()
    d.val = torch.from_numpy(np.concatenate([np.zeros(base), M.val])).cuda()
    return d


@settings(max_examples=int(os.environ.get("FUZZ_EXAMPLES", "60")), deadline=None, derandomize=True,
          suppress_health_check=[HealthCheck.too_slow, HealthCheck.data_too_large])
@given(seed=st.integers(0, 2**31 - 1), m=st.integers(0, 300), k=st.integers(1, 400), n=st.integers(1, 3000),
       deg=st.floats(0.0, 12.0), hubs=st.integers(0, 3), kind=st.sampled_from(["real", "int", "zeros"]),
       fused=st.booleans(), ring=st.integers(1, 3), chunk=st.sampled_from([0, 1, 97, 5000]),
       panels=st.sampled_from([0, 0, 2, 3]), order=st.booleans(), device=st.booleans(),
       split=st.booleans())
def test_fuzz_parity(seed, m, k, n, deg, hubs, kind, fused, ring, chunk, panels, order, device, split):
    rng = np.random.default_rng(seed)
    A = make(rng, m, k, deg, hubs, kind)
    B = make(rng, k, n, deg, hubs, kind)
    E = oracle.spgemm(A, B)
    total = int(E["row_ptr"][-1])
    # row panel [r0, r1) with a global base (a multi-GPU rank's slice) or all rows
    r0, r1 = (m // 3, m - m // 4) if split and m > 2 else (0, m)
    base = int(E["row_ptr"][r0])
    nloc = int(E["row_ptr"][r1]) - base
    kw = dict(ring=ring, chunk_nnz=chunk, col_panels=panels, row_begin=r0, row_end=r1, row_ptr_base=base,
              fused=fused and panels < 2, order=int(order and not fused and panels < 2))
    a_in = to_dev(A, 5) if device else A
    b_in = to_dev(B, 3) if device else B
    with capi.Plan(a_in, b_in, 0, capi.opts(**kw)) as P:
        rp = torch.empty(r1 - r0 + 1, dtype=torch.int64, pin_memory=True)
        col = torch.empty(max(nloc, 1), dtype=torch.int32, pin_memory=True)
        val = torch.empty(max(nloc, 1), dtype=torch.float64, pin_memory=True)
        z = P.execute_capacity(rp, col, val, nloc)
    assert z == nloc
    rows = np.arange(r0, r1)
    Es = oracle.spgemm(A, B, rows=rows) if (r0, r1) != (0, m) else E
    res = oracle.compare(rp.numpy() - base, col.numpy()[:nloc], val.numpy()[:nloc], Es)
    assert res["ok"], (res, kw, total)
    if kind == "int":
        assert np.array_equal(val.numpy()[:nloc], Es["val"])


@settings(max_examples=int(os.environ.get("FUZZ_EXAMPLES", "30")), deadline=None, derandomize=True,
          suppress_health_check=[HealthCheck.too_slow, HealthCheck.data_too_large,
                                 HealthCheck.function_scoped_fixture])
@given(seed=st.integers(0, 2**31 - 1), m=st.integers(1, 3000), deg=st.floats(0.0, 9.0), hubs=st.integers(0, 2),
       kind=st.sampled_from(["real", "int", "zeros"]), ring=st.integers(1, 3),
       chunk=st.sampled_from([0, 1, 97, 5000]), piece=st.sampled_from([1, 50, 999, 0]), split=st.booleans(),
       host_cut=st.booleans())
def test_fuzz_square_host_operands(seed, m, deg, hubs, kind, ring, chunk, piece, split, host_cut, monkeypatch):
    """C = A*A with the same host arrays for A and B (fused): the host-cut plan (chunks cut from
    A.row_ptr, count per chunk in execute, interleaved operand pieces of SPGEMM_PIECE_NNZ entries)
    whenever ncols <= 4096 or the rows are short, else the counted plan; both against the oracle."""
    rng = np.random.default_rng(seed)
    A = make(rng, m, m, deg, hubs, kind)
    monkeypatch.setenv("SPGEMM_NO_HOST_CUT", "0" if host_cut else "1")
    if piece:
        monkeypatch.setenv("SPGEMM_PIECE_NNZ", str(piece))
    else:
        monkeypatch.delenv("SPGEMM_PIECE_NNZ", raising=False)
    E = oracle.spgemm(A, A)
    r0, r1 = (m // 3, m - m // 4) if split and m > 2 else (0, m)
    base = int(E["row_ptr"][r0])
    nloc = int(E["row_ptr"][r1]) - base
    kw = dict(ring=ring, chunk_nnz=chunk, row_begin=r0, row_end=r1, row_ptr_base=base, fused=True)
    with capi.Plan(A, A, 0, capi.opts(**kw)) as P:
        rp = torch.empty(r1 - r0 + 1, dtype=torch.int64, pin_memory=True)
        col = torch.empty(max(nloc, 1), dtype=torch.int32, pin_memory=True)
        val = torch.empty(max(nloc, 1), dtype=torch.float64, pin_memory=True)
        z = P.execute_capacity(rp, col, val, nloc)
        info = P.info()
    assert z == nloc
    u = oracle.products(A, A)
    assert info["products"] == int(u[r0:r1].sum())
    Es = oracle.spgemm(A, A, rows=np.arange(r0, r1)) if (r0, r1) != (0, m) else E
    res = oracle.compare(rp.numpy() - base, col.numpy()[:nloc], val.numpy()[:nloc], Es)
    assert res["ok"], (res, kw)
    if kind == "int":
        assert np.array_equal(val.numpy()[:nloc], Es["val"])
