"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

Bar: row_ptr and col_idx bit-identical; every value within
|c - ref| <= 1e-12 * sum_k |a_ik b_kj| (BASELINE.json north_star), exact (bit-equal) on
the integer-valued stencil configs.  All inputs come from `workloads` (seeded).
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

import paper_conf_ipps_xia0ar21_b200 as spg  # noqa: E402
from paper_conf_ipps_xia0ar21_b200 import capi  # noqa: E402


def run(A, B, budget=0, **kw):
    """plan + execute_into pinned torch buffers; returns (rp, col, val, info, chunks)."""
    o = capi.opts(**kw)
    with capi.Plan(A, B, budget, o) as P:
        info = P.info()
        rp = torch.empty(info["nrows"] + 1, dtype=torch.int64, pin_memory=True)
        col = torch.empty(info["nnz"], dtype=torch.int32, pin_memory=True)
        val = torch.empty(info["nnz"], dtype=torch.float64, pin_memory=True)
        P.execute_into(rp, col, val)
        chunks = P.chunks()
    return rp.numpy(), col.numpy(), val.numpy(), info, chunks


def assert_parity(A, B, rp, col, val, rows=None, exact=False, base=0):
    E = oracle.spgemm(A, B, rows=rows)
    if rows is None:
        res = oracle.compare(rp, col, val, E, rows_offset=base)
    else:
        # gather the selected rows out of the full GPU result
        rs = np.asarray(rows)
        n = rp[rs + 1] - rp[rs]
        gp = np.zeros(len(rs) + 1, dtype=np.int64)
        np.cumsum(n, out=gp[1:])
        idx = np.concatenate([np.arange(rp[r] - base, rp[r + 1] - base) for r in rs]) if len(rs) else np.zeros(0, int)
        res = oracle.compare(gp, col[idx], val[idx], E)
    assert res["ok"], res
    if exact:
        assert np.array_equal(val if rows is None else val[idx], E["val"])
    return res


# ------------------------------------------------------------------------------------- paper pins

def test_fig2_example():
    A, B = W.fig2_instance()
    rp, col, val, info, _ = run(A, B)
    assert list(rp) == [0, 2] and list(col) == [0, 3] and list(val) == [43.0, 14.0]
    assert info["products"] == 3


def test_c1_full_bit_exact():
    """BASELINE config 0 in full, in-core: values are small integers -> bit-exact in any order."""
    A = W.stencil_2d5(64)
    rp, col, val, info, _ = run(A, A)
    assert info["products"] == 100104 and info["nnz"] == 51972
    assert_parity(A, A, rp, col, val, exact=True)
    i = np.repeat(np.arange(A.nrows), np.diff(rp))
    assert np.array_equal(val, CF.c1_entry(64, i, col.astype(np.int64)))
    assert val.sum() == 264.0


@pytest.mark.parametrize("n", [8, 24, 40])
def test_c2_small_bit_exact(n):
    A = W.stencil_3d27(n)
    rp, col, val, info, _ = run(A, A)
    p, z = CF.c2_totals(n)
    assert info["products"] == p and info["nnz"] == z
    assert_parity(A, A, rp, col, val, exact=True)
    assert val.sum() == CF.c2_sum(n)


# ------------------------------------------------------------------------------------- random

@pytest.mark.parametrize("seed", range(8))
def test_random_rectangular(seed):
    rng = np.random.default_rng(seed)
    m, k, n = (int(x) for x in rng.integers(1, 3000, size=3))
    A = W.random_csr_sparse(m, k, float(rng.uniform(0.5, 12)), seed=seed)
    B = W.random_csr_sparse(k, n, float(rng.uniform(0.5, 12)), seed=seed + 1000)
    rp, col, val, info, _ = run(A, B, validate=True)
    assert_parity(A, B, rp, col, val)


@pytest.mark.parametrize("shape", [(0, 5, 7), (5, 0, 7), (6, 5, 0), (1, 1, 1), (3, 4, 5)])
def test_degenerate(shape):
    m, k, n = shape
    A = W.random_csr(m, k, 0.6, seed=1, empty_rows=0.3)
    B = W.random_csr(k, n, 0.6, seed=2, empty_rows=0.3)
    rp, col, val, info, _ = run(A, B)
    assert_parity(A, B, rp, col, val)


def test_empty_b_rows_and_explicit_zeros():
    A = W.random_csr_sparse(500, 400, 6.0, seed=3)
    B = W.random_csr_sparse(400, 450, 6.0, seed=4)
    # blank every third row of B, zero some values (structure must stay)
    keep = np.ones(B.nnz, bool)
    for r in range(0, B.nrows, 3):
        keep[B.row_ptr[r]:B.row_ptr[r + 1]] = False
    cnt = np.add.reduceat(keep.astype(np.int64), B.row_ptr[:-1]) * (np.diff(B.row_ptr) > 0)
    rp = np.zeros(B.nrows + 1, np.int64)
    np.cumsum(cnt, out=rp[1:])
    B = W.CSR(B.nrows, B.ncols, rp, B.col[keep], B.val[keep].copy())
    B.val[::5] = 0.0
    A.val[::7] = 0.0
    r, c, v, info, _ = run(A, B)
    assert_parity(A, B, r, c, v)


# ------------------------------------------------------------------------------------- tiers

def _long_rows_case(seed=0, wide=60000, deg=240):
    """A few rows whose products/nnz exceed the warp tier and one CTA-tier piece."""
    rng = np.random.default_rng(seed)
    k = 800
    B = W.random_csr_sparse(k, wide, deg, seed=seed + 1)
    rows = []
    for i in range(300):
        if i % 100 == 0:
            d = 300            # ~300 * 240 = 72k products over 60k columns -> pieced CTA tier
        elif i % 10 == 0:
            d = 12             # ~2.9k products -> B tier
        else:
            d = int(rng.integers(0, 3))
        rows.append(np.sort(rng.choice(k, size=d, replace=False)))
    rp = np.zeros(301, np.int64)
    np.cumsum([len(r) for r in rows], out=rp[1:])
    col = np.concatenate(rows).astype(np.int32)
    A = W.CSR(300, k, rp, col, rng.uniform(-1, 1, len(col)))
    return A, B


def test_tiers_warp_block_pieced():
    """Warp rows, one-piece CTA rows and (72k products over 60k columns) pieced CTA rows."""
    A, B = _long_rows_case()
    rp, col, val, info, _ = run(A, B)
    assert info["rows_block"] > 0 and info["rows_warp"] > 0, info
    assert_parity(A, B, rp, col, val)


@pytest.mark.parametrize("fused", [False, True])
@pytest.mark.parametrize("medium", [True, False])
def test_medium_tier(fused, medium, monkeypatch):
    """Rows of a few hundred to two thousand products (the R-MAT bulk) go to the 128-thread medium
    CTA tier; SPGEMM_NO_MEDIUM=1 sends them to the 512-thread tier instead.  Same C either way."""
    if not medium:
        monkeypatch.setenv("SPGEMM_NO_MEDIUM", "1")
    rng = np.random.default_rng(31)
    ncols = 200_000
    brows = [np.sort(rng.choice(ncols, int(rng.integers(5, 60)), replace=False)) for _ in range(4000)]
    B = _csr_from_rows(brows, ncols, rng)
    arows = []
    for i in range(1500):
        d = [3, 12, 25, 40, 70][i % 5]          # ~100 .. 2300 products per row
        arows.append(np.sort(rng.choice(B.nrows, d, replace=False)))
    arows[7] = np.sort(rng.choice(200, 60, replace=False))   # clustered columns (overlapping B rows)
    A = _csr_from_rows(arows, B.nrows, rng)
    r = run_fused(A, B) if fused else run(A, B)
    info = r[3]
    if medium:
        assert info["rows_medium"] > 300, info
    else:
        assert info["rows_medium"] == 0 and info["rows_block"] > 300, info
    assert_parity(A, B, r[0], r[1], r[2])


def _csr_from_rows(rows, ncols, rng):
    rp = np.zeros(len(rows) + 1, np.int64)
    np.cumsum([len(r) for r in rows], out=rp[1:])
    col = np.concatenate(rows).astype(np.int32) if rows else np.zeros(0, np.int32)
    return W.CSR(len(rows), ncols, rp, col, rng.uniform(-1, 1, len(col)))


@pytest.mark.parametrize("fused", [False, True])
def test_pieced_cta_tier_and_dense_tier(fused):
    """Long rows: a clustered row (its column pieces overflow the CTA table and are halved until
    they fit), a scattered row (plain column pieces), and a row beyond the pieced tier (dense)."""
    rng = np.random.default_rng(17)
    ncols = 1_000_000
    brows = []
    for k in range(30):                      # clustered in [0, 50000) + one far outlier
        brows.append(np.append(np.sort(rng.choice(50_000, 1000, replace=False)), ncols - 1))
    for k in range(40):                      # scattered
        brows.append(np.sort(rng.choice(ncols, 1000, replace=False)))
    for k in range(600):                     # long scattered rows for the dense tier
        brows.append(np.sort(rng.choice(ncols, 1500, replace=False)))
    B = _csr_from_rows(brows, ncols, rng)
    arows = [np.arange(0, 30), np.arange(30, 70), np.arange(70, 670), np.array([3, 40, 100])]
    A = _csr_from_rows(arows, B.nrows, rng)
    r = run_fused(A, B) if fused else run(A, B)
    info = r[3]
    assert info["rows_global"] >= 1 and info["rows_block"] >= 2, info
    assert_parity(A, B, r[0], r[1], r[2])


@pytest.mark.parametrize("slots", [None, "2"])
@pytest.mark.parametrize("fused", [False, True])
def test_dense_tier_split_rows(fused, slots, monkeypatch):
    """Rows beyond the pieced CTA tier (> 32 pieces: the C3 hubs) are shared by several CTAs per
    row and swept in column ranges; with only 2 dense slots (test hook) the rows beyond the
    slots take the one-CTA-per-row kernels.  Rows of different lengths, an empty row between."""
    if slots:
        monkeypatch.setenv("SPGEMM_MAX_GSLOTS", slots)
    rng = np.random.default_rng(41)
    ncols = 600_000
    brows = [np.sort(rng.choice(ncols, int(rng.integers(200, 900), ), replace=False)) for _ in range(3000)]
    B = _csr_from_rows(brows, ncols, rng)
    arows = []
    for i in range(9):
        d = [600, 700, 0, 1000, 650, 3, 800, 720, 850][i]   # ~330K-550K products per row
        arows.append(np.sort(rng.choice(B.nrows, d, replace=False)))
    A = _csr_from_rows(arows, B.nrows, rng)
    r = run_fused(A, B) if fused else run(A, B)
    assert r[3]["rows_global"] >= 6, r[3]
    assert_parity(A, B, r[0], r[1], r[2])


@pytest.mark.parametrize("fused", [False, True])
def test_pieced_rows_many_entries_and_dense_fallback(fused):
    """Pieced rows whose A rows hold many entries (cursor scratch per entry), one A row longer than
    the cursor scratch (CURSOR_MAX = 32768 entries: the dense tier takes it), empty B rows among
    the entries, and pieces whose column ranges hold no product at all."""
    rng = np.random.default_rng(23)
    ncols = 3_000_000
    brows = [np.sort(rng.choice(ncols, int(rng.integers(0, 4)), replace=False)) for _ in range(50_000)]
    brows += [np.sort(rng.choice(ncols, 400, replace=False)) for _ in range(100)]
    B = _csr_from_rows(brows, ncols, rng)
    arows = [np.sort(rng.choice(50_000, 12_000, replace=False)),            # ~18k products, pieced
             np.arange(50_000, 50_100),                                    # 40k products, pieced
             np.sort(rng.choice(50_000, 40_000, replace=False)),           # > CURSOR_MAX entries
             np.array([0, 1, 2]), np.array([], dtype=np.int64)]
    A = _csr_from_rows(arows, B.nrows, rng)
    r = run_fused(A, B) if fused else run(A, B)
    assert_parity(A, B, r[0], r[1], r[2])


@pytest.mark.parametrize("fused", [False, True])
def test_wide_column_space(fused):
    """ncols > 2^23: the numeric sort switches to 64-bit packed keys (column << 9 | slot)."""
    n = (1 << 23) + 4099
    B = W.random_csr_sparse(300, n, 40.0, seed=31)
    B.col[-3:] = [n - 3, n - 2, n - 1]  # touch the top of the column range (rows stay sorted)
    B.col = np.ascontiguousarray(B.col)
    last = B.nrows - 1
    seg = np.sort(np.unique(B.col[B.row_ptr[last]:B.row_ptr[last + 1]]))
    assert len(seg) == B.row_ptr[last + 1] - B.row_ptr[last]
    A = W.random_csr_sparse(500, 300, 6.0, seed=32)
    r = run_fused(A, B) if fused else run(A, B)
    assert_parity(A, B, r[0], r[1], r[2])


def test_rmat_skewed():
    A = W.rmat(14, 16, seed=5)
    rp, col, val, info, _ = run(A, A)
    assert_parity(A, A, rp, col, val)
    assert info["products"] == int(oracle.products(A, A).sum())


# ------------------------------------------------------------------------------------- out-of-core

def test_forced_chunking_invariance():
    """Any chunking, ring 1 (synchronous) or 2/3: every run equals the oracle, bit for bit on this
    integer-valued stencil (S8-S10 must not change the result; P:L122 chunk independence)."""
    A = W.stencil_3d27(20)
    E = oracle.spgemm(A, A)
    for kw in ({}, {"chunk_nnz": 5000}, {"chunk_nnz": 5000, "ring": 1}, {"chunk_nnz": 777, "ring": 3},
               {"min_chunks": 17}):
        rp, col, val, info, chunks = run(A, A, **kw)
        assert kw == {} or info["num_chunks"] > 2
        assert oracle.compare(rp, col, val, E)["ok"] and np.array_equal(val, E["val"])
        rows, offs = chunks
        assert rows[0] == 0 and rows[-1] == A.nrows and np.all(np.diff(offs) <= info["chunk_capacity"])


def test_budget_forces_chunks_and_fits():
    A = W.stencil_3d27(32)
    nnzC = CF.c2_totals(32)[1]
    budget = 24 << 20   # 24 MiB: A (~9 MB) + row arrays + ring << 12 * nnz(C) (~25 MB)
    rp, col, val, info, _ = run(A, A, budget=budget)
    assert info["nnz"] == nnzC and info["num_chunks"] >= 2 and info["arena_used"] <= budget
    assert_parity(A, A, rp, col, val, exact=True)


def test_one_row_per_chunk():
    A = W.random_csr_sparse(60, 50, 4.0, seed=9)
    B = W.random_csr_sparse(50, 70, 4.0, seed=10)
    rp, col, val, info, chunks = run(A, B, chunk_nnz=1)
    assert info["num_chunks"] >= 40
    assert_parity(A, B, rp, col, val)


def test_execute_stream_sink_matches():
    A = W.rmat(12, 16, seed=2)
    got_rp, got_col, got_val = [0], [], []
    with capi.Plan(A, A, 0, capi.opts(chunk_nnz=20000, ring=2)) as P:
        seen = []

        def sink(r0, r1, rp, col, val):
            seen.append((r0, r1))
            got_rp.extend((rp[1:] + got_rp[-1]).tolist())
            got_col.append(col.copy())
            got_val.append(val.copy())

        P.execute_stream(sink)
        assert len(seen) == P.info()["num_copies"] and seen[0][0] == 0 and seen[-1][1] == A.nrows
    assert all(a[1] == b[0] for a, b in zip(seen, seen[1:]))  # consecutive row ranges, in order
    # values: fp64 atomics make the summation order (not the bound) run-dependent (R10)
    assert_parity(A, A, np.array(got_rp), np.concatenate(got_col), np.concatenate(got_val))


@pytest.mark.parametrize("fused", [False, True])
def test_repeat_execute_same_plan(fused):
    """Every execution of one plan equals the oracle, and the plan's info does not drift between
    executions (per-tier row counts are per execution)."""
    A = W.stencil_3d27(16)
    E = oracle.spgemm(A, A)
    z = len(E["col"])
    infos = []
    with capi.Plan(A, A, 0, capi.opts(chunk_nnz=3000, fused=fused)) as P:
        for _ in range(3):
            if fused:
                rp = torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True)
                col = torch.empty(z, dtype=torch.int32, pin_memory=True)
                val = torch.empty(z, dtype=torch.float64, pin_memory=True)
                assert P.execute_capacity(rp, col, val, z) == z
                got = (rp.numpy(), col.numpy(), val.numpy())
            else:
                got = [x.copy() for x in P.execute()]
            assert oracle.compare(*got, E)["ok"] and np.array_equal(got[2], E["val"])
            infos.append(P.info())
    for k in ("nnz", "products", "rows_warp", "rows_medium", "rows_block", "rows_global", "max_row_nnz"):
        assert infos[0][k] == infos[1][k] == infos[2][k], k
    i0 = infos[0]
    assert i0["rows_warp"] + i0["rows_medium"] + i0["rows_block"] + i0["rows_global"] <= A.nrows


# ------------------------------------------------------------------------------------- device inputs

def _to_dev(M, base=0):
    class D:
        pass
    d = D()
    d.nrows, d.ncols = M.nrows, M.ncols
    pad = np.zeros(base, np.int32)
    d.row_ptr = torch.from_numpy(M.row_ptr + base).cuda()
    d.col = torch.from_numpy(np.concatenate([pad, M.col])).cuda()
    d.val = torch.from_numpy(np.concatenate([pad.astype(np.float64), M.val])).cuda()
    return d


def test_device_inputs_with_base_and_row_panels():
    """Device-resident operands (e.g. B after an NCCL broadcast), arbitrary row_ptr base, and a
    row panel [row_begin, row_end) with a global row_ptr base: the union of panels == whole."""
    A = W.rmat(12, 8, seed=7)
    B = W.random_csr_sparse(A.ncols, 3000, 5.0, seed=8)
    E = oracle.spgemm(A, B)
    dA, dB = _to_dev(A, base=13), _to_dev(B, base=5)
    rp, col, val, _, _ = run(dA, dB, stream=torch.cuda.current_stream().cuda_stream)
    assert oracle.compare(rp, col, val, E)["ok"]
    cuts = [0, 700, 701, 2500, A.nrows]
    for r0, r1 in zip(cuts[:-1], cuts[1:]):
        base = int(E["row_ptr"][r0])  # the global offset of the panel (what the ranks exchange)
        prp, pcol, pval, info, _ = run(dA, dB, row_begin=r0, row_end=r1, row_ptr_base=base)
        assert prp[0] == base
        Ep = oracle.spgemm(A, B, rows=np.arange(r0, r1))
        assert oracle.compare(prp, pcol, pval, Ep, rows_offset=base)["ok"]


def test_no_leak_across_plans():
    """Library-owned arenas, streams, events and pinned staging are released by spgemm_free."""
    A = W.rmat(11, 8, seed=3)
    torch.cuda.synchronize()
    for _ in range(2):  # warm the process-wide caches
        with capi.Plan(A, A, 256 << 20, capi.opts(fused=True, chunk_nnz=20000)) as P:
            P.execute_stream(lambda *a: 0)
    free0 = torch.cuda.mem_get_info()[0]
    for k in range(12):
        with capi.Plan(A, A, 256 << 20, capi.opts(fused=bool(k & 1), chunk_nnz=20000, ring=1 + k % 3)) as P:
            P.execute_stream(lambda *a: 0)
    torch.cuda.synchronize()
    assert abs(torch.cuda.mem_get_info()[0] - free0) < (8 << 20)


def test_workspace_from_torch():
    A = W.stencil_3d27(12)
    ws = torch.empty(64 << 20, dtype=torch.uint8, device="cuda")
    rp, col, val, info, _ = run(A, A, budget=ws.numel(), workspace=ws)
    assert info["arena_bytes"] == ws.numel()
    assert_parity(A, A, rp, col, val, exact=True)


# ------------------------------------------------------------------------------------- errors

def test_errors():
    A = W.random_csr(4, 5, 0.5, seed=1)
    B = W.random_csr(6, 3, 0.5, seed=2)
    with pytest.raises(capi.SpgemmError) as e:
        capi.Plan(A, B)
    assert e.value.status == capi.ERR_SHAPE
    C = W.stencil_3d27(16)
    with pytest.raises(capi.SpgemmError) as e:
        capi.Plan(C, C, 1 << 16)
    assert e.value.status == capi.ERR_BUDGET
    bad = W.random_csr(5, 5, 0.8, seed=3)
    bad.col = bad.col[::-1].copy()
    with pytest.raises(capi.SpgemmError) as e:
        capi.Plan(bad, W.identity(5), 0, capi.opts(validate=True))
    assert e.value.status == capi.ERR_INVALID_ARGUMENT
    with pytest.raises(capi.SpgemmError) as e:
        capi.Plan(A, W.random_csr(5, 3, 0.5, 2), 0, capi.opts(row_begin=3, row_end=9))
    assert e.value.status == capi.ERR_SHAPE
    # capacity error of the one-shot API
    AA = W.stencil_2d5(8)
    out = [torch.empty(65, dtype=torch.int64), torch.empty(10, dtype=torch.int32), torch.empty(10, dtype=torch.float64)]
    with pytest.raises(capi.SpgemmError) as e:
        capi.spgemm_multiply(AA, AA, 0, None, *out, capacity=10)
    assert e.value.status == capi.ERR_CAPACITY


def _mutated(M, kind):
    """A copy of M broken in one way (validate must catch each before any kernel reads)."""
    X = W.CSR(M.nrows, M.ncols, M.row_ptr.copy(), M.col.copy(), M.val.copy())
    if kind == "col_high":
        X.col[len(X.col) // 2] = M.ncols + 1000
    elif kind == "col_high_last":
        X.col[-1] = 2 ** 31 - 1
    elif kind == "col_neg":
        X.col[len(X.col) // 3] = -7
    elif kind == "rp_decreasing":
        r = M.nrows // 2
        X.row_ptr[r] = X.row_ptr[r + 1] + 5  # rows r-1, r: one past the next offset
    elif kind == "unsorted":
        r = int(np.argmax(np.diff(M.row_ptr) >= 2))
        p = int(M.row_ptr[r])
        X.col[p], X.col[p + 1] = X.col[p + 1], X.col[p]
    elif kind == "duplicate":
        r = int(np.argmax(np.diff(M.row_ptr) >= 2))
        p = int(M.row_ptr[r])
        X.col[p + 1] = X.col[p]
    return X


@pytest.mark.parametrize("where", ["host", "device"])
@pytest.mark.parametrize("operand", ["A", "B"])
@pytest.mark.parametrize("kind", ["col_high", "col_high_last", "col_neg", "rp_decreasing", "unsorted", "duplicate"])
def test_validate_rejects_bad_operands_before_reading(kind, operand, where):
    """validate = 1: every malformed operand is SPGEMM_ERR_INVALID_ARGUMENT (not an illegal address
    / sticky CUDA error), for host and device operands, in-core and column-panel plans; the
    context stays healthy (a valid multiply afterwards matches the oracle)."""
    A = W.random_csr_sparse(300, 200, 6.0, seed=5)
    B = W.random_csr_sparse(200, 260, 6.0, seed=6)
    bad = _mutated(A if operand == "A" else B, kind)
    X, Y = (bad, B) if operand == "A" else (A, bad)
    if where == "device":
        X, Y = _to_dev(X, base=3), _to_dev(Y, base=0)
    for cp in (1, 3):
        with pytest.raises(capi.SpgemmError) as e:
            capi.Plan(X, Y, 0, capi.opts(validate=True, col_panels=cp))
        assert e.value.status == capi.ERR_INVALID_ARGUMENT, (kind, operand, where, cp, str(e.value))
    torch.cuda.synchronize()
    rp, col, val, _, _ = run(A, B, validate=True)
    assert_parity(A, B, rp, col, val)


@pytest.mark.parametrize("fused", [False, True])
def test_duplicates_unvalidated_keep_structure(fused):
    """validate = 0 with a column repeated inside rows of B (include/spgemm.h, DESIGN R2): the
    structure of C is that of the deduplicated B, exactly; values are undefined there, and exact
    elsewhere (rows that touch no damaged B row)."""
    A = W.random_csr_sparse(400, 300, 5.0, seed=8)
    B = W.random_csr_sparse(300, 250, 40.0, seed=9)   # long B rows: the G = 32 warp tier
    Bd = W.CSR(B.nrows, B.ncols, B.row_ptr.copy(), B.col.copy(), B.val.copy())
    damaged = []
    for k in range(0, B.nrows, 7):
        s, e = int(B.row_ptr[k]), int(B.row_ptr[k + 1])
        if e - s >= 2:
            Bd.col[s + 1] = Bd.col[s]
            damaged.append(k)
    # the same matrix with the duplicate dropped (structure reference)
    keep = np.ones(len(Bd.col), bool)
    for k in damaged:
        keep[int(B.row_ptr[k]) + 1] = False
    cnt = np.diff(B.row_ptr) - np.isin(np.arange(B.nrows), damaged)
    Bu = W.CSR(B.nrows, B.ncols, np.concatenate([[0], np.cumsum(cnt)]).astype(np.int64), Bd.col[keep].copy(),
               Bd.val[keep].copy())
    with pytest.raises(capi.SpgemmError):
        capi.Plan(A, Bd, 0, capi.opts(validate=True))
    if fused:
        rp, col, val, info, _ = run_fused(A, Bd)
    else:
        rp, col, val, info, _ = run(A, Bd)
    E = oracle.spgemm(A, Bu)
    assert np.array_equal(rp, E["row_ptr"]) and np.array_equal(col, E["col"])
    clean = np.array([not np.isin(A.col[A.row_ptr[i]:A.row_ptr[i + 1]], damaged).any() for i in range(A.nrows)])
    rows = np.nonzero(clean)[0]
    assert len(rows) > 10
    assert_parity(A, Bu, rp, col, val, rows=rows)


@pytest.mark.parametrize("case", ["stencil", "rmat", "rect"])
def test_row_products_and_plan_bounds_per_row(case):
    """S2 per row: the library's count kernel gives u_i == the oracle's Alg. 1 line-4 trip count for
    EVERY row (spgemm_row_products), and the plan's own bound array is min(u_i, ncols) for every
    row (spgemm_plan_row_bounds) -- in two-phase and fused plans, host and device operands, and a
    row panel."""
    if case == "stencil":
        A = B = W.stencil_3d27(20)
    elif case == "rmat":
        A = B = W.rmat(13, 16, seed=4)
    else:
        A = W.rmat_rect(12, 10, 40_000, seed=5)
        B = W.rmat_rect(10, 13, 30_000, seed=6)
    u = oracle.products(A, B)
    got, tot = capi.row_products(A, B)
    assert np.array_equal(got, u) and tot == int(u.sum())
    dA, dB = _to_dev(A, base=11), _to_dev(B, base=2)
    r0, r1 = A.nrows // 3, A.nrows - 5
    got, tot = capi.row_products(dA, dB, capi.opts(row_begin=r0, row_end=r1))
    assert np.array_equal(got, u[r0:r1]) and tot == int(u[r0:r1].sum())
    for fused in (False, True):
        with capi.Plan(A, B, 0, capi.opts(fused=fused)) as P:
            if fused:  # host-cut plans (short host rows) count inside execute
                P.execute_stream(lambda *a: 0)
            assert np.array_equal(P.row_bounds(), np.minimum(u, B.ncols))
            assert P.info()["products"] == int(u.sum())
        with capi.Plan(dA, dB, 0, capi.opts(fused=fused, row_begin=r0, row_end=r1)) as P:
            assert np.array_equal(P.row_bounds(), np.minimum(u[r0:r1], B.ncols))


def test_multiply_one_shot():
    A = W.stencil_2d5(16)
    z = int(oracle.row_nnz(A, A).sum())
    rp = torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True)
    col = torch.empty(z, dtype=torch.int32, pin_memory=True)
    val = torch.empty(z, dtype=torch.float64, pin_memory=True)
    n = capi.spgemm_multiply(A, A, 0, None, rp, col, val, capacity=z)
    assert n == z
    assert_parity(A, A, rp.numpy(), col.numpy(), val.numpy(), exact=True)


# ------------------------------------------------------------------------------------- fused plans

def run_fused(A, B, budget=0, capacity=None, **kw):
    o = capi.opts(fused=True, **kw)
    with capi.Plan(A, B, budget, o) as P:
        info0 = P.info()
        assert info0["fused"] == 1 and info0["nnz"] == -1
        cap = capacity if capacity is not None else int(oracle.row_nnz(A, B).sum())
        rp = torch.empty(info0["nrows"] + 1, dtype=torch.int64, pin_memory=True)
        col = torch.empty(max(cap, 0), dtype=torch.int32, pin_memory=True)
        val = torch.empty(max(cap, 0), dtype=torch.float64, pin_memory=True)
        n = P.execute_capacity(rp, col, val, cap)
        info = P.info()
        chunks = P.chunks()
    return rp.numpy(), col.numpy()[:n], val.numpy()[:n], info, chunks


@pytest.mark.parametrize("case", ["c2", "rmat", "rect", "tiers", "degenerate"])
def test_fused_matches_oracle(case):
    if case == "c2":
        A = B = W.stencil_3d27(24)
        kw = {"min_chunks": 9}
    elif case == "rmat":
        A = B = W.rmat(13, 16, seed=3)
        kw = {"chunk_nnz": 50000}
    elif case == "rect":
        A = W.random_csr_sparse(2500, 1700, 7.0, seed=21)
        B = W.random_csr_sparse(1700, 3100, 5.0, seed=22)
        kw = {"chunk_nnz": 4000, "ring": 3}
    elif case == "tiers":
        A, B = _long_rows_case(seed=4)
        kw = {}
    else:
        A = W.random_csr(40, 30, 0.0, seed=1)
        B = W.random_csr(30, 20, 0.5, seed=2)
        kw = {}
    rp, col, val, info, (rows, offs) = run_fused(A, B, **kw)
    assert info["nnz"] == len(col)
    assert_parity(A, B, rp, col, val, exact=(case == "c2"))
    if info["num_chunks"]:
        assert rows[0] == 0 and rows[-1] == A.nrows and offs[-1] == info["nnz"]


def test_fused_two_phase_and_ring1_match_oracle():
    A = W.rmat(12, 16, seed=9)
    E = oracle.spgemm(A, A)
    for r in (run(A, A, chunk_nnz=30000), run_fused(A, A, chunk_nnz=30000, ring=1)):
        assert oracle.compare(r[0], r[1], r[2], E)["ok"]


def test_fused_capacity_error_reports_nnz_and_plan_stays_usable():
    A = W.stencil_3d27(12)
    z = int(oracle.row_nnz(A, A).sum())
    with capi.Plan(A, A, 0, capi.opts(fused=True, min_chunks=5)) as P:
        rp = torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True)
        col = torch.empty(z, dtype=torch.int32, pin_memory=True)
        val = torch.empty(z, dtype=torch.float64, pin_memory=True)
        with pytest.raises(capi.SpgemmError) as e:
            P.execute_capacity(rp, col, val, z // 3)
        assert e.value.status == capi.ERR_CAPACITY and e.value.nnz == z
        assert P.execute_capacity(rp, col, val, z) == z
        assert_parity(A, A, rp.numpy(), col.numpy(), val.numpy(), exact=True)
        # nnz is now known: execute_into works on the fused plan too
        P.execute_into(rp, col, val)
        assert_parity(A, A, rp.numpy(), col.numpy(), val.numpy(), exact=True)


def test_fused_sink_and_base():
    A = W.rmat(12, 16, seed=11)
    E = oracle.spgemm(A, A)
    parts = []
    with capi.Plan(A, A, 0, capi.opts(fused=True, chunk_nnz=40000, ring=2, row_ptr_base=1000)) as P:
        P.execute_stream(lambda r0, r1, rp, col, val: parts.append((r0, r1, rp.copy(), col.copy(), val.copy())))
    assert parts[0][0] == 0 and parts[-1][1] == A.nrows
    rpg = [0]
    for p in parts:
        rpg.extend((p[2][1:] + rpg[-1]).tolist())
    assert oracle.compare(np.array(rpg), np.concatenate([p[3] for p in parts]), np.concatenate([p[4] for p in parts]),
                          E)["ok"]
    rp, c, v, info, _ = run_fused(A, A, row_ptr_base=777)
    assert rp[0] == 777 and oracle.compare(rp, c, v, E, rows_offset=777)["ok"]


def test_chunk_order_by_flops():
    """§IV-C: chunks computed and transferred in decreasing order of flops give the
    same C as row order; fused plans and sink mode reject the reordering."""
    A = W.rmat(13, 16, seed=21)
    r = run(A, A, chunk_nnz=40000, order=1)
    assert r[3]["num_chunks"] > 4
    assert_parity(A, A, r[0], r[1], r[2])
    S = W.stencil_3d27(20)
    rs = run(S, S, chunk_nnz=5000, order=1, profile=True)
    assert_parity(S, S, rs[0], rs[1], rs[2], exact=True)
    with pytest.raises(capi.SpgemmError) as e:
        capi.Plan(A, A, 0, capi.opts(order=1, fused=True))
    assert e.value.status == capi.ERR_INVALID_ARGUMENT
    with capi.Plan(A, A, 0, capi.opts(order=1, chunk_nnz=40000)) as P:
        with pytest.raises(capi.SpgemmError) as e:
            P.execute_stream(lambda *a: 0)
        assert e.value.status == capi.ERR_INVALID_ARGUMENT


def test_matmul_scipy_inputs():
    """The Python convenience wrapper with scipy.sparse operands (unsorted indices are sorted)."""
    sp = pytest.importorskip("scipy.sparse")
    rng = np.random.default_rng(4)
    A = sp.random(300, 200, density=0.05, random_state=1, format="csr") + sp.identity(300, format="csr")[:, :200]
    B = sp.random(200, 500, density=0.04, random_state=2, format="csr")
    A = A.tocsr()
    A.indices = A.indices.copy()
    C = spg.matmul(A, B)
    Aw = spg.as_csr(A)
    Bw = spg.as_csr(B)
    Ao = W.CSR(Aw.nrows, Aw.ncols, Aw.row_ptr, Aw.col, Aw.val)
    Bo = W.CSR(Bw.nrows, Bw.ncols, Bw.row_ptr, Bw.col, Bw.val)
    assert_parity(Ao, Bo, C.row_ptr.numpy(), C.col.numpy(), C.val.numpy())
    C2 = spg.matmul(Ao, Bo, col_panels=2)
    assert np.array_equal(C2.col.numpy(), C.col.numpy())


@pytest.mark.parametrize("case", ["c2", "c1", "random", "slice", "empty_rows"])
def test_host_cut_matches_oracle(case, monkeypatch):
    """Fused C = A*A with host operands and short rows: chunks cut on the host from A.row_ptr,
    per-chunk count inside execute, operands uploaded in interleaved row_ptr/col/value pieces
    (SPGEMM_PIECE_NNZ forces many pieces so chunks wait on different ones).  Same C as the
    oracle, and as the same plan with the host cut disabled; products known after execute."""
    kw = {"fused": True}
    rows = None
    if case == "c2":
        A = W.stencil_3d27(20)
        kw["min_chunks"] = 9
    elif case == "c1":
        A = W.stencil_2d5(64)
        kw["chunk_nnz"] = 3000
    elif case == "random":
        A = W.random_csr_sparse(3000, 3000, 6.0, seed=31)
        kw["chunk_nnz"] = 20000
    elif case == "slice":
        A = W.stencil_3d27(16)
        kw.update(row_begin=700, row_end=3500, chunk_nnz=40000)
        rows = list(range(700, 3500))
    else:
        A = W.random_csr(2000, 2000, 0.002, seed=5)  # many empty rows
        kw["chunk_nnz"] = 5000
    monkeypatch.setenv("SPGEMM_PIECE_NNZ", "7000")
    outs = []
    for off in ("0", "1"):
        monkeypatch.setenv("SPGEMM_NO_HOST_CUT", off)
        with capi.Plan(A, A, 0, capi.opts(**kw)) as P:
            pre = P.info()
            n = info_nrows = pre["nrows"]
            cap = int(oracle.row_nnz(A, A, rows=rows).sum()) if rows else int(oracle.row_nnz(A, A).sum())
            rp = torch.empty(info_nrows + 1, dtype=torch.int64, pin_memory=True)
            col = torch.empty(max(cap, 1), dtype=torch.int32, pin_memory=True)
            val = torch.empty(max(cap, 1), dtype=torch.float64, pin_memory=True)
            z = P.execute_capacity(rp, col, val, cap)
            info = P.info()
            assert z == cap == info["nnz"] and n == info["nrows"]
            u = oracle.products(A, A)
            p = int(u[rows].sum()) if rows else int(u.sum())
            assert info["products"] == p
            if off == "0" and case != "empty_rows":
                assert pre["products"] == -1  # host cut: counted inside execute
            # a second execution of the same plan (count totals reset, not accumulated)
            z2 = P.execute_capacity(rp, col, val, cap)
            assert z2 == z and P.info()["products"] == p
        outs.append((rp.numpy().copy(), col.numpy()[:z].copy(), val.numpy()[:z].copy()))
    rp, col, val = outs[0]
    if rows is None:
        assert_parity(A, A, rp, col, val, exact=case in ("c2", "c1"))
    else:  # the slice's C (row_ptr from 0) against the oracle's selected rows
        E = oracle.spgemm(A, A, rows=rows)
        assert oracle.compare(rp, col, val, E)["ok"] and np.array_equal(val, E["val"])
    assert all(np.array_equal(x, y) for x, y in zip(outs[0][:2], outs[1][:2]))


@pytest.mark.parametrize("shift", [0, 1, 3, 17])
def test_unaligned_host_outputs(shift):
    """Output chunks are padded in their ring slots to the host destination's alignment and copied
    as a head + an aligned bulk: host buffers at any element offset get the same C (fused and
    two-phase plans, small chunks so that many chunks start at odd offsets)."""
    A = W.stencil_3d27(14)
    z = int(oracle.row_nnz(A, A).sum())
    E = oracle.spgemm(A, A)
    for fused in (True, False):
        with capi.Plan(A, A, 0, capi.opts(fused=fused, chunk_nnz=9000, ring=3)) as P:
            rp = torch.empty(A.nrows + 1, dtype=torch.int64, pin_memory=True)
            colb = torch.full((z + shift,), -7, dtype=torch.int32, pin_memory=True)
            valb = torch.full((z + shift,), -7.0, dtype=torch.float64, pin_memory=True)
            col, val = colb[shift:], valb[shift:]
            assert P.execute_capacity(rp, col, val, z) == z
        assert (colb[:shift] == -7).all() and (valb[:shift] == -7.0).all()
        res = oracle.compare(rp.numpy(), col.numpy(), val.numpy(), E)
        assert res["ok"], res
        assert np.array_equal(val.numpy(), E["val"])
