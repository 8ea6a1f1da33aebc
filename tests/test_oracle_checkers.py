"""Pins for the parity checkers (`-m "not gpu"`): oracle.compare() and oracle.verify().

Every GPU parity test ends in one of these two functions, so each is pinned by MUTATION: a
candidate that differs from C = A x B (§I; Alg. 1 L33-50) in any one part -- a
row_ptr entry, a column, a value just outside BASELINE.json's bound |c - ref| <= 1e-12 sum|a*b|,
an infinity of the wrong sign, a NaN where a number belongs -- must be rejected, and a correct
one accepted, including the special cases of SURVEY.md §8(c)'s comparison rule (equal
infinities, NaN against NaN, +-0.0 when every product is zero).  The expected outcome of each
case is fixed by the rule, not by the checkers.  Finally, three plausible bugs in the checker
itself (always ok; values compared with themselves instead of the reference; the bound's `<=`
flipped) are injected and each must make at least one pin fail.
"""
import numpy as np
import pytest

import oracle
import workloads as W

INF, NAN = float("inf"), float("nan")


def _csr(dense_rows, ncols):
    """CSR from {row: [(col, val), ...]} (columns given in increasing order)."""
    nrows = len(dense_rows)
    rp, col, val = [0], [], []
    for i in range(nrows):
        for c, v in dense_rows[i]:
            col.append(c)
            val.append(v)
        rp.append(len(col))
    return W.CSR(nrows, ncols, np.array(rp, dtype=np.int64), np.array(col, dtype=np.int32),
                 np.array(val, dtype=np.float64))


def _cand(E):
    return E["row_ptr"].copy(), E["col"].copy(), E["val"].copy()


def _random_case(seed=3):
    A = W.random_csr(40, 30, 0.2, seed)
    B = W.random_csr(30, 50, 0.2, seed + 1)
    return A, B, oracle.spgemm(A, B)


def _cases():
    """(name, A, B, candidate (rp, col, val), should_pass, expected failing kind)."""
    out = []
    A, B, E = _random_case()
    out.append(("exact", A, B, _cand(E), True, None))
    # row_ptr: one interior entry moved by one (two rows' lengths change)
    rp, col, val = _cand(E)
    r = int(np.argmax(np.diff(E["row_ptr"]) > 1)) + 1
    rp[r] += 1
    out.append(("row_ptr+1", A, B, (rp, col, val), False, "row_ptr"))
    # column: two neighbours swapped (unsorted row)
    rp, col, val = _cand(E)
    i = int(np.argmax(np.diff(E["row_ptr"]) >= 2))
    p = int(E["row_ptr"][i])
    col[p], col[p + 1] = col[p + 1], col[p]
    out.append(("col_swap", A, B, (rp, col, val), False, "col"))
    # column: one entry replaced by a column NOT in the row's structure, order kept
    rp, col, val = _cand(E)
    done = False
    for i in range(A.nrows):
        s, e = int(E["row_ptr"][i]), int(E["row_ptr"][i + 1])
        for p in range(s, e):
            lo = col[p - 1] + 1 if p > s else 0
            hi = col[p + 1] if p + 1 < e else B.ncols
            free = [c for c in range(lo, hi) if c != col[p]]
            if free:
                col[p] = free[0]
                done = True
                break
        if done:
            break
    assert done
    out.append(("col_outside_set", A, B, (rp, col, val), False, "col"))
    # values: inside and just outside the bound
    k = int(np.argmax(E["tol"] > 0))
    for frac, ok in ((0.5, True), (1.0, True), (2.0, False), (-2.0, False)):
        rp, col, val = _cand(E)
        v = E["ref"][k] + frac * E["tol"][k]
        if frac == 1.0:  # the largest double whose distance from ref is still <= tol (at the bound)
            while abs(v - E["ref"][k]) > E["tol"][k]:
                v = np.nextafter(v, -np.inf)
            assert abs(np.nextafter(v, np.inf) - E["ref"][k]) > E["tol"][k]
        val[k] = v
        out.append((f"val_{frac}tol", A, B, (rp, col, val), ok, None if ok else "val"))
    # every product zero (explicit zero in A): ref = tol = 0, only +-0.0 passes (reading R1)
    Az = _csr([[(0, 0.0)]], 1)
    Bz = _csr([[(0, 3.0)]], 1)
    Ez = oracle.spgemm(Az, Bz)
    assert Ez["tol"][0] == 0.0 and Ez["ref"][0] == 0.0
    for v, ok in ((0.0, True), (-0.0, True), (1e-300, False)):
        out.append((f"zero_{v}", Az, Bz, (Ez["row_ptr"].copy(), Ez["col"].copy(), np.array([v])), ok,
                    None if ok else "val"))
    # infinities: C00 = +inf * 2 = +inf
    Ai = _csr([[(0, INF)]], 1)
    Bi = _csr([[(0, 2.0)]], 1)
    Ei = oracle.spgemm(Ai, Bi)
    assert Ei["ref"][0] == INF
    for v, ok in ((INF, True), (-INF, False), (1.7e308, False), (NAN, False)):
        out.append((f"inf_{v}", Ai, Bi, (Ei["row_ptr"].copy(), Ei["col"].copy(), np.array([v])), ok,
                    None if ok else "val"))
    # finite reference, infinite candidate
    Af = _csr([[(0, 1.0)]], 1)
    Ef = oracle.spgemm(Af, Bi)
    out.append(("finite_vs_inf", Af, Bi, (Ef["row_ptr"].copy(), Ef["col"].copy(), np.array([INF])), False, "val"))
    # NaN: inf * 0 (IEEE propagation, reading R18)
    An = _csr([[(0, INF)]], 1)
    Bn = _csr([[(0, 0.0)]], 1)
    En = oracle.spgemm(An, Bn)
    assert np.isnan(En["ref"][0])
    for v, ok in ((NAN, True), (0.0, False), (INF, False)):
        out.append((f"nan_{v}", An, Bn, (En["row_ptr"].copy(), En["col"].copy(), np.array([v])), ok,
                    None if ok else "val"))
    # -inf against -inf (the other sign) is good
    Am = _csr([[(0, -INF)]], 1)
    Em = oracle.spgemm(Am, Bi)
    out.append(("neg_inf_equal", Am, Bi, (Em["row_ptr"].copy(), Em["col"].copy(), np.array([-INF])), True, None))
    return out


CASES = _cases()


def _compare_outcome(cmp, A, B, cand):
    E = oracle.spgemm(A, B)
    res = cmp(*cand, E)
    return bool(res["ok"]), (res.get("first_bad") or (None,))[0]


@pytest.mark.parametrize("case", CASES, ids=[c[0] for c in CASES])
def test_compare_pins(case):
    name, A, B, cand, should, kind = case
    ok, got = _compare_outcome(oracle.compare, A, B, cand)
    assert ok == should, name
    if not should:
        assert got == kind, (name, got)


@pytest.mark.parametrize("case", CASES, ids=[c[0] for c in CASES])
def test_verify_pins_agree_with_rule(case):
    name, A, B, cand, should, kind = case
    rp, col, val = cand
    res = oracle.verify(A, B, 0, rp, col, val, threads=2)
    assert res["ok"] == should, (name, res)
    if not should:
        assert res["first_bad_kind"] == kind, (name, res)
    else:
        assert res["rows"] == A.nrows and res["entries"] == int(rp[-1])


def test_compare_length_mismatch_rejected():
    A, B, E = _random_case()
    rp, col, val = _cand(E)
    res = oracle.compare(rp, np.append(col, 0), np.append(val, 0.0), E)
    assert not res["ok"] and res["first_bad"][0] == "length"
    res = oracle.compare(rp[:-1], col, val, E)
    assert not res["ok"] and res["first_bad"][0] == "row_ptr"


def test_compare_rows_offset_semantics():
    A, B, E = _random_case()
    rp, col, val = _cand(E)
    assert oracle.compare(rp + 1000, col, val, E, rows_offset=1000)["ok"]
    assert not oracle.compare(rp + 1000, col, val, E)["ok"]


def test_worst_ratio_reported():
    A, B, E = _random_case()
    rp, col, val = _cand(E)
    k = int(np.argmax(E["tol"]))
    val[k] = E["ref"][k] + 0.25 * E["tol"][k]
    r = oracle.compare(rp, col, val, E)
    assert r["ok"] and 0.2 < r["worst_ratio"] <= 0.3
    v = oracle.verify(A, B, 0, rp, col, val)
    assert v["ok"] and 0.2 < v["worst_ratio"] <= 0.3


def test_verify_products_and_row_windows():
    """verify() on a window of rows [row0, row0 + n) with any row_ptr base, and the optional
    per-row product counts (Alg. 1 line-4 trip counts, §III-B)."""
    A, B, E = _random_case(7)
    u = oracle.products(A, B)
    r0, r1 = 5, 23
    rp = E["row_ptr"][r0:r1 + 1] + 777
    s, e = int(E["row_ptr"][r0]), int(E["row_ptr"][r1])
    res = oracle.verify(A, B, r0, rp, E["col"][s:e], E["val"][s:e], products=u[r0:r1])
    assert res["ok"] and res["rows"] == r1 - r0 and res["products"] == int(u[r0:r1].sum())
    bad = u[r0:r1].copy()
    bad[3] += 1
    res = oracle.verify(A, B, r0, rp, E["col"][s:e], E["val"][s:e], products=bad)
    assert not res["ok"] and res["first_bad_kind"] == "products" and res["first_bad_row"] == r0 + 3
    with pytest.raises(RuntimeError):
        oracle.verify(A, B, A.nrows - 2, E["row_ptr"][:5], E["col"], E["val"])


def test_verify_equals_compare_on_rmat():
    """The two checkers agree on a skewed input with thousands of rows, and on the mutation of
    one value in the middle."""
    A = W.rmat(10, 8)
    E = oracle.spgemm(A, A)
    rp, col, val = _cand(E)
    assert oracle.compare(rp, col, val, E)["ok"] and oracle.verify(A, A, 0, rp, col, val)["ok"]
    k = len(val) // 2
    val[k] = E["ref"][k] + 3 * E["tol"][k] + 1e-300
    assert not oracle.compare(rp, col, val, E)["ok"]
    res = oracle.verify(A, A, 0, rp, col, val)
    assert not res["ok"] and res["bad_val"] == 1


# ---------------------------------------------------------------- mutated checkers must be caught

def _mut_always_ok(rp, col, val, expect, rows_offset=0):
    return {"ok": True, "worst_ratio": 0.0, "n": 0, "first_bad": None}


def _mut_value_against_self(monkeypatch):
    real = oracle._value_good
    monkeypatch.setattr(oracle, "_value_good", lambda val, ref, tol: real(val, val, tol))


def _mut_flipped_bound(monkeypatch):
    def flipped(val, ref, tol):
        with np.errstate(invalid="ignore"):
            err = np.abs(val - ref)
        return (err >= tol) | (np.isnan(val) & np.isnan(ref)), np.zeros(len(val))
    monkeypatch.setattr(oracle, "_value_good", flipped)


def _pins_failing(cmp):
    bad = 0
    for name, A, B, cand, should, kind in CASES:
        ok, _ = _compare_outcome(cmp, A, B, cand)
        bad += ok != should
    return bad


def test_pins_catch_mutated_checkers(monkeypatch):
    assert _pins_failing(oracle.compare) == 0
    assert _pins_failing(_mut_always_ok) > 0
    with monkeypatch.context() as m:
        _mut_value_against_self(m)
        assert _pins_failing(oracle.compare) > 0
    with monkeypatch.context() as m:
        _mut_flipped_bound(m)
        assert _pins_failing(oracle.compare) > 0


def test_verify_chunked_with_persistent_scratch():
    """The sink's usage: one Operands (persistent per-thread marker arrays) and many chunk windows;
    stale marks from earlier windows must never count as structure of a later row."""
    A = W.rmat(11, 8, seed=5)
    E = oracle.spgemm(A, A)
    ops = oracle.Operands(A, A, threads=3)
    rp = E["row_ptr"]
    cuts = [0, 1, 2, 300, 301, 1000, A.nrows]
    tot = 0
    for a, b in zip(cuts[:-1], cuts[1:]):
        r = oracle.verify(A, A, a, rp[a:b + 1], E["col"][rp[a]:rp[b]], E["val"][rp[a]:rp[b]], ops=ops)
        assert r["ok"] and r["rows"] == b - a
        tot += r["entries"]
    assert tot == len(E["col"])
    # a row of the last window claiming a column that belonged to the row checked just before it
    a, b = 1000, A.nrows
    col = E["col"][rp[a]:rp[b]].copy()
    i = next(i for i in range(a, b) if rp[i + 1] > rp[i] and rp[i] > rp[i - 1])
    prev_cols = set(E["col"][rp[i - 1]:rp[i]]) - set(E["col"][rp[i]:rp[i + 1]])
    if prev_cols:
        j = sorted(prev_cols)[0]
        row = np.array(sorted(set(E["col"][rp[i]:rp[i + 1]][1:]) | {j}), dtype=np.int32)
        if len(row) == rp[i + 1] - rp[i]:
            col[rp[i] - rp[a]:rp[i + 1] - rp[a]] = row
            r = oracle.verify(A, A, a, rp[a:b + 1], col, E["val"][rp[a]:rp[b]], ops=ops)
            assert not r["ok"] and r["first_bad_kind"] == "col"
