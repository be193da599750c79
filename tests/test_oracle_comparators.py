"""Pins of the oracle's NEXT-2 / NEXT-3 additions (no GPU).

* SEA-ABFT comparator bound (§III): the paper's Table II / III "AVG. SEA-ABFT"
  columns (tests/golden/), a closed form on all-ones matrices, the library norm,
  and "it is a bound" against the exact checksum error.
* Check / correct against an external eps (fixed-eps ABFT of Table I; SEA):
  integer-exact special cases and equivalence with the A-ABFT check when its own eps is
  passed in.
* Alg 3 "errorVecMul" (site 4): on integer data the injected error is exactly
  (fl(a*b) XOR mask) - a*b, computed here with numpy bit views.
"""
import json
import os

import numpy as np
import pytest

import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def gen(recipe, r, c, seed, mid, dtype=np.float64, **kw):
    return synth.generate(recipe, r, c, seed=seed, matrix_id=mid, dtype=dtype, **kw)


def _golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


# --------------------------------------------------------------------------- SEA bound
@pytest.mark.parametrize("table", ["table2_uniform1.json", "table3_uniform100.json"])
@pytest.mark.parametrize("n", [512, 1024, 2048])
def test_sea_table_column(orc, n, table):
    """Table II / III "AVG. SEA-ABFT": mean SEA bound over every checksum element
    of the full-checksum blocks -- BS column checksums, BS row checksums and the corner per
    BS x BS block (reading R25), BS = 32, t = 52.  Within 5% (measured 0.996-1.008)."""
    g = _golden(table)
    paper = g["rows"][str(n)]["avg_sea_abft"]
    A = gen(g["recipe"], n, n, 1, 0)
    B = gen(g["recipe"], n, n, 2, 1)
    bs = 32
    Acs, Bcs = orc.encode_cols(A, bs), orc.encode_rows(B, bs)
    s = orc.sea_bounds(A, B, Acs, Bcs, bs)
    tot = s["eps_col"].sum() + s["eps_row"].sum() + s["eps_corner"].sum()
    cnt = s["eps_col"].size + s["eps_row"].size + s["eps_corner"].size
    m = tot / cnt
    assert 0.95 * paper <= m <= 1.05 * paper, (n, m, paper, m / paper)
    # without the corner the mean sits ~7% low: the corner reading is what the table averages
    m_nc = (s["eps_col"].mean() + s["eps_row"].mean()) / 2
    assert m_nc < 0.95 * paper


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_sea_closed_form_all_ones(orc, dtype):
    """A = B = 1: ||a_i|| = ||b_j|| = sqrt(K), ||Acs_I|| = ||Bcs_J|| = m sqrt(K), so
    eps_col = eps_row = m K (2K + 2m - 2) 2^-t and the corner = m^2 K (2K + 2m - 2) 2^-t."""
    M, N, K, bs = 64, 96, 40, 16
    A = np.ones((M, K), dtype)
    B = np.ones((K, N), dtype)
    t = 52 if dtype == np.float64 else 23
    s = orc.sea_bounds(A, B, orc.encode_cols(A, bs), orc.encode_rows(B, bs), bs)
    m = bs
    want = m * K * (2 * K + 2 * m - 2) * 2.0 ** -t
    np.testing.assert_allclose(s["eps_col"], want, rtol=1e-14)
    np.testing.assert_allclose(s["eps_row"], want, rtol=1e-14)
    np.testing.assert_allclose(s["eps_corner"], m * want, rtol=1e-14)


def test_sea_norms_are_the_2_norm(orc):
    A = gen("wide", 37, 53, 5, 0)
    np.testing.assert_allclose(orc.norms_rows(A), np.linalg.norm(A, axis=1), rtol=1e-14)
    np.testing.assert_allclose(orc.norms_cols(A), np.linalg.norm(A, axis=0), rtol=1e-14)
    A32 = A.astype(np.float32)
    np.testing.assert_allclose(orc.norms_rows(A32), np.linalg.norm(A32.astype(np.float64), axis=1),
                               rtol=1e-14)


@pytest.mark.parametrize("recipe", ["uniform", "wide", "positive"])
def test_sea_bounds_the_exact_error_and_is_looser(orc, recipe):
    """SEA is a bound: |carried checksum - exact| below it everywhere; and it is far
    looser than A-ABFT's eps ('typically two orders of magnitude')."""
    n, bs = 256, 32
    A = gen(recipe, n, n, 11, 0)
    B = gen(recipe, n, n, 12, 1)
    r = orc.protected_matmul(A, B, bs=bs, p=2)
    Acs, Bcs = r["enc"]["Acs"], r["enc"]["Bcs"]
    ex_col = np.zeros(r["Ccol"].shape, np.longdouble)
    ex_row = np.zeros(r["Crow"].shape, np.longdouble)
    for k in range(n):
        ex_col += np.outer(Acs[:, k].astype(np.longdouble), B[k].astype(np.longdouble))
        ex_row += np.outer(A[:, k].astype(np.longdouble), Bcs[k].astype(np.longdouble))
    err_col = np.abs(r["Ccol"].astype(np.longdouble) - ex_col).astype(np.float64)
    err_row = np.abs(r["Crow"].astype(np.longdouble) - ex_row).astype(np.float64)
    s = orc.sea_bounds(A, B, Acs, Bcs, bs)
    assert np.all(err_col < s["eps_col"]) and np.all(err_row < s["eps_row"])
    b = orc.bounds_all(n, n, n, bs, 2, r["enc"]["topA"], r["enc"]["topB"])
    ratio = s["eps_col"].mean() / b["eps_col"].mean()
    assert 10 < ratio < 1000, ratio


# --------------------------------------------------------------------------- external eps
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_fixed_eps_integer_exact(orc, dtype):
    """Integer data: every checksum is exact, so eps = 0 is consistent; a +3 fault is located
    and corrected bit-exactly; with eps above the fault it stays silent."""
    A = gen("integer", 32, 48, 3, 0, dtype=dtype, q=7)
    B = gen("integer", 48, 32, 4, 1, dtype=dtype, q=7)
    clean = orc.abft_matmul_ext(A, B, bs=8, mode="fixed", eps_fixed=0.0)
    assert clean["check"].counts[1] == 16 and clean["check"].counts[7] == 0
    f = [dict(row=13, col=22, site=2, add=3.0)]
    r = orc.abft_matmul_ext(A, B, bs=8, mode="fixed", eps_fixed=0.0, faults=f)
    assert r["check"].status[1, 2] == 1 and r["check"].counts[2] == 1
    assert np.array_equal(r["C"], clean["C"])
    r = orc.abft_matmul_ext(A, B, bs=8, mode="fixed", eps_fixed=3.5, faults=f)
    assert r["check"].counts[1] == 16
    assert r["C"][13, 22] == clean["C"][13, 22] + 3


def test_ext_check_with_aabft_eps_matches_check(orc):
    """Passing A-ABFT's own eps as external eps reproduces the A-ABFT verdicts (the check and
    correction logic is shared; only the eps source differs)."""
    M, K, bs = 96, 80, 16
    A = gen("uniform", M, K, 1, 0)
    B = gen("uniform", K, M, 2, 1)
    enc = orc.encode(A, B, bs, 2)
    b = orc.bounds_all(M, M, K, bs, 2, enc["topA"], enc["topB"])
    faults = [dict(row=5, col=7, site=0, xor_mask=1 << 62), dict(row=40, col=70, site=2, add=1e-3),
              dict(row=90, col=3, site=2, add=1e-18), dict(row=M + 2, col=50, site=2, add=0.5)]
    r1 = orc.protected_matmul(A, B, bs=bs, p=2, faults=faults)
    r2 = orc.protected_matmul(A, B, bs=bs, p=2, faults=faults, do_correct=False)
    ch = orc.check_ext(r2["C"], r2["Ccol"], r2["Crow"], bs, eps_col=b["eps_col"],
                       eps_row=b["eps_row"])
    orc.correct_ext(r2["C"], r2["Ccol"], r2["Crow"], bs, ch, eps_row=b["eps_row"])
    assert np.array_equal(ch.status, r1["check"].status)
    assert np.array_equal(ch.row, r1["check"].row) and np.array_equal(ch.col, r1["check"].col)
    assert ch.counts[7] == r1["check"].counts[7] and ch.counts[2] == r1["check"].counts[2]
    assert np.array_equal(r2["C"], r1["C"])


# --------------------------------------------------------------------------- Alg 3 mul site
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_mul_fault_site4_integer(orc, dtype):
    """errorVecMul: accum += (rA*rB) XOR mask at one step.  Integer data keeps
    every sum exact, so the faulty element equals clean + ((p ^ mask) - p), p = a_ik b_kj."""
    M, K, N, bs = 16, 24, 16, 8
    A = gen("integer", M, K, 7, 0, dtype=dtype, q=9)
    B = gen("integer", K, N, 8, 1, dtype=dtype, q=9)
    clean = orc.protected_matmul(A, B, bs=bs, p=2)
    ut = np.uint64 if dtype == np.float64 else np.uint32
    rng = np.random.default_rng(1)
    for trial in range(40):
        i, j, k = int(rng.integers(0, M)), int(rng.integers(0, N)), int(rng.integers(0, K))
        p = A[i, k] * B[k, j]
        if p == 0:
            continue
        nb = 64 if dtype == np.float64 else 32
        bit = int(rng.integers(nb - 12, nb - 1))  # exponent bits: large, still finite mostly
        pf = np.array([p], dtype).view(ut) ^ ut(1 << bit)
        e = float(pf.view(dtype)[0]) - float(p)
        f = dict(row=i, col=j, site=4, k_step=k, xor_mask=1 << bit)
        r = orc.protected_matmul(A, B, bs=bs, p=2, faults=[f], do_correct=False)
        got = float(r["C"][i, j]) - float(clean["C"][i, j])
        if np.isfinite(e) and abs(e) < 2.0 ** 20:
            assert got == e, (i, j, k, bit, got, e)
        if not np.isfinite(e) or abs(e) >= 1:
            assert r["check"].status[i // bs, j // bs] == 4
    # mask 0 is the fault-free separately-rounded step: identical on integer data
    r = orc.protected_matmul(A, B, bs=bs, p=2, faults=[dict(row=3, col=4, site=4, k_step=5)])
    assert np.array_equal(r["C"], clean["C"])


def test_mul_fault_site4_equals_nonfma_step(orc):
    """With fma_model = 0 every step is c + fl(a*b); site 4 with mask 0 must then be a no-op
    on any data (the fault-free product is the separately rounded one)."""
    a = gen("uniform", 1, 300, 3, 0)[0]
    b = gen("uniform", 300, 1, 4, 1)[:, 0].copy()
    ref = orc.dot_fault(a, b, fma_model=0)
    for k in (0, 17, 299):
        assert orc.dot_fault(a, b, fma_model=0, site=4, k_step=k, xor_mask=0) == ref
