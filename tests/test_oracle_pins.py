"""Pins of the CPU oracle against what the paper and mathematics fix (no GPU).

Each test names the PAPER.md passage (P:Lnn) it pins.  None of them re-types the
oracle's formula: they use closed forms derived independently, brute force,
exact integer arithmetic, statistical checks of the rounding model, and the
paper's printed Table II/III numbers (tests/golden/).
"""
import itertools
import json
import os

import numpy as np
import pytest

import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def gen(recipe, r, c, seed, mid, dtype=np.float64, **kw):
    return synth.generate(recipe, r, c, seed=seed, matrix_id=mid, dtype=dtype, **kw)


# --------------------------------------------------------------------------- O2 encode
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("bs", [4, 8, 32])
def test_encode_integer_exact(orc, dtype, bs):
    """Eq 1/2: with integer data every checksum is the exact integer sum."""
    A = gen("integer", 64, 48, 1, 0, dtype, q=50)
    B = gen("integer", 48, 64, 2, 1, dtype, q=50)
    Acs = orc.encode_cols(A, bs)
    Bcs = orc.encode_rows(B, bs)
    Ai = A.astype(np.int64)
    Bi = B.astype(np.int64)
    assert np.array_equal(Acs.astype(np.int64), Ai.reshape(64 // bs, bs, 48).sum(axis=1))
    assert np.array_equal(Bcs.astype(np.int64), Bi.reshape(48, 64 // bs, bs).sum(axis=2))
    # sum over all partitions = full column / row sum (exact for integers)
    assert np.array_equal(Acs.astype(np.int64).sum(0), Ai.sum(0))
    assert np.array_equal(Bcs.astype(np.int64).sum(1), Bi.sum(1))


def test_encode_closed_forms(orc):
    """A = ones => Acs == BS; A = I => checksum rows are block indicator vectors."""
    bs = 8
    ones = np.ones((32, 24))
    assert np.all(orc.encode_cols(ones, bs) == bs)
    assert np.all(orc.encode_rows(np.ones((24, 32)), bs) == bs)
    eye = np.eye(32)
    Acs = orc.encode_cols(eye, bs)
    for I in range(4):
        ind = np.zeros(32)
        ind[I * bs:(I + 1) * bs] = 1
        assert np.array_equal(Acs[I], ind)
    Bcs = orc.encode_rows(eye, bs)
    for J in range(4):
        ind = np.zeros(32)
        ind[J * bs:(J + 1) * bs] = 1
        assert np.array_equal(Bcs[:, J], ind)


def test_encode_sequential_order(orc):
    """Alg 1: each column is summed top to bottom.  A cancellation case
    distinguishes sequential order from pairwise / reversed order."""
    A = np.zeros((4, 1))
    A[:, 0] = [1e16, 1.0, -1e16, 1.0]   # sequential: ((1e16+1)-1e16)+1 = 1.0 ; exact = 2
    Acs = orc.encode_cols(A, 4)
    assert Acs[0, 0] == 1.0
    B = A.T.copy()
    assert orc.encode_rows(B, 4)[0, 0] == 1.0


# --------------------------------------------------------------------------- O3 top-p
def _brute_topp(x, p):
    order = sorted(range(len(x)), key=lambda k: (-abs(float(x[k])), k))
    return np.array([abs(float(x[k])) for k in order[:p]]), np.array(order[:p])


@pytest.mark.parametrize("recipe", ["uniform", "integer"])
def test_topp_brute_force(orc, recipe):
    """§IV-E / Alg 1: p largest |values|, ties -> lowest index."""
    rng = np.random.default_rng(7)
    for trial in range(300):
        n = int(rng.integers(1, 20))
        p = int(rng.integers(1, min(n, 8) + 1))
        x = gen(recipe, 1, n, trial, 3, q=3)[0]
        v, i = orc.topp_vector(x, p)
        bv, bi = _brute_topp(x, p)
        assert np.array_equal(v, bv) and np.array_equal(i, bi), (x, p)


def test_topp_p_equals_len_returns_all(orc):
    x = gen("uniform", 1, 9, 5, 5)[0]
    v, i = orc.topp_vector(x, 8)
    assert sorted(i.tolist()) == sorted(np.argsort(-np.abs(x))[:8].tolist())
    v, i = orc.topp_vector(x[:8], 8)
    assert sorted(i.tolist()) == list(range(8))


def test_topp_rows_cols_cover_checksums(orc):
    """Reading R4: checksum rows of A and checksum columns of B are in the top-p tables."""
    A = gen("uniform", 16, 12, 1, 0)
    B = gen("uniform", 12, 16, 2, 1)
    Acs = orc.encode_cols(A, 8)
    Bcs = orc.encode_rows(B, 8)
    va, ia = orc.topp_rows(A, Acs, 8, 2)
    vb, ib = orc.topp_cols(B, Bcs, 8, 2)
    assert va.shape == (18, 2) and vb.shape == (18, 2)
    for r in range(16):
        assert np.array_equal(va[r], _brute_topp(A[r], 2)[0])
    for I in range(2):
        assert np.array_equal(va[16 + I], _brute_topp(Acs[I], 2)[0])
    for J in range(2):
        assert np.array_equal(vb[16 + J], _brute_topp(Bcs[:, J], 2)[0])


# --------------------------------------------------------------------------- O5 y
def _alt_topsets(x, p):
    """Every valid top-p index set of |x| (all tie-breaks)."""
    ax = np.abs(x)
    srt = np.sort(ax)[::-1]
    thr = srt[p - 1]
    above = [k for k in range(len(x)) if ax[k] > thr]
    at = [k for k in range(len(x)) if ax[k] == thr]
    for comb in itertools.combinations(at, p - len(above)):
        idx = sorted(above + list(comb), key=lambda k: -ax[k])
        yield ax[idx], np.array(idx, np.int32)


def test_y_upper_bound_exact_and_tie_invariant(orc):
    """Eq 46: y >= |a_k b_k| for all k; y is exact when p >= K; y does not depend
    on which equal-valued elements the top-p tie-break picks (brute force)."""
    rng = np.random.default_rng(11)
    n_checked = 0
    for trial in range(3000):
        K = int(rng.integers(1, 9))
        p = int(rng.integers(1, min(K, 4) + 1))
        if trial % 2:
            a = rng.integers(-3, 4, K).astype(float)
            b = rng.integers(-3, 4, K).astype(float)
        else:
            a = rng.uniform(-1, 1, K)
            b = rng.uniform(-1, 1, K)
        true_max = float(np.max(np.abs(a * b)))
        ys = set()
        for (va, ia) in _alt_topsets(a, p):
            for (vb, ib) in _alt_topsets(b, p):
                y = orc.y_of(va, ia, vb, ib)
                assert y >= true_max, (a, b, p)
                ys.add(y)
                n_checked += 1
        assert len(ys) == 1, (a, b, p, ys)
        if p >= K:
            assert ys.pop() == true_max
    assert n_checked > 3000


def test_y_three_cases_examples(orc):
    """§IV-E bullets on hand-made vectors."""
    # S = {0}: case 1 gives |a0 b0| = 6, case 2 = 3*1, case 3 = 2*1 -> 6
    assert orc.y_of([3, 1], [0, 1], [2, 1], [0, 2]) == 6.0
    # S empty: max(va)*min(vb) = 5*0.5 vs max(vb)*min(va) = 4*0.25
    assert orc.y_of([5, 0.25], [0, 1], [4, 0.5], [2, 3]) == 2.5


# --------------------------------------------------------------------------- O6 sigma
@pytest.mark.parametrize("n", [1, 2, 3, 4, 17, 128, 1000, 4096])
def test_sigma_coeff_is_the_derivation_sum(orc, n):
    """Eq 26 -> 28: Var_Sum <= 1/8 * 2^-2t * sum_{k<=n} (k y)^2, so
    sigma/(y 2^-t) = sqrt(sum k^2 / 8); P:L287 adds Var_Prod <= n/12 2^-2t y^2 (Eq 41).
    Here the sums are done by brute force (Python integers), not the closed form."""
    s2 = sum(k * k for k in range(1, n + 1))
    assert orc.sigma_coeff(n, 1) == pytest.approx((s2 / 8) ** 0.5, rel=1e-15)
    assert orc.sigma_coeff(n, 0) == pytest.approx((s2 / 8 + n / 12) ** 0.5, rel=1e-15)


def test_bound_scaling(orc):
    """eps = omega * sigma (Eq 7), sigma proportional to y * 2^-t (Eq 28)."""
    s1, e1 = orc.bound(100, 1.0, t=52, omega=3.0)
    s2, e2 = orc.bound(100, 4.0, t=52, omega=3.0)
    s3, e3 = orc.bound(100, 1.0, t=23, omega=1.0)
    assert s2 == 4 * s1 and e1 == 3 * s1 and s3 == s1 * 2.0 ** 29 and e3 == s3
    s0, e0 = orc.bound(100, 0.0)
    assert s0 == 0 and e0 == 0


def test_rounding_model_covers_actual_error(orc):
    """The probabilistic model (§IV-B, Eq 28): the actual rounding error of a sequential
    fused inner product stays well inside 3 sigma.  Error measured against a long-double
    reference (exact to ~2^-64 relative)."""
    rng = np.random.default_rng(3)
    K = 512
    worst = 0.0
    for trial in range(200):
        a = rng.uniform(-1, 1, K)
        b = rng.uniform(-1, 1, K)
        c = orc.dot_fault(a, b, 1)
        exact = float(np.sum(a.astype(np.longdouble) * b.astype(np.longdouble)))
        va, ia = orc.topp_vector(a, 2)
        vb, ib = orc.topp_vector(b, 2)
        y = orc.y_of(va, ia, vb, ib)
        sig, eps = orc.bound(K, y)
        worst = max(worst, abs(c - exact) / eps)
    assert worst < 0.1


# --------------------------------------------------------------------------- Tables II / III
def _mean_eps(orc, n, recipe, bs=32, p=2, fma_model=0):
    A = gen(recipe, n, n, 1, 0)
    B = gen(recipe, n, n, 2, 1)
    enc = orc.encode(A, B, bs, p)
    b = orc.bounds_all(n, n, n, bs, p, enc["topA"], enc["topB"], omega=3.0, t=52,
                       fma_model=fma_model)
    allv = np.concatenate([b["eps_col"].ravel(), b["eps_row"].ravel()])
    return float(allv.mean()), enc, A, B


def _golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


@pytest.mark.parametrize("n", [512, 1024, 2048])
@pytest.mark.parametrize("table", ["table2_uniform1.json", "table3_uniform100.json"])
def test_table_bound_column(orc, n, table):
    """Table II / III "AVG. A-ABFT": mean eps over all carried checksum
    elements, BS = 32, p = 2, 3 sigma, t = 52 (reading R1/R2)."""
    g = _golden(table)
    recipe = g["recipe"]
    paper = g["rows"][str(n)]["avg_aabft"]
    for fm in (0, 1):
        m, *_ = _mean_eps(orc, n, recipe, fma_model=fm)
        assert 0.95 * paper <= m <= 1.05 * paper, (n, fm, m, paper)


@pytest.mark.parametrize("n", [512, 1024])
def test_table2_rnd_error_column(orc, n):
    """Table II "AVG. Rnd. Error": mean |carried column checksum - exact|,
    sequential k accumulation, BS = 32 (reading R2/R11).  Exact via long double."""
    g = _golden("table2_uniform1.json")
    paper = g["rows"][str(n)]["avg_rnd_error"]
    A = gen("uniform", n, n, 1, 0)
    B = gen("uniform", n, n, 2, 1)
    Acs = orc.encode_cols(A, 32)
    Ccol = orc.gemm(Acs, B, fma_model=0)
    exact = np.zeros(Ccol.shape, dtype=np.longdouble)
    Al = Acs.astype(np.longdouble)
    Bl = B.astype(np.longdouble)
    for k in range(n):
        exact += np.outer(Al[:, k], Bl[k])
    err = float(np.mean(np.abs(Ccol.astype(np.longdouble) - exact)))
    assert 0.85 * paper <= err <= 1.15 * paper, (err, paper)


# --------------------------------------------------------------------------- O4 GEMM
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_gemm_integer_exact(orc, dtype):
    A = gen("integer", 24, 40, 1, 0, dtype, q=20)
    B = gen("integer", 40, 16, 2, 1, dtype, q=20)
    for fm in (0, 1):
        Cm = orc.gemm(A, B, fm)
        assert np.array_equal(Cm.astype(np.int64), A.astype(np.int64) @ B.astype(np.int64))


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_gemm_textbook_error_bound(orc, dtype):
    """|C - C_exact| <= gamma_K |A||B| (Higham [25] Thm 3.5), exact via long double."""
    A = gen("uniform", 20, 300, 1, 0, dtype)
    B = gen("uniform", 300, 12, 2, 1, dtype)
    u = np.finfo(dtype).eps / 2
    K = 300
    gamma = K * u / (1 - K * u)
    exact = A.astype(np.longdouble) @ B.astype(np.longdouble)
    absab = np.abs(A).astype(np.longdouble) @ np.abs(B).astype(np.longdouble)
    for fm in (0, 1):
        Cm = orc.gemm(A, B, fm).astype(np.longdouble)
        assert np.all(np.abs(Cm - exact) <= gamma * absab)


def test_gemm_sequential_k_order(orc):
    """Alg 3: ascending-k accumulation (a cancellation case)."""
    a = np.array([[1e16, 1.0, -1e16, 1.0]])
    b = np.ones((4, 1))
    assert orc.gemm(a, b, 0)[0, 0] == 1.0
    assert orc.gemm(a, b, 1)[0, 0] == 1.0


def test_fma_model_differs_from_separate_rounding(orc):
    """§IV-D: FMA rounds only the sum.  a*a - p with p = fl(a*a) exposes it."""
    a = 1.0 + 2.0 ** -30
    pr = a * a
    v = orc.dot_fault(np.array([a, -1.0]), np.array([a, pr]), fma_model=1)
    w = orc.dot_fault(np.array([a, -1.0]), np.array([a, pr]), fma_model=0)
    assert w == 0.0 and v == 0.0  # first step starts from c=0: fma(a,a,0)=fl(a*a)
    # order matters: accumulate -pr first, then fma(a, a, -pr) keeps the exact tail
    v = orc.dot_fault(np.array([-1.0, a]), np.array([pr, a]), fma_model=1)
    w = orc.dot_fault(np.array([-1.0, a]), np.array([pr, a]), fma_model=0)
    assert w == 0.0 and v == 2.0 ** -60


# --------------------------------------------------------------------------- O7/O8 check + correct
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_check_integer_inputs_all_rounding(orc, dtype):
    """Eq 5: with exact arithmetic carried == reference, d == 0."""
    A = gen("integer", 32, 64, 1, 0, dtype, q=10)
    B = gen("integer", 64, 32, 2, 1, dtype, q=10)
    r = orc.protected_matmul(A, B, bs=8, p=2)
    assert np.all(r["check"].d_col == 0) and np.all(r["check"].d_row == 0)
    assert np.all(r["check"].status == 0)
    assert r["check"].counts[5] == 2 * (32 // 8) * 32 and r["check"].counts[7] == 0


@pytest.mark.parametrize("recipe,dtype,M,K,bs,limit", [
    ("uniform", np.float64, 128, 128, 32, 0.2),
    ("positive", np.float64, 128, 128, 32, 0.8),
    ("wide", np.float64, 128, 128, 32, 0.2),
    ("uniform", np.float32, 128, 256, 64, 0.2),
    ("wide", np.float32, 128, 256, 64, 0.2),
    ("uniform", np.float64, 64, 16, 8, 0.8),
])
def test_clean_runs_zero_critical(orc, recipe, dtype, M, K, bs, limit):
    """Zero false positives on clean runs (north_star); margin max|d|/eps recorded."""
    worst = 0.0
    for seed in range(4):
        A = gen(recipe, M, K, seed, 0, dtype)
        B = gen(recipe, K, M, seed, 1, dtype)
        r = orc.protected_matmul(A, B, bs=bs, p=2)
        assert r["check"].counts[7] == 0
        assert np.all(r["check"].status == 0)
        worst = max(worst, r["check"].max_ratio)
    assert worst < limit


def _run_fault(orc, A, B, bs, fault):
    return orc.protected_matmul(A, B, bs=bs, p=2, faults=[fault])


@pytest.mark.parametrize("bs", [4, 8])
def test_single_fault_brute_force_integer(orc, bs):
    """Brute force on a tiny integer problem (Alg 2): every element x a spread of
    bits.  Integer data: d equals the injected error exactly, the location is exact, and
    correction restores C bit for bit.  Outside the 2x band the verdict is forced."""
    M = N = 16
    K = 32
    A = gen("integer", M, K, 3, 0, q=7)
    B = gen("integer", K, N, 4, 1, q=7)
    clean = orc.protected_matmul(A, B, bs=bs, p=2)
    Cc = clean["C"]
    b = orc.bounds_all(M, N, K, bs, 2, clean["enc"]["topA"], clean["enc"]["topB"])
    nforced = 0
    for i in range(M):
        for j in range(N):
            for bit in (0, 20, 40, 47, 51, 52, 55, 60, 62, 63):
                r = _run_fault(orc, A, B, bs, dict(row=i, col=j, site=0, xor_mask=1 << bit))
                ch = r["check"]
                I, J = i // bs, j // bs
                faulty = np.frombuffer(np.float64(Cc[i, j]).tobytes(), np.uint64)[0] ^ np.uint64(1 << bit)
                e = float(np.frombuffer(faulty.tobytes(), np.float64)[0]) - Cc[i, j]
                lo = min(b["eps_col"][I, j], b["eps_row"][i, J])
                hi = max(b["eps_col"][I, j], b["eps_row"][i, J])
                if not np.isfinite(e) or abs(e) > 2 * hi:
                    nforced += 1
                    assert ch.status[I, J] == 1, (i, j, bit)
                    assert r["C"][i, j] == Cc[i, j]
                    assert np.array_equal(r["C"], Cc)
                    assert ch.counts[2] == 1 and ch.counts[4] == 0
                elif abs(e) < 0.5 * lo:
                    assert ch.status[I, J] == 0
                    assert np.array_equal(np.delete(r["C"].ravel(), i * N + j),
                                          np.delete(Cc.ravel(), i * N + j))
                others = np.ones_like(ch.status, bool)
                others[I, J] = False
                assert np.all(ch.status[others] == 0)
    assert nforced > M * N * 5


def test_fault_in_checksum_is_checksum_only(orc):
    """A fault that hits a carried checksum trips one side only -> data untouched (R16)."""
    A = gen("integer", 16, 32, 3, 0, q=7)
    B = gen("integer", 32, 16, 4, 1, q=7)
    clean = orc.protected_matmul(A, B, bs=8, p=2)
    for f in (dict(row=16 + 1, col=5, site=2, add=1.0), dict(row=3, col=16 + 1, site=2, add=-4.0)):
        r = orc.protected_matmul(A, B, bs=8, p=2, faults=[f])
        assert np.array_equal(r["C"], clean["C"])
        st = r["check"].status
        assert (st == 2).sum() == 1 and (st != 0).sum() == 1
        assert r["check"].counts[3] == 1


def test_multiple_faults_uncorrectable(orc):
    """Two critical rows and columns in one block cannot be located (R16)."""
    A = gen("integer", 16, 32, 3, 0, q=7)
    B = gen("integer", 32, 16, 4, 1, q=7)
    r = orc.protected_matmul(A, B, bs=8, p=2, faults=[dict(row=1, col=2, site=2, add=3.0),
                                                      dict(row=4, col=6, site=2, add=5.0)])
    assert r["check"].status[0, 0] == 3 and r["check"].counts[4] == 1
    r = orc.protected_matmul(A, B, bs=8, p=2, faults=[dict(row=1, col=2, site=2, add=3.0),
                                                      dict(row=1, col=6, site=2, add=5.0)])
    assert r["check"].status[0, 0] == 3  # one row, two columns


def test_accumulator_fault_site1(orc):
    """Alg 3 errorVecAdd1: XOR into the partial sum after step k; for integer data
    the final error is exactly the XOR-induced change carried to the end (no rounding)."""
    A = gen("integer", 16, 32, 5, 0, q=5)
    B = gen("integer", 32, 16, 6, 1, q=5)
    clean = orc.protected_matmul(A, B, bs=8, p=2)
    r = orc.protected_matmul(A, B, bs=8, p=2, faults=[dict(row=9, col=3, site=1, k_step=10,
                                                           xor_mask=1 << 62)],
                             do_correct=True)
    assert r["check"].status[1, 0] == 1
    assert np.array_equal(r["C"], clean["C"])


def test_nan_inf_are_critical(orc):
    """Reading R9: CRITICAL iff !(|d| <= eps); exponent flips to Inf/NaN are detected and the
    correction recomputes from the column checksum (P:L545 '100% of exponent flips')."""
    A = gen("uniform", 32, 64, 1, 0)
    B = gen("uniform", 64, 32, 2, 1)
    clean = orc.protected_matmul(A, B, bs=8, p=2)
    for add in (np.inf, -np.inf, np.nan):
        r = orc.protected_matmul(A, B, bs=8, p=2, faults=[dict(row=5, col=9, site=2, add=add)])
        assert r["check"].status[0, 1] == 1
        assert abs(r["C"][5, 9] - clean["C"][5, 9]) <= 1e-12


@pytest.mark.parametrize("dtype", [np.float64])
def test_sign_exponent_flips_all_detected(orc, dtype):
    """'A-ABFT ... detected all faults that have been injected into the sign bit or
    the exponent' (U[-1,1], FP64).  Sampled elements of a 128^3 BS 32 problem."""
    M = 128
    A = gen("uniform", M, M, 1, 0)
    B = gen("uniform", M, M, 2, 1)
    rng = np.random.default_rng(0)
    for trial in range(24):
        i, j = (int(v) for v in rng.integers(0, M, 2))
        bit = int(rng.integers(52, 64))
        r = orc.protected_matmul(A, B, bs=32, p=2,
                                 faults=[dict(row=i, col=j, site=0, xor_mask=1 << bit)])
        assert r["check"].status[i // 32, j // 32] in (1, 3), (i, j, bit)
        assert r["check"].counts[7] >= 2
