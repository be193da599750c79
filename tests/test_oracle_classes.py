"""Pins of the oracle parts the round-1 review found unpinned (no GPU).

* The runtime three-class classification (§VI-C "rounding error / tolerable /
  critical", §I; reading R10): ROUNDING |d| <= sigma, TOLERABLE sigma < |d| <= eps,
  CRITICAL otherwise.  Integer inputs make every clean check d == 0 exactly and a fault's
  d equal to its realised error e; a small t (eps_M = 2^-t) makes sigma large
  against the rounding of the reference sums, so faults at 0.5, 2 and 4 sigma of a check
  fall in known classes.  The expected classes below come from the paper's definitions
  applied to the realised e, not from the oracle's classify().
* The non-FMA mean term (Eq 43: EV_Prod <= n/3 * 2^-2t * y; reading R7): with
  omega = 0 the bound IS that term, exactly, for K a multiple of 3 and y a power of two.
* Fault site 3 (additive accumulator fault at the errorVecAdd1 point, Alg 3 P:L528;
  reading R23): on integer data faulty - clean equals the added value exactly, for every
  k_step.
"""
import numpy as np
import pytest

import synth


def gen(recipe, r, c, seed, mid, dtype=np.float64, **kw):
    return synth.generate(recipe, r, c, seed=seed, matrix_id=mid, dtype=dtype, **kw)


def _paper_class(a, sig, eps):
    """P:L470-474 with reading R10 (the classes as the paper names them)."""
    if a <= sig:
        return 0   # "rounding error"
    if a <= eps:
        return 1   # "tolerable" (within the confidence interval, above one sigma)
    return 2       # "critical"


def class_fault_set(orc, A, B, bs, p, t, omega, rng, mults=(0.5, 2.0, 4.0)):
    """One additive final-value fault (site 2) per block at m * sigma of ONE of its two
    checks (alternating column / row check), m cycling over `mults`.  Returns the faults
    and the expected per-block report fields and global class counts, derived from the
    realised errors with the paper's class definitions."""
    M, K = A.shape
    N = B.shape[1]
    enc = orc.encode(A, B, bs, p)
    b = orc.bounds_all(M, N, K, bs, p, enc["topA"], enc["topB"], omega=omega, t=t)
    C0 = orc.gemm(A, B)
    nI, nJ = M // bs, N // bs
    faults = []
    exp = dict(status=np.zeros((nI, nJ), int), worst=np.zeros((nI, nJ), int),
               nrows=np.zeros((nI, nJ), int), ncols=np.zeros((nI, nJ), int),
               row=-np.ones((nI, nJ), int), col=-np.ones((nI, nJ), int))
    ncls = np.zeros(3, int)
    n = 0
    for I in range(nI):
        for J in range(nJ):
            i = I * bs + int(rng.integers(bs))
            j = J * bs + int(rng.integers(bs))
            m = mults[n % len(mults)]
            on_col = (n // len(mults)) % 2 == 0
            n += 1
            sc, ec = b["sig_col"][I, j], b["eps_col"][I, j]
            sr, er = b["sig_row"][i, J], b["eps_row"][i, J]
            # (1 + 2^-10): keeps |e| off the other check's class edges when the two y are
            # in an integer ratio
            add = m * (1 + 2.0 ** -10) * (sc if on_col else sr) * (1 if rng.integers(2) else -1)
            # realised error of the stored value (site 2: c + add rounded to the dtype)
            e = float(A.dtype.type(np.float64(C0[i, j]) + add)) - float(C0[i, j])
            cc, cr = _paper_class(abs(e), sc, ec), _paper_class(abs(e), sr, er)
            faults.append(dict(row=i, col=j, site=2, add=add, realised=e, cls=(cc, cr)))
            ncls[cc] += 1
            ncls[cr] += 1
            exp["worst"][I, J] = max(cc, cr)
            exp["ncols"][I, J] = int(cc == 2)
            exp["nrows"][I, J] = int(cr == 2)
            if cc == 2 and cr == 2:
                exp["status"][I, J] = 4
                exp["row"][I, J], exp["col"][I, J] = i, j
            elif cc == 2 or cr == 2:
                exp["status"][I, J] = 2
    total = nI * N + M * nJ
    ncls[0] += total - 2 * nI * nJ  # every other check: d == 0 exactly (Eq 5)
    return faults, exp, ncls


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_three_classes_exact(orc, dtype):
    """ROUNDING / TOLERABLE / CRITICAL counts, worst class, bad row/column counts and the
    located element of every block equal the paper's definitions on realised errors."""
    M, N, K, bs, p = 64, 96, 48, 8, 2
    t, omega = (20, 3.0) if dtype == np.float64 else (10, 3.0)
    A = gen("integer", M, K, 7, 0, dtype, q=5)
    B = gen("integer", K, N, 7, 1, dtype, q=5)
    rng = np.random.default_rng(3)
    faults, exp, ncls = class_fault_set(orc, A, B, bs, p, t, omega, rng)
    assert ncls[1] > 20 and ncls[2] > 20  # both non-trivial classes are exercised
    clean = orc.gemm(A, B)
    r = orc.protected_matmul(A, B, bs=bs, p=p, omega=omega, t=t, faults=faults,
                             do_correct=False)
    ch = r["check"]
    assert ch.counts[5:8].tolist() == ncls.tolist()
    for k, name in (("worst", "worst"), ("nrows", "nrows"), ("ncols", "ncols"),
                    ("status", "status"), ("row", "row"), ("col", "col")):
        assert np.array_equal(getattr(ch, name), exp[k]), k
    # the max ratio of a block is its fault's |e| / eps of the tripped check (exact d)
    for f in faults:
        I, J = f["row"] // bs, f["col"] // bs
        assert ch.ratio[I, J] > 0
    # correction: every located block is restored exactly (integer data)
    r2 = orc.protected_matmul(A, B, bs=bs, p=p, omega=omega, t=t, faults=faults)
    st = r2["check"].status
    assert np.all(st[exp["status"] == 4] == 1)
    fixed = exp["status"] == 4
    for f in faults:
        I, J = f["row"] // bs, f["col"] // bs
        if fixed[I, J]:
            assert r2["C"][f["row"], f["col"]] == clean[f["row"], f["col"]]
    assert r2["check"].counts[2] == int(fixed.sum())


def test_tolerable_is_not_rounding_nor_critical(orc):
    """A single check at 2 sigma (< eps = 3 sigma) is TOLERABLE: the block stays CLEAN (only
    CRITICAL triggers locate/correct, reading R10) but its worst class is 1."""
    M = N = 16
    K, bs, t = 32, 8, 20
    A = gen("integer", M, K, 2, 0, q=3)
    B = gen("integer", K, N, 2, 1, q=3)
    enc = orc.encode(A, B, bs, 2)
    b = orc.bounds_all(M, N, K, bs, 2, enc["topA"], enc["topB"], t=t)
    # an element whose two sigmas are within 2x, so 1.2 * the larger is above both sigmas
    # and below both eps = 3 sigma
    cand = [(i, j) for i in range(bs) for j in range(bs)
            if max(b["sig_col"][0, j], b["sig_row"][i, 0])
            < 1.9 * min(b["sig_col"][0, j], b["sig_row"][i, 0])]
    i, j = cand[0]
    s_max = max(b["sig_col"][0, j], b["sig_row"][i, 0])
    add = 1.2 * s_max
    assert add < min(b["eps_col"][0, j], b["eps_row"][i, 0])
    r = orc.protected_matmul(A, B, bs=bs, p=2, t=t, faults=[dict(row=i, col=j, site=2, add=add)])
    ch = r["check"]
    assert ch.status[0, 0] == 0 and ch.worst[0, 0] == 1
    assert ch.counts[6] == 2 and ch.counts[7] == 0


@pytest.mark.parametrize("K", [3, 48, 3 * 1024])
@pytest.mark.parametrize("y", [1.0, 0.25, 2.0 ** 10])
@pytest.mark.parametrize("t", [10, 23, 52])
def test_ev_term_closed_form(orc, K, y, t):
    """Eq 43: EV_Prod <= n/3 * 2^-2t * y.  With omega = 0 the non-FMA bound is that
    term alone (exact: K/3 an integer, y a power of two); the FMA model has no mean term
    (Eq 27), so its bound is 0."""
    sig0, eps0 = orc.bound(K, y, fma_model=0, t=t, omega=0.0)
    assert eps0 == (K // 3) * y * 2.0 ** (-2 * t)
    sig1, eps1 = orc.bound(K, y, fma_model=1, t=t, omega=0.0)
    assert eps1 == 0.0


def test_ev_term_adds_to_omega_sigma(orc):
    """eps = omega sigma + |EV| (Eq 7 with Eq 43); small t makes the mean term visible."""
    K, y, t = 3000, 4.0, 8
    sig, eps = orc.bound(K, y, fma_model=0, t=t, omega=3.0)
    ev = K / 3 * 2.0 ** (-2 * t) * y
    assert ev > 1e-6 * eps
    assert (eps - 3.0 * sig) == pytest.approx(ev, rel=1e-9)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("k_step", [0, 17, 63])
@pytest.mark.parametrize("add", [5.0, -3.0, 1024.0])
def test_site3_additive_accumulator_exact(orc, dtype, k_step, add):
    """Alg 3 errorVecAdd1 point, additive variant (site 3): integer data, so every
    later accumulation step is exact and faulty - clean == add for C, Ccol and Crow
    elements alike."""
    M, N, K, bs = 16, 16, 64, 8
    A = gen("integer", M, K, 4, 0, dtype, q=6)
    B = gen("integer", K, N, 4, 1, dtype, q=6)
    clean = orc.protected_matmul(A, B, bs=bs, p=2, do_correct=False)
    for (r_, c_), key in (((3, 9), "C"), ((M + 1, 4), "Ccol"), ((5, N + 1), "Crow")):
        f = dict(row=r_, col=c_, site=3, k_step=k_step, add=add)
        r = orc.protected_matmul(A, B, bs=bs, p=2, faults=[f], do_correct=False)
        rr = r_ - M if key == "Ccol" else r_
        cc = c_ - N if key == "Crow" else c_
        assert float(r[key][rr, cc]) - float(clean[key][rr, cc]) == add
        diff = r[key] != clean[key]
        assert diff.sum() == 1


def test_site3_k_step_beyond_end_is_noop(orc):
    """A k_step outside [0, K) never fires (the fault point does not exist)."""
    A = gen("integer", 8, 16, 4, 0, q=6)
    B = gen("integer", 16, 8, 4, 1, q=6)
    c = orc.dot_fault(A[0], np.ascontiguousarray(B[:, 0]), site=3, k_step=16, add=7.0)
    assert c == float(A[0] @ B[:, 0])


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("k_step", [0, 5, 30, 31])
def test_site1_xor_point_exact(orc, dtype, k_step):
    """Alg 3 errorVecAdd1: the XOR hits the partial sum right AFTER step k_step.
    A sign-bit flip on integer data turns s_k into -s_k exactly, so the faulty result is
    -(sum_{k' <= k_step} a b) + sum_{k' > k_step} a b, computed here in integers."""
    K = 32
    a = gen("integer", 1, K, 9, 0, dtype, q=9)[0]
    b = gen("integer", K, 1, 9, 1, dtype, q=9)[:, 0].copy()
    ai, bi = a.astype(np.int64), b.astype(np.int64)
    head = int((ai[:k_step + 1] * bi[:k_step + 1]).sum())
    tail = int((ai[k_step + 1:] * bi[k_step + 1:]).sum())
    sign = 1 << (63 if dtype == np.float64 else 31)
    c = orc.dot_fault(a, b, site=1, k_step=k_step, xor_mask=sign)
    assert c == float(-head + tail)
