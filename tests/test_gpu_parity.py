"""GPU parity: the sm_100a path (through the C ABI) against the CPU oracle, element by element.

Bars (north_star / SURVEY §8(c)):
  * Acs, Bcs, top-p values and indices, eps/sigma: bit-identical (sequential encode order).
  * C, Ccol, Crow: |gpu - oracle| / (|A||B|) <= 1e-13 (FP64, DMMA order differs from the
    sequential oracle) ; FP32 FFMA accumulates in the oracle's order -> bit-identical.
  * Clean runs: zero CRITICAL, identical block verdicts.
  * Faults outside 2x the bound: identical verdicts; located and corrected.
"""
import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TD = {np.float64: torch.float64, np.float32: torch.float32}


@pytest.fixture(scope="module")
def P():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_dsn_braunhw14_b200 import api
    return api


def gen(recipe, r, c, seed, mid, dtype=np.float64, **kw):
    return synth.generate(recipe, r, c, seed=seed, matrix_id=mid, dtype=dtype, **kw)


def to_dev(X):
    """Row-major device copy whose pitch is a multiple of 16 bytes (ABI alignment rule)."""
    X = np.ascontiguousarray(X)
    r, c = X.shape
    q = 16 // X.itemsize
    ld = (c + q - 1) // q * q
    buf = torch.zeros(r, ld, dtype=TD[X.dtype.type], device="cuda")
    buf[:, :c] = torch.from_numpy(X).cuda()
    return buf[:, :c]


def host(t):
    return t.detach().cpu().numpy()


def norm_err(G, O, A, B):
    denom = np.abs(A).astype(np.float64) @ np.abs(B).astype(np.float64)
    denom[denom == 0] = 1.0
    return float(np.max(np.abs(G.astype(np.float64) - O.astype(np.float64)) / denom))


def xor_val(v, mask, dtype):
    ut = np.uint64 if dtype == np.float64 else np.uint32
    a = np.array([v], dtype=dtype).view(ut) ^ ut(mask)
    with np.errstate(all="ignore"):
        return float(a.view(dtype)[0])


def run_both(P, orc, M, N, K, bs, p, dtype=np.float64, recipe="uniform", faults=(), seed=1,
             correct=True, q=8, fused=True):
    A = gen(recipe, M, K, seed, 0, dtype, q=q)
    B = gen(recipe, K, N, seed, 1, dtype, q=q)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=p, fused=fused)
    res = plan.run(to_dev(A), to_dev(B), faults=list(faults), correct=correct)
    torch.cuda.synchronize()
    o = orc.protected_matmul(A, B, bs=bs, p=p, faults=list(faults), do_correct=correct)
    return A, B, plan, res, o


SHAPES = [
    # M, N, K, bs, p  (ragged: not multiples of the 128 tiles / 16-deep k-tiles)
    (128, 128, 128, 32, 2),
    (192, 320, 200, 64, 2),
    (64, 96, 37, 8, 3),
    (256, 256, 300, 256, 1),
    (8, 8, 16, 8, 8),
    (384, 128, 1000, 128, 4),
]


ENCODE_SHAPES = SHAPES + [
    (512, 768, 2048, 64, 2),   # many 128-column chunks of A, several k-chunks of B, p = 2
    (256, 256, 4099, 32, 3),   # ragged last chunk with an odd K
]


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("shape", ENCODE_SHAPES)
def test_encode_bit_exact(P, orc, dtype, shape):
    M, N, K, bs, p = shape
    A = gen("uniform", M, K, 3, 0, dtype)
    B = gen("wide", K, N, 3, 1, dtype)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=p)
    plan.encode(to_dev(A), to_dev(B))
    torch.cuda.synchronize()
    enc = orc.encode(A, B, bs, p)
    assert np.array_equal(host(plan.Acs), enc["Acs"])
    assert np.array_equal(host(plan.Bcs), enc["Bcs"])
    assert np.array_equal(host(plan.topA_val), enc["topA"][0])
    assert np.array_equal(host(plan.topA_idx), enc["topA"][1])
    assert np.array_equal(host(plan.topB_val), enc["topB"][0])
    assert np.array_equal(host(plan.topB_idx), enc["topB"][1])


TOPP_GEMM_SHAPES = ENCODE_SHAPES + [
    (1024, 1024, 2048, 64, 2),  # data-parallel waves + stream-K split tiles (partial lists)
    (704, 1216, 777, 32, 4),    # ragged K tail inside a k-tile, p = 4
    (2048, 128, 4096, 64, 1),   # long K: many k-tiles per segment
]


@pytest.mark.parametrize("faults", [False, True])
@pytest.mark.parametrize("shape", TOPP_GEMM_SHAPES)
def test_topp_in_gemm_bit_exact(P, orc, shape, faults):
    """AABFT_FLAG_TOPP_IN_GEMM: the top-p tables selected by the GEMM's producer warp from the
    operand tiles (P:L320 'in parallel to the matrix multiplication') equal the oracle's
    sequential scan bit for bit -- values and indices, data and checksum vectors -- including
    stream-K split tiles whose partial lists are merged by the tile owner, and in the fault
    instantiation of the kernel."""
    M, N, K, bs, p = shape
    A = gen("uniform", M, K, 5, 0)
    B = gen("wide", K, N, 5, 1)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p, topp_in_gemm=True)
    fl = [dict(row=1, col=1, site=2, add=1.0)] if faults else None
    plan.topA_val.fill_(-7.0)  # stale contents must be overwritten
    plan.topB_idx.fill_(-7)
    plan.run(to_dev(A), to_dev(B), faults=fl)
    torch.cuda.synchronize()
    enc = orc.encode(A, B, bs, p)
    assert np.array_equal(host(plan.Acs), enc["Acs"])
    assert np.array_equal(host(plan.Bcs), enc["Bcs"])
    assert np.array_equal(host(plan.topA_val), enc["topA"][0])
    assert np.array_equal(host(plan.topA_idx), enc["topA"][1])
    assert np.array_equal(host(plan.topB_val), enc["topB"][0])
    assert np.array_equal(host(plan.topB_idx), enc["topB"][1])


def test_topp_in_gemm_ties_integer_data(P, orc):
    """Many equal |values| (integer data): the GEMM-side selection keeps the lowest index."""
    M, N, K, bs, p = 256, 320, 900, 32, 4
    A = gen("integer", M, K, 6, 0, q=2)
    B = gen("integer", K, N, 6, 1, q=2)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p, topp_in_gemm=True)
    plan.run(to_dev(A), to_dev(B))
    torch.cuda.synchronize()
    enc = orc.encode(A, B, bs, p)
    assert np.array_equal(host(plan.topA_idx), enc["topA"][1])
    assert np.array_equal(host(plan.topB_idx), enc["topB"][1])
    assert np.array_equal(host(plan.topA_val), enc["topA"][0])
    assert np.array_equal(host(plan.topB_val), enc["topB"][0])


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_encode_ties_integer_data(P, orc, dtype):
    """Many equal |values|: the tie rule (lowest index) must match exactly."""
    M, N, K, bs, p = 64, 64, 300, 16, 4
    A = gen("integer", M, K, 5, 0, dtype, q=2)
    B = gen("integer", K, N, 5, 1, dtype, q=2)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=p)
    plan.encode(to_dev(A), to_dev(B))
    torch.cuda.synchronize()
    enc = orc.encode(A, B, bs, p)
    assert np.array_equal(host(plan.topA_idx), enc["topA"][1])
    assert np.array_equal(host(plan.topB_idx), enc["topB"][1])
    assert np.array_equal(host(plan.topA_val), enc["topA"][0])


@pytest.mark.parametrize("fma_model", [1, 0])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_bound_bit_exact(P, orc, dtype, fma_model):
    M, N, K, bs, p = 192, 256, 333, 64, 2
    A = gen("uniform100", M, K, 4, 0, dtype)
    B = gen("uniform", K, N, 4, 1, dtype)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=p, fma_model=fma_model)
    plan.encode(to_dev(A), to_dev(B))
    b = plan.bound()
    torch.cuda.synchronize()
    enc = orc.encode(A, B, bs, p)
    o = orc.bounds_all(M, N, K, bs, p, enc["topA"], enc["topB"], t=orc.default_t(dtype),
                       fma_model=fma_model)
    for k in ("eps_col", "sig_col", "eps_row", "sig_row"):
        assert np.array_equal(host(b[k]), o[k]), k


@pytest.mark.parametrize("shape", SHAPES)
def test_gemm_parity_f64(P, orc, shape):
    M, N, K, bs, p = shape
    A, B, plan, res, o = run_both(P, orc, M, N, K, bs, p)
    enc = o["enc"]
    assert norm_err(host(res.C), o["C"], A, B) <= 1e-13
    assert norm_err(host(res.Ccol), o["Ccol"], enc["Acs"], B) <= 1e-13
    assert norm_err(host(res.Crow), o["Crow"], A, enc["Bcs"]) <= 1e-13


@pytest.mark.parametrize("shape", SHAPES)
def test_gemm_parity_f32_bit_exact(P, orc, shape):
    M, N, K, bs, p = shape
    A, B, plan, res, o = run_both(P, orc, M, N, K, bs, p, dtype=np.float32, recipe="wide")
    enc = o["enc"]
    assert norm_err(host(res.C), o["C"], A, B) <= 1e-5
    assert np.array_equal(host(res.C), o["C"])
    assert np.array_equal(host(res.Ccol), o["Ccol"])
    assert np.array_equal(host(res.Crow), o["Crow"])


def test_gemm_plain_same_family(P, orc):
    M, N, K = 256, 384, 520
    for dtype in (np.float64, np.float32):
        A = gen("uniform", M, K, 9, 0, dtype)
        B = gen("uniform", K, N, 9, 1, dtype)
        plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=64, p=2)
        dA, dB = to_dev(A), to_dev(B)
        plan.run(dA, dB)
        Cp = P.gemm_plain(dA, dB)
        torch.cuda.synchronize()
        # same kernel family; the stream-K split of the ragged tail may differ between the
        # two launches (different tile sets), so compare by tolerance, not bits
        assert norm_err(host(Cp), host(plan.C), A, B) <= (1e-13 if dtype == np.float64 else 0)
        assert norm_err(host(Cp), orc.gemm(A, B), A, B) <= (1e-13 if dtype == np.float64 else 1e-5)


@pytest.mark.parametrize("fused", [True, False])
@pytest.mark.parametrize("dtype,recipe", [(np.float64, "uniform"), (np.float64, "positive"),
                                          (np.float64, "wide"), (np.float32, "uniform"),
                                          (np.float32, "wide"), (np.float64, "integer")])
def test_clean_run_verdicts(P, orc, dtype, recipe, fused):
    M, N, K, bs, p = 256, 192, 512, 64, 2
    A, B, plan, res, o = run_both(P, orc, M, N, K, bs, p, dtype=dtype, recipe=recipe, fused=fused)
    rep = res.reports()
    cnt = res.counts()
    assert cnt["checks_critical"] == 0 and o["check"].counts[7] == 0
    assert np.all(rep["status"] == 0)
    assert np.array_equal(rep["status"], o["check"].status)
    assert cnt["blocks"] == (M // bs) * (N // bs) == cnt["clean"]
    assert cnt["checks_rounding"] + cnt["checks_tolerable"] == (M // bs) * N + M * (N // bs)
    assert cnt["max_ratio"] < 0.9
    # every report field and class counter.  A clean check whose |d| lies near sigma (U[0,1)
    # data: clean |d| reaches ~1.3 sigma) may be ROUNDING on one side and TOLERABLE on the
    # other -- the GPU sums in another order (reading R11) -- so the worst class is compared
    # on blocks without such a check and the class counters up to their number
    amb_blk, n_amb = ambiguous_checks(orc, A, B, o, bs, p)
    assert_reports_equal(rep, o["check"], mask=~amb_blk)
    assert_reports_equal(rep, o["check"], fields=("status", "n_bad_rows", "n_bad_cols", "row", "col"))
    got = np.array([cnt["checks_rounding"], cnt["checks_tolerable"], cnt["checks_critical"]])
    assert np.all(np.abs(got - o["check"].counts[5:8]) <= n_amb), (got, o["check"].counts, n_amb)
    if recipe != "positive":
        assert n_amb == 0
    if recipe == "integer":
        assert cnt["max_ratio"] == 0.0 and cnt["checks_rounding"] == o["check"].counts[5]


REPORT_FIELDS = {"status": "status", "worst_class": "worst", "n_bad_rows": "nrows",
                 "n_bad_cols": "ncols", "row": "row", "col": "col"}


def ambiguous_checks(orc, A, B, o, bs, p, band=(0.7, 1.45)):
    """Checks whose oracle |d| sits within `band` of sigma or eps (class edges where the
    GPU's summation order may decide differently).  Returns (per-block mask, count)."""
    M, K = A.shape
    N = B.shape[1]
    enc = o["enc"]
    b = orc.bounds_all(M, N, K, bs, p, enc["topA"], enc["topB"], t=orc.default_t(A.dtype))
    och = o["check"]
    amb_c = np.zeros(och.d_col.shape, bool)
    amb_r = np.zeros(och.d_row.shape, bool)
    for d, am, sg, ep in ((och.d_col, amb_c, b["sig_col"], b["eps_col"]),
                          (och.d_row, amb_r, b["sig_row"], b["eps_row"])):
        with np.errstate(divide="ignore", invalid="ignore"):
            for edge in (sg, ep):
                q = np.abs(d) / edge
                am |= (q >= band[0]) & (q <= band[1])
    nI, nJ = M // bs, N // bs
    blk = amb_c.reshape(nI, nJ, bs).any(axis=2) | amb_r.reshape(nI, bs, nJ).any(axis=1)
    return blk, int(amb_c.sum() + amb_r.sum())


def assert_reports_equal(rep, och, mask=None, ratio=False, fields=tuple(REPORT_FIELDS)):
    """Block reports GPU vs oracle, field by field (status, worst class, bad row / column
    counts, located element; optionally max |d|/eps to float precision)."""
    m = np.ones(rep.shape, bool) if mask is None else mask
    for g in fields:
        o = REPORT_FIELDS[g]
        gv, ov = rep[g][m].astype(np.int64), getattr(och, o)[m].astype(np.int64)
        assert np.array_equal(gv, ov), (g, np.argwhere(m)[np.flatnonzero(gv != ov)][:5],
                                        gv[gv != ov][:5], ov[gv != ov][:5])
    if ratio:
        gr, orr = rep["max_ratio"][m].astype(np.float64), och.ratio[m]
        fin = np.isfinite(orr)
        assert np.array_equal(np.isfinite(gr), fin)
        assert np.allclose(gr[fin], orr[fin], rtol=2e-6, atol=0), np.max(np.abs(gr[fin] / orr[fin] - 1))


@pytest.mark.parametrize("dtype,fused,bs", [(np.float64, True, 8), (np.float64, True, 16),
                                            (np.float64, True, 32), (np.float64, True, 64),
                                            (np.float64, False, 64), (np.float64, False, 128),
                                            (np.float32, False, 8), (np.float32, False, 64)])
def test_three_classes_every_field(P, orc, dtype, fused, bs):
    """The runtime classes (reading R10) at block granularity: integer data and a
    small t make d equal the realised fault error, faults at 0.5 / 2 / 4 sigma of one check
    per block give ROUNDING, TOLERABLE and CRITICAL checks; every report field, the three
    class counters and the per-block max |d|/eps must equal the oracle's, and the expected
    values (paper definitions on realised errors, tests/test_oracle_classes.py) too."""
    from test_oracle_classes import class_fault_set
    M, N, K, p = 256, 384, 96, 2
    t = 20 if dtype == np.float64 else 10
    A = gen("integer", M, K, 17, 0, dtype, q=5)
    B = gen("integer", K, N, 17, 1, dtype, q=5)
    faults, exp, ncls = class_fault_set(orc, A, B, bs, p, t, 3.0, np.random.default_rng(bs))
    assert ncls[1] > 0 and ncls[2] > 0
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=p, t=t, fused=fused)
    fl = [dict(row=f["row"], col=f["col"], site=2, add=f["add"]) for f in faults]
    res = plan.run(to_dev(A), to_dev(B), faults=fl, correct=False)
    torch.cuda.synchronize()
    rep, cnt = res.reports(), res.counts()
    o = orc.protected_matmul(A, B, bs=bs, p=p, t=t, faults=fl, do_correct=False)
    assert_reports_equal(rep, o["check"], ratio=True)
    for g, k in (("status", "status"), ("worst_class", "worst"), ("n_bad_rows", "nrows"),
                 ("n_bad_cols", "ncols"), ("row", "row"), ("col", "col")):
        assert np.array_equal(rep[g].astype(np.int64), exp[k]), g
    got = [cnt["checks_rounding"], cnt["checks_tolerable"], cnt["checks_critical"]]
    assert got == o["check"].counts[5:8].tolist() == ncls.tolist()
    for k, name in enumerate(("blocks", "clean", "corrected", "checksum_only", "uncorrectable")):
        assert cnt[name] == o["check"].counts[k], name
    assert cnt["max_ratio"] == pytest.approx(o["check"].max_ratio, rel=2e-6)
    # correction of the located blocks (CORRECTED count and exact restoration)
    res = plan.run(to_dev(A), to_dev(B), faults=fl, correct=True)
    torch.cuda.synchronize()
    o2 = orc.protected_matmul(A, B, bs=bs, p=p, t=t, faults=fl, do_correct=True)
    assert np.array_equal(res.reports()["status"].astype(np.int64), o2["check"].status)
    assert res.counts()["corrected"] == o2["check"].counts[2] == int((exp["status"] == 4).sum())
    assert np.array_equal(host(res.C), o2["C"])


def _fault_set(orc, A, B, bs, p, rng, dtype, n_per_mag=1):
    """One fault per block: additive magnitudes r * max(eps_col, eps_row) across the band and
    exponent/sign XOR flips."""
    M, K = A.shape
    N = B.shape[1]
    enc = orc.encode(A, B, bs, p)
    b = orc.bounds_all(M, N, K, bs, p, enc["topA"], enc["topB"], t=orc.default_t(dtype))
    faults, labels = [], []
    mags = [2.0 ** -8, 2.0 ** -4, 2.0 ** -2, 2.0 ** 2, 2.0 ** 5, 2.0 ** 12]
    nI, nJ = M // bs, N // bs
    n = 0
    for I in range(nI):
        for J in range(nJ):
            i = I * bs + int(rng.integers(bs))
            j = J * bs + int(rng.integers(bs))
            lo = min(b["eps_col"][I, j], b["eps_row"][i, J])
            hi = max(b["eps_col"][I, j], b["eps_row"][i, J])
            kind = n % 8
            n += 1
            if kind < len(mags):
                r = mags[kind] * (1 if rng.integers(2) else -1)
                add = float(r * hi)
                faults.append(dict(row=i, col=j, site=2, add=add))
                labels.append("detect" if abs(add) > 2 * hi else ("silent" if abs(add) < 0.5 * lo else "band"))
            elif kind == 6:
                bit = 63 if dtype == np.float64 else 31
                faults.append(dict(row=i, col=j, site=0, xor_mask=1 << bit))
                labels.append(("xor", lo, hi))
            else:
                bit = int(rng.integers(52, 63)) if dtype == np.float64 else int(rng.integers(23, 31))
                faults.append(dict(row=i, col=j, site=0, xor_mask=1 << bit))
                labels.append(("xor", lo, hi))
    return faults, labels


@pytest.mark.parametrize("dtype,fused,bs", [(np.float64, True, 64), (np.float64, False, 64),
                                            (np.float64, True, 32), (np.float64, True, 16),
                                            (np.float64, True, 8), (np.float32, False, 64),
                                            (np.float32, True, 64), (np.float32, True, 8),
                                            (np.float32, True, 128),
                                            # unfused streaming check: many / one / wide blocks
                                            (np.float32, False, 8), (np.float32, False, 128),
                                            (np.float64, False, 128), (np.float64, False, 256)])
def test_fault_verdicts_outside_band(P, orc, dtype, fused, bs):
    M, N, K, p = 512, 512, 256, 2
    rng = np.random.default_rng(42)
    A = gen("uniform", M, K, 11, 0, dtype)
    B = gen("uniform", K, N, 11, 1, dtype)
    faults, labels = _fault_set(orc, A, B, bs, p, rng, dtype)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=p, fused=fused)
    assert plan.fused == (fused and (bs <= 64 if dtype == np.float64 else bs <= 128))
    dA, dB = to_dev(A), to_dev(B)
    clean = host(plan.run(dA, dB).C).copy()
    res = plan.run(dA, dB, faults=faults)
    torch.cuda.synchronize()
    rep = res.reports()
    o = orc.protected_matmul(A, B, bs=bs, p=p, faults=faults)
    ost = o["check"].status
    Cg = host(res.C)
    nchk = 0
    nonband = np.zeros(ost.shape, bool)
    for f, lab in zip(faults, labels):
        I, J = f["row"] // bs, f["col"] // bs
        g, og = rep["status"][I, J], ost[I, J]
        clean_v = clean[f["row"], f["col"]]
        if lab == "detect":
            assert g == 1 and og == 1, (f, g, og)
        elif lab == "silent":
            assert g == 0 and og == 0, (f, g, og)
        elif isinstance(lab, tuple):  # bit flip: realised e against the band (reading R22)
            e = abs(xor_val(clean_v, f["xor_mask"], dtype) - clean_v)
            _, lo, hi = lab
            if not np.isfinite(e) or e > 2 * hi:
                assert g == 1 and og == 1, (f, g, og)
                lab = "detect"
            elif e < 0.5 * lo:
                assert g == 0 and og == 0, (f, g, og)
                lab = "silent"
            else:
                lab = "band"
        if g == 1:
            tol = 1e-12 if dtype == np.float64 else 1e-3
            assert abs(Cg[f["row"], f["col"]] - clean_v) <= tol * max(1.0, abs(clean_v))
        if lab != "band":
            assert g == og, (f, lab, g, og)
            nchk += 1
            nonband[I, J] = True
    assert nchk > len(faults) // 2
    # located element and bad row / column counts of every non-band block (their worst class
    # may sit at the sigma edge for a 'silent' fault, so it is compared where the fault is
    # critical: then every side is CRITICAL)
    och = o["check"]
    for fld, ofld in (("n_bad_rows", "nrows"), ("n_bad_cols", "ncols"), ("row", "row"),
                      ("col", "col")):
        assert np.array_equal(rep[fld][nonband].astype(np.int64),
                              getattr(och, ofld)[nonband].astype(np.int64)), fld
    crit = nonband & (ost != 0)
    assert np.array_equal(rep["worst_class"][crit], och.worst[crit])
    # untouched elements are bit-identical to the clean run
    mask = np.ones_like(Cg, bool)
    for f in faults:
        mask[f["row"], f["col"]] = False
    assert np.array_equal(Cg[mask], clean[mask])


def test_accumulator_fault_site1(P, orc):
    M, N, K, bs, p = 256, 256, 512, 64, 2
    A = gen("uniform", M, K, 12, 0)
    B = gen("uniform", K, N, 12, 1)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p)
    dA, dB = to_dev(A), to_dev(B)
    clean = host(plan.run(dA, dB).C).copy()
    faults = [dict(row=70, col=130, site=1, k_step=200, xor_mask=1 << 61),
              dict(row=5, col=7, site=1, k_step=0, xor_mask=1 << 62),
              dict(row=200, col=250, site=1, k_step=511, xor_mask=1 << 63)]
    res = plan.run(dA, dB, faults=faults)
    torch.cuda.synchronize()
    rep = res.reports()
    for f in faults:
        assert rep["status"][f["row"] // bs, f["col"] // bs] == 1
    assert np.allclose(host(res.C), clean, rtol=0, atol=1e-12)


def test_checksum_faults_checksum_only(P, orc):
    M, N, K, bs, p = 256, 256, 256, 64, 2
    A = gen("uniform", M, K, 13, 0)
    B = gen("uniform", K, N, 13, 1)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p)
    dA, dB = to_dev(A), to_dev(B)
    clean = host(plan.run(dA, dB).C).copy()
    faults = [dict(row=M + 1, col=100, site=2, add=1.0),      # Ccol row 1
              dict(row=10, col=N + 2, site=0, xor_mask=1 << 62)]  # Crow col 2
    res = plan.run(dA, dB, faults=faults)
    torch.cuda.synchronize()
    rep = res.reports()
    assert rep["status"][1, 100 // bs] == 2 and rep["status"][0, 2] == 2
    assert res.counts()["checksum_only"] == 2
    assert np.array_equal(host(res.C), clean)


def test_multi_fault_block_uncorrectable(P, orc):
    M, N, K, bs, p = 128, 128, 128, 64, 2
    A = gen("uniform", M, K, 14, 0)
    B = gen("uniform", K, N, 14, 1)
    faults = [dict(row=3, col=4, site=2, add=5.0), dict(row=9, col=20, site=2, add=-3.0)]
    A_, B_, plan, res, o = run_both(P, orc, M, N, K, bs, p, faults=faults, seed=14)
    rep = res.reports()
    assert rep["status"][0, 0] == 3 == o["check"].status[0, 0]
    assert res.counts()["uncorrectable"] == 1


@pytest.mark.parametrize("M,N,K,bs", [(256, 128, 200, 64), (1024, 1024, 256, 64),
                                     (1088, 1216, 130, 64), (1024, 2048, 64, 32)])
def test_host_entry_point_e2e(P, orc, M, N, K, bs):
    """aabft_protected_gemm_host: host buffers in, corrected C + counts out (pipelined S x S
    blocks with overlapped copies when M, N are large enough)."""
    import ctypes as C
    from paper_conf_dsn_braunhw14_b200 import _abi
    A = gen("uniform", M, K, 15, 0)
    B = gen("uniform", K, N, 15, 1)
    cfg = _abi.Config(0, bs, M, N, K, 2, 0, 3.0, 1, 0)
    L = _abi.lib()
    nbytes = L.aabft_host_arena_bytes(C.byref(cfg))
    arena = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    Ch = np.zeros((M, N))
    cnt = _abi.Counts()
    st = L.aabft_protected_gemm_host(C.byref(cfg), A.ctypes.data, B.ctypes.data, Ch.ctypes.data,
                                     C.addressof(cnt), arena.data_ptr(), nbytes,
                                     torch.cuda.current_stream().cuda_stream)
    _abi.ok(st, "aabft_protected_gemm_host")
    assert norm_err(Ch, orc.gemm(A, B), A, B) <= 1e-13
    assert cnt.n[0] == (M // bs) * (N // bs) == cnt.n[1] and cnt.n[7] == 0


def test_full_size_c2_sampled(P, orc):
    """BASELINE configs[1]: 4096^3 FP64, BS 64, the bench launch configuration.  The oracle
    checks sampled rows / columns / blocks one by one."""
    M = N = K = 4096
    bs, p = 64, 2
    A = gen("uniform", M, K, 1, 0)
    B = gen("uniform", K, N, 2, 1)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p)
    res = plan.run(to_dev(A), to_dev(B))
    torch.cuda.synchronize()
    cnt = res.counts()
    assert cnt["blocks"] == 4096 and cnt["clean"] == 4096 and cnt["checks_critical"] == 0
    assert cnt["max_ratio"] < 0.5
    rng = np.random.default_rng(0)
    tav, tai = host(plan.topA_val), host(plan.topA_idx)
    tbv, tbi = host(plan.topB_val), host(plan.topB_idx)
    Acs, Bcs, C = host(plan.Acs), host(plan.Bcs), host(res.C)
    for i in rng.integers(0, M, 16):
        v, ix = orc.topp_vector(A[i], p)
        assert np.array_equal(tav[i], v) and np.array_equal(tai[i], ix)
    for j in rng.integers(0, N, 16):
        v, ix = orc.topp_vector(np.ascontiguousarray(B[:, j]), p)
        assert np.array_equal(tbv[j], v) and np.array_equal(tbi[j], ix)
    rows = rng.integers(0, M, 8)
    assert norm_err(C[rows], orc.gemm(A[rows], B), A[rows], B) <= 1e-13
    for (I, J) in [(0, 0), (63, 63), (17, 42), (40, 3)]:
        Ab = A[I * bs:(I + 1) * bs]
        Bb = np.ascontiguousarray(B[:, J * bs:(J + 1) * bs])
        ob = orc.protected_matmul(Ab, Bb, bs=bs, p=p)
        assert np.array_equal(Acs[I], ob["enc"]["Acs"][0])
        assert np.array_equal(Bcs[:, J], ob["enc"]["Bcs"][:, 0])
        assert np.array_equal(tav[M + I], ob["enc"]["topA"][0][bs])
        assert np.array_equal(tbv[N + J], ob["enc"]["topB"][0][bs])
        assert ob["check"].status[0, 0] == res.reports()["status"][I, J] == 0
        assert norm_err(C[I * bs:(I + 1) * bs, J * bs:(J + 1) * bs], ob["C"], Ab, Bb) <= 1e-13


@pytest.mark.parametrize("cfg", [
    # BASELINE configs[2]: 8192^2 FP32 FFMA, wide exponents, BS 64 (bench --workload c3)
    dict(name="c3", M=8192, N=8192, K=8192, dtype=np.float32, recipe="wide", tol=None),
    # BASELINE configs[4]: M=N=8192, K=65536 FP64, BS 64 (bench --workload c5 at one GPU)
    dict(name="c5", M=8192, N=8192, K=65536, dtype=np.float64, recipe="uniform", tol=1e-13),
], ids=lambda c: c["name"])
def test_full_size_sampled(P, orc, cfg):
    """Full-size parity in the bench launch configuration: clean verdicts everywhere, and the
    oracle recomputes sampled top-p vectors, rows of C and whole BS x BS blocks one by one.
    FP32 (FFMA, ascending k) is bit-identical; FP64 within 1e-13 of |A||B|."""
    M, N, K, dt = cfg["M"], cfg["N"], cfg["K"], cfg["dtype"]
    bs, p = 64, 2
    A = gen(cfg["recipe"], M, K, 1, 0, dt)
    B = gen(cfg["recipe"], K, N, 2, 1, dt)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dt], bs=bs, p=p)
    res = plan.run(to_dev(A), to_dev(B))
    torch.cuda.synchronize()
    cnt = res.counts()
    nb = (M // bs) * (N // bs)
    assert cnt["blocks"] == nb and cnt["clean"] == nb and cnt["checks_critical"] == 0
    rng = np.random.default_rng(1)
    tav, tai = host(plan.topA_val), host(plan.topA_idx)
    tbv, tbi = host(plan.topB_val), host(plan.topB_idx)
    Acs, Bcs, C = host(plan.Acs), host(plan.Bcs), host(res.C)
    for i in rng.integers(0, M, 8):
        v, ix = orc.topp_vector(A[i], p)
        assert np.array_equal(tav[i], v) and np.array_equal(tai[i], ix)
    for j in rng.integers(0, N, 8):
        v, ix = orc.topp_vector(np.ascontiguousarray(B[:, j]), p)
        assert np.array_equal(tbv[j], v) and np.array_equal(tbi[j], ix)
    rows = np.sort(rng.integers(0, M, 4))
    ref = orc.gemm(A[rows], B)
    if cfg["tol"] is None:
        assert np.array_equal(C[rows], ref)
    else:
        assert norm_err(C[rows], ref, A[rows], B) <= cfg["tol"]
    nI, nJ = M // bs, N // bs
    for (I, J) in [(0, 0), (nI - 1, nJ - 1), (int(rng.integers(nI)), int(rng.integers(nJ)))]:
        Ab = A[I * bs:(I + 1) * bs]
        Bb = np.ascontiguousarray(B[:, J * bs:(J + 1) * bs])
        ob = orc.protected_matmul(Ab, Bb, bs=bs, p=p)
        assert np.array_equal(Acs[I], ob["enc"]["Acs"][0])
        assert np.array_equal(Bcs[:, J], ob["enc"]["Bcs"][:, 0])
        assert np.array_equal(tav[M + I], ob["enc"]["topA"][0][bs])
        assert np.array_equal(tbv[N + J], ob["enc"]["topB"][0][bs])
        assert ob["check"].status[0, 0] == res.reports()["status"][I, J] == 0
        Cb = C[I * bs:(I + 1) * bs, J * bs:(J + 1) * bs]
        if cfg["tol"] is None:
            assert np.array_equal(Cb, ob["C"])
        else:
            assert norm_err(Cb, ob["C"], Ab, Bb) <= cfg["tol"]
    del plan, res
    torch.cuda.empty_cache()


def test_distributed_single_rank_nccl(P, orc):
    """The distributed driver (row shard + NCCL counter all-reduce) at world size 1."""
    import os
    import torch.distributed as dist
    from paper_conf_dsn_braunhw14_b200 import distributed as D
    if not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29533")
        dist.init_process_group("nccl", rank=0, world_size=1)
    M, N, K, bs = 256, 256, 128, 64
    A = gen("uniform", M, K, 21, 0)
    B = gen("uniform", K, N, 21, 1)
    r0, n = D.shard_rows(M, 1, 0, bs)
    res, cnt = D.protected_matmul(to_dev(A[r0:r0 + n]), to_dev(B), bs=bs,
                                  faults=[dict(row=3, col=5, site=2, add=1.0)])
    torch.cuda.synchronize()
    assert cnt["blocks"] == 16 and cnt["corrected"] == 1 and cnt["clean"] == 15
    assert norm_err(host(res.C), orc.gemm(A, B), A, B) <= 1e-13
    dist.destroy_process_group()


@pytest.mark.parametrize("dtype,bs", [(np.float64, 8), (np.float64, 16), (np.float64, 32),
                                      (np.float64, 64), (np.float32, 8), (np.float32, 16),
                                      (np.float32, 32), (np.float32, 64), (np.float32, 128)])
def test_fused_reference_sums(P, orc, dtype, bs):
    """The epilogue reference sums (complete after aabft_check) equal the definition (Eq 4) up to
    summation order -- FP64 (64 x 64 DMMA tiles) and FP32 (128 x 128 FFMA tiles)."""
    M, N, K = 384, 256, 300
    A = gen("uniform", M, K, 31, 0, dtype)
    B = gen("uniform", K, N, 31, 1, dtype)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=2)
    assert plan.fused
    res = plan.run(to_dev(A), to_dev(B))
    torch.cuda.synchronize()
    C = host(res.C).astype(np.float64)
    Rcol = C.reshape(M // bs, bs, N).sum(axis=1)
    Rrow = C.reshape(M, N // bs, bs).sum(axis=2)
    scale = np.abs(C).max() * bs
    assert np.max(np.abs(host(plan.Rcol) - Rcol)) <= 1e-14 * scale
    assert np.max(np.abs(host(plan.Rrow) - Rrow)) <= 1e-14 * scale
    assert res.counts()["checks_critical"] == 0


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_bound_elements_bit_exact(P, orc, dtype):
    """aabft_bound_elements: sigma/eps of arbitrary C_fc elements (data and checksum) == oracle."""
    M, N, K, bs, p = 128, 192, 211, 32, 3
    A = gen("wide", M, K, 41, 0, dtype)
    B = gen("uniform", K, N, 41, 1, dtype)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=p)
    plan.encode(to_dev(A), to_dev(B))
    rng = np.random.default_rng(3)
    rows = rng.integers(0, M + M // bs, 200)
    cols = rng.integers(0, N + N // bs, 200)
    sig, eps = plan.bound_elements(torch.from_numpy(rows), torch.from_numpy(cols))
    torch.cuda.synchronize()
    enc = orc.encode(A, B, bs, p)
    (av, ai), (bv, bi) = enc["topA"], enc["topB"]
    for n, (r, c) in enumerate(zip(rows, cols)):
        y = orc.y_of(av[r], ai[r], bv[c], bi[c])
        s_o, e_o = orc.bound(K, y, t=orc.default_t(dtype))
        assert host(sig)[n] == s_o and host(eps)[n] == e_o


def test_accumulator_additive_fault_site3(P, orc):
    """site 3: additive fault into the accumulator mid-k (magnitude-sweep site of SURVEY §8(d))."""
    M, N, K, bs, p = 256, 256, 512, 64, 2
    A = gen("uniform", M, K, 42, 0)
    B = gen("uniform", K, N, 42, 1)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p)
    dA, dB = to_dev(A), to_dev(B)
    clean = host(plan.run(dA, dB).C).copy()
    faults = [dict(row=3, col=4, site=3, k_step=K // 2, add=1e-3),
              dict(row=100, col=200, site=3, k_step=7, add=-0.5)]
    res = plan.run(dA, dB, faults=faults, correct=False)
    torch.cuda.synchronize()
    C1 = host(res.C)
    assert abs((C1[3, 4] - clean[3, 4]) - 1e-3) < 1e-12
    assert abs((C1[100, 200] - clean[100, 200]) + 0.5) < 1e-12
    rep = res.reports()
    assert rep["status"][0, 0] == 4 and rep["status"][1, 3] == 4   # located (SINGLE)


def test_checksum_errors_double_double(P, orc):
    """NEXT-1 diagnostic: carried - exact checksum error with the exact inner product formed in
    double-double on the GPU, against exact rational arithmetic (fractions) on sampled
    elements; Dot2's own error (~2^-104 sum|terms|) is far below the tolerance."""
    from fractions import Fraction
    M, N, K, bs = 128, 128, 300, 32
    A = gen("uniform", M, K, 51, 0)
    B = gen("uniform", K, N, 51, 1)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=2)
    dA, dB = to_dev(A), to_dev(B)
    res = plan.run(dA, dB)
    ec, er = plan.checksum_errors(dA, dB)
    torch.cuda.synchronize()
    Acs, Bcs, Ccol, Crow = host(plan.Acs), host(plan.Bcs), host(res.Ccol), host(res.Crow)
    ec, er = host(ec), host(er)
    rng = np.random.default_rng(5)
    for _ in range(24):
        I, j = int(rng.integers(M // bs)), int(rng.integers(N))
        exact = sum(Fraction(float(Acs[I, k])) * Fraction(float(B[k, j])) for k in range(K))
        ref = float(Fraction(float(Ccol[I, j])) - exact)
        assert abs(ec[I, j] - ref) <= 1e-28 + 1e-12 * abs(ref)
        i, J = int(rng.integers(M)), int(rng.integers(N // bs))
        exact = sum(Fraction(float(A[i, k])) * Fraction(float(Bcs[k, J])) for k in range(K))
        ref = float(Fraction(float(Crow[i, J])) - exact)
        assert abs(er[i, J] - ref) <= 1e-28 + 1e-12 * abs(ref)
    assert np.abs(ec).max() > 0  # the GEMM does round


@pytest.mark.parametrize("n", [512, 1024, 2048, 4096])
@pytest.mark.parametrize("table", ["table2_uniform1.json", "table3_uniform100.json"])
def test_gpu_bound_column_tables(P, orc, n, table):
    """Published-number pin of the GPU encode + bound path at full size: mean eps over all
    carried checksum elements (BS 32, p 2, 3 sigma, t 52) within 5% of Table II / III."""
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", table)))
    A = gen(g["recipe"], n, n, 1, 0)
    B = gen(g["recipe"], n, n, 2, 1)
    plan = P.ProtectedGemm(n, n, n, dtype=torch.float64, bs=32, p=2)
    plan.encode(to_dev(A), to_dev(B))
    b = plan.bound()
    torch.cuda.synchronize()
    m = float(torch.cat([b["eps_col"].ravel(), b["eps_row"].ravel()]).mean())
    paper = g["rows"][str(n)]["avg_aabft"]
    assert 0.95 * paper <= m <= 1.05 * paper, (m, paper)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_cuda_graph_replay(P, orc, dtype):
    """The four C-ABI calls captured in one CUDA graph: a replay equals the eager run bit for
    bit, and picks up new contents of the captured input buffers."""
    M = N = K = 128
    bs, p = 32, 2
    A = gen("uniform", M, K, 31, 0, dtype)
    B = gen("uniform", K, N, 31, 1, dtype)
    dA, dB = to_dev(A), to_dev(B)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=p)
    g = plan.capture(dA, dB)
    g.replay()
    torch.cuda.synchronize()
    C1, cnt1 = host(plan.C).copy(), plan.result().counts()
    eager = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=p)
    res = eager.run(dA, dB)
    torch.cuda.synchronize()
    assert np.array_equal(C1, host(res.C)) and cnt1 == res.counts()
    A2 = gen("uniform", M, K, 32, 0, dtype)
    dA.copy_(torch.from_numpy(A2).cuda())
    g.replay()
    torch.cuda.synchronize()
    o = orc.protected_matmul(A2, B, bs=bs, p=p)
    assert norm_err(host(plan.C), o["C"], A2, B) <= (1e-13 if dtype == np.float64 else 0.0)
    assert plan.result().counts()["clean"] == (M // bs) * (N // bs)


@pytest.mark.parametrize("fused", [True, False])
def test_memory_corruption_between_gemm_and_check(P, orc, fused):
    """Fault model of the two check modes.  The paper's
    check re-sums the result sub-matrix from memory: the unfused check does that and
    catches a C element corrupted in HBM after the GEMM stored it.  The fused check compares
    the reference sums the GEMM epilogue formed in registers (computational faults, Alg 3
    P:L501-541), so such a memory corruption is outside its fault model and reads CLEAN."""
    M, N, K, bs, p = 256, 256, 256, 64, 2
    A = gen("uniform", M, K, 61, 0)
    B = gen("uniform", K, N, 61, 1)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p, fused=fused)
    dA, dB = to_dev(A), to_dev(B)
    clean = host(plan.run(dA, dB).C).copy()
    plan.encode(dA, dB)
    plan.gemm(dA, dB)
    plan._C[70, 130] += 5.0  # corrupt the stored result in device memory
    plan.check()
    plan.correct()
    torch.cuda.synchronize()
    rep = plan.result().reports()
    if fused:
        assert plan.result().counts()["clean"] == 16
        assert host(plan.C)[70, 130] == clean[70, 130] + 5.0
    else:
        assert rep["status"][1, 2] == 1 and plan.result().counts()["corrected"] == 1
        assert abs(host(plan.C)[70, 130] - clean[70, 130]) <= 1e-12


def test_recheck_after_correction_is_clean(P, orc):
    """aabft_correct refreshes the fused reference sums it invalidates: checking
    the corrected product again reports every block CLEAN and nothing to correct."""
    M, N, K, bs, p = 256, 256, 256, 64, 2
    A = gen("uniform", M, K, 62, 0)
    B = gen("uniform", K, N, 62, 1)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p)
    dA, dB = to_dev(A), to_dev(B)
    res = plan.run(dA, dB, faults=[dict(row=3, col=200, site=2, add=1.0),
                                   dict(row=150, col=20, site=0, xor_mask=1 << 62)])
    torch.cuda.synchronize()
    assert res.counts()["corrected"] == 2
    plan.check()
    torch.cuda.synchronize()
    cnt = plan.result().counts()
    assert cnt["clean"] == 16 and cnt["checks_critical"] == 0, cnt
    assert cnt["max_ratio"] < 0.5


@pytest.mark.parametrize("fused", [True, False])
@pytest.mark.parametrize("topp_in_gemm", [True, False])
def test_zero_padded_operands(P, orc, fused, topp_in_gemm):
    """Caller zero-padding ("padded matrix A", Alg 1; reading R20): zero rows of A and
    zero columns of B give y = 0, eps = 0 and d = 0 for their checks, which must read CLEAN
    (|d| <= eps with equality, reading R9); zeros are selectable in the top-p (R14).  Tables,
    C and every report field equal the oracle's; a fault inside the padding is critical."""
    M, N, K, bs, p = 256, 192, 200, 64, 2
    A = gen("uniform", M, K, 71, 0)
    B = gen("uniform", K, N, 71, 1)
    A[M - bs:] = 0.0      # last block-row padded
    B[:, N - bs:] = 0.0   # last block-column padded
    A[5, :] = 0.0         # and one all-zero data row inside a live block
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p, fused=fused,
                           topp_in_gemm=topp_in_gemm)
    res = plan.run(to_dev(A), to_dev(B))
    torch.cuda.synchronize()
    o = orc.protected_matmul(A, B, bs=bs, p=p)
    enc = o["enc"]
    assert np.array_equal(host(plan.topA_val), enc["topA"][0])
    assert np.array_equal(host(plan.topA_idx), enc["topA"][1])
    assert np.array_equal(host(plan.topB_val), enc["topB"][0])
    assert np.array_equal(host(plan.topB_idx), enc["topB"][1])
    assert norm_err(host(res.C), o["C"], A, B) <= 1e-13
    assert np.all(host(res.C)[M - bs:] == 0) and np.all(host(res.C)[:, N - bs:] == 0)
    assert_reports_equal(res.reports(), o["check"])
    cnt = res.counts()
    assert cnt["clean"] == cnt["blocks"] == (M // bs) * (N // bs) and cnt["checks_critical"] == 0
    # a fault in the padded corner: eps = 0 there, so any nonzero error is critical
    f = [dict(row=M - 3, col=N - 5, site=2, add=1e-300)]
    res = plan.run(to_dev(A), to_dev(B), faults=f)
    torch.cuda.synchronize()
    of = orc.protected_matmul(A, B, bs=bs, p=p, faults=f)
    assert res.reports()["status"][M // bs - 1, N // bs - 1] == 1 == of["check"].status[-1, -1]
    assert np.all(host(res.C)[M - bs:] == 0)
