"""GPU parity of the NEXT-3 comparators (through the C ABI) against the oracle.

* checksums-only encode (aabft_encode with NULL top-p tables): Acs / Bcs bit-identical, top-p
  tables untouched;
* SEA-ABFT bound (aabft_sea_bound, §III): eps_col / eps_row / eps_corner
  bit-identical to oracle O11 (sequential norms, same evaluation order), and the GPU path
  reproduces Table II / III "AVG. SEA-ABFT" at full size;
* external-eps check / correct (aabft_check_ext / aabft_correct_ext, reading R26): fixed-eps
  ABFT on integer data is exact; SEA-ABFT verdicts equal the oracle's outside the 2x band;
  the A-ABFT eps fed back through check_ext reproduces aabft_check; fused reference sums may
  be checked twice.
"""
import json
import os

import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TD = {np.float64: torch.float64, np.float32: torch.float32}
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


@pytest.fixture(scope="module")
def P():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_dsn_braunhw14_b200 import api
    return api


def gen(recipe, r, c, seed, mid, dtype=np.float64, **kw):
    return synth.generate(recipe, r, c, seed=seed, matrix_id=mid, dtype=dtype, **kw)


def to_dev(X):
    X = np.ascontiguousarray(X)
    r, c = X.shape
    q = 16 // X.itemsize
    ld = (c + q - 1) // q * q
    buf = torch.zeros(r, ld, dtype=TD[X.dtype.type], device="cuda")
    buf[:, :c] = torch.from_numpy(X).cuda()
    return buf[:, :c]


def host(t):
    return t.detach().cpu().numpy()


SHAPES = [(128, 128, 128, 32), (192, 320, 200, 64), (64, 96, 37, 8), (256, 256, 1000, 128)]


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("shape", SHAPES)
def test_checksums_only_encode(P, orc, dtype, shape):
    M, N, K, bs = shape
    A = gen("wide", M, K, 3, 0, dtype)
    B = gen("wide", K, N, 3, 1, dtype)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=2)
    plan.topA_val.fill_(7.0)
    plan.topB_val.fill_(7.0)
    plan.encode(to_dev(A), to_dev(B), topp=False)
    torch.cuda.synchronize()
    assert np.array_equal(host(plan.Acs), orc.encode_cols(A, bs))
    assert np.array_equal(host(plan.Bcs), orc.encode_rows(B, bs))
    assert bool((plan.topA_val == 7.0).all()) and bool((plan.topB_val == 7.0).all())


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("recipe", ["uniform", "wide"])
def test_sea_bound_bit_exact(P, orc, dtype, shape, recipe):
    M, N, K, bs = shape
    A = gen(recipe, M, K, 4, 0, dtype)
    B = gen(recipe, K, N, 4, 1, dtype)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=2)
    dA, dB = to_dev(A), to_dev(B)
    plan.encode(dA, dB, topp=False)
    d = plan.sea_bound(dA, dB, corner=True)
    torch.cuda.synchronize()
    o = orc.sea_bounds(A, B, orc.encode_cols(A, bs), orc.encode_rows(B, bs), bs)
    for k in ("eps_col", "eps_row", "eps_corner"):
        assert np.array_equal(host(d[k]), o[k]), k


@pytest.mark.parametrize("n", [512, 1024, 2048, 4096, 8192])
@pytest.mark.parametrize("table", ["table2_uniform1.json", "table3_uniform100.json"])
def test_gpu_sea_column_tables(P, n, table):
    """Published-number pin at full size: mean SEA eps over every checksum element of the
    full-checksum blocks (column, row and corner, reading R25; BS 32, t 52) within 5% of the
    paper's "AVG. SEA-ABFT" column."""
    g = json.load(open(os.path.join(GOLDEN, table)))
    A = gen(g["recipe"], n, n, 1, 0)
    B = gen(g["recipe"], n, n, 2, 1)
    plan = P.ProtectedGemm(n, n, n, dtype=torch.float64, bs=32, p=2)
    dA, dB = to_dev(A), to_dev(B)
    plan.encode(dA, dB, topp=False)
    d = plan.sea_bound(dA, dB, corner=True)
    v = torch.cat([d["eps_col"].ravel(), d["eps_row"].ravel(), d["eps_corner"].ravel()])
    m = float(v.mean())
    paper = g["rows"][str(n)]["avg_sea_abft"]
    assert 0.95 * paper <= m <= 1.05 * paper, (m, paper, m / paper)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("fused", [True, False])
def test_fixed_eps_integer_exact(P, orc, dtype, fused):
    """Fixed-eps ABFT (Table I "ABFT") on integer data: every checksum is exact, so
    eps = 0.5 separates clean (d = 0) from any integer fault; location and correction exact."""
    M, N, K, bs = 256, 192, 96, 32
    A = gen("integer", M, K, 6, 0, dtype, q=4)
    B = gen("integer", K, N, 6, 1, dtype, q=4)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=2, fused=fused)
    dA, dB = to_dev(A), to_dev(B)
    res = plan.run_ext(dA, dB, mode="fixed", eps_fixed=0.5)
    torch.cuda.synchronize()
    clean = host(res.C).copy()
    cnt = res.counts()
    assert cnt["clean"] == cnt["blocks"] == (M // bs) * (N // bs)
    assert cnt["checks_rounding"] == (M // bs) * N + M * (N // bs) and cnt["max_ratio"] == 0.0
    faults = [dict(row=3, col=5, site=2, add=3.0), dict(row=100, col=70, site=2, add=-1.0),
              dict(row=M + 2, col=40, site=2, add=2.0), dict(row=200, col=N + 1, site=2, add=5.0)]
    res = plan.run_ext(dA, dB, mode="fixed", eps_fixed=0.5, faults=faults)
    torch.cuda.synchronize()
    rep = res.reports()
    o = orc.abft_matmul_ext(A, B, bs=bs, mode="fixed", eps_fixed=0.5, faults=faults)
    assert np.array_equal(rep["status"], o["check"].status)
    assert rep["status"][0, 0] == 1 and rep["status"][100 // bs, 70 // bs] == 1
    assert rep["status"][2, 40 // bs] == 2 and rep["status"][200 // bs, 1] == 2
    assert np.array_equal(host(res.C), clean)
    assert np.array_equal(res.counts_buf.cpu().numpy()[:8], o["check"].counts)


@pytest.mark.parametrize("dtype,fused", [(np.float64, True), (np.float64, False),
                                         (np.float32, False)])
def test_sea_verdicts_outside_band(P, orc, dtype, fused):
    """SEA-ABFT check (NEXT-3): clean run zero critical; one additive fault per block at
    magnitudes r * max(eps_SEA) across the band -- verdicts identical to the oracle outside the
    2x band (north_star rule applied to the comparator's own eps)."""
    M, N, K, bs = 512, 384, 256, 64
    A = gen("uniform", M, K, 21, 0, dtype)
    B = gen("uniform", K, N, 21, 1, dtype)
    Acs, Bcs = orc.encode_cols(A, bs), orc.encode_rows(B, bs)
    sea = orc.sea_bounds(A, B, Acs, Bcs, bs)
    plan = P.ProtectedGemm(M, N, K, dtype=TD[dtype], bs=bs, p=2, fused=fused)
    dA, dB = to_dev(A), to_dev(B)
    res = plan.run_ext(dA, dB, mode="sea")
    torch.cuda.synchronize()
    clean = host(res.C).copy()
    cnt = res.counts()
    assert cnt["clean"] == cnt["blocks"] and cnt["checks_critical"] == 0
    assert cnt["max_ratio"] < 0.05  # SEA is loose (Tables II/III: ~2 orders above A-ABFT)
    rng = np.random.default_rng(8)
    faults, labels = [], []
    mags = [2.0 ** -6, 2.0 ** -2, 2.0 ** 2, 2.0 ** 6]
    for I in range(M // bs):
        for J in range(N // bs):
            i, j = I * bs + int(rng.integers(bs)), J * bs + int(rng.integers(bs))
            lo = min(sea["eps_col"][I, j], sea["eps_row"][i, J])
            hi = max(sea["eps_col"][I, j], sea["eps_row"][i, J])
            add = float(mags[(I + J) % 4] * hi * (1 if rng.integers(2) else -1))
            faults.append(dict(row=i, col=j, site=2, add=add))
            labels.append("detect" if abs(add) > 2 * hi else ("silent" if abs(add) < 0.5 * lo else "band"))
    res = plan.run_ext(dA, dB, mode="sea", faults=faults)
    torch.cuda.synchronize()
    rep = res.reports()
    o = orc.abft_matmul_ext(A, B, bs=bs, mode="sea", faults=faults)
    ost = o["check"].status
    Cg = host(res.C)
    n_det = 0
    for f, lab in zip(faults, labels):
        I, J = f["row"] // bs, f["col"] // bs
        if lab == "detect":
            assert rep["status"][I, J] == 1 and ost[I, J] == 1, f
            tol = 1e-12 if dtype == np.float64 else 1e-3
            cv = clean[f["row"], f["col"]]
            assert abs(Cg[f["row"], f["col"]] - cv) <= tol * max(1.0, abs(cv))
            n_det += 1
        elif lab == "silent":
            assert rep["status"][I, J] == 0 and ost[I, J] == 0, f
    assert n_det >= len(faults) // 4


def test_check_ext_with_aabft_eps_reproduces_check(P, orc):
    """aabft_check_ext fed the A-ABFT eps (aabft_bound) gives the A-ABFT verdicts (the CRITICAL
    threshold is the same; sigma is not passed, so only ROUNDING / CRITICAL classes), and the
    fused reference sums survive being checked twice."""
    M, N, K, bs = 256, 256, 512, 64
    A = gen("uniform", M, K, 31, 0)
    B = gen("uniform", K, N, 31, 1)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=2, fused=True)
    dA, dB = to_dev(A), to_dev(B)
    faults = [dict(row=10, col=20, site=2, add=1e-6), dict(row=130, col=200, site=0, xor_mask=1 << 62),
              dict(row=M + 1, col=77, site=2, add=1e-5)]
    fb = P.make_faults(faults, dA.device)
    plan.encode(dA, dB)
    plan.gemm(dA, dB, fb, len(faults))
    plan.check()
    rep1 = plan.result().reports().copy()
    b = plan.bound()
    plan.check_ext(eps_col=b["eps_col"], eps_row=b["eps_row"])
    torch.cuda.synchronize()
    rep2 = plan.result().reports().copy()
    assert np.array_equal(rep1["status"], rep2["status"])
    assert np.array_equal(rep1["row"], rep2["row"]) and np.array_equal(rep1["col"], rep2["col"])
    assert np.array_equal(rep1["n_bad_rows"], rep2["n_bad_rows"])
    assert rep1["status"][0, 0] == 4 and rep1["status"][2, 3] == 4 and rep1["status"][1, 1] == 2
    # and a third pass with the A-ABFT check again: still identical (idempotent fused sums)
    plan.check()
    torch.cuda.synchronize()
    assert np.array_equal(plan.result().reports()["status"], rep1["status"])


# --------------------------------------------------------------------------- NEXT-2 (Alg 3)
def test_f32_instruction_exact_faults(P, orc):
    """FP32 FFMA path (NEXT-2, Alg 3): mul (site 4, errorVecMul), accumulator XOR /
    add after an arbitrary step (sites 1 / 3, errorVecAdd1) and final-value faults (sites 0 / 2,
    errorVecAdd2) land in C, Ccol and Crow bit-identical to the oracle's step-exact dot_fault;
    k_step anywhere (not only at k-tile ends), several faults per tile, ragged K."""
    M, N, K, bs = 256, 384, 203, 64
    A = gen("wide", M, K, 41, 0, np.float32)
    B = gen("wide", K, N, 41, 1, np.float32)
    rng = np.random.default_rng(3)
    faults = []
    for n in range(60):
        site = [4, 1, 3, 0, 2, 4][n % 6]
        if n % 10 == 7:
            row, col = M + int(rng.integers(M // bs)), int(rng.integers(N))
        elif n % 10 == 9:
            row, col = int(rng.integers(M)), N + int(rng.integers(N // bs))
        else:
            row, col = int(rng.integers(M)), int(rng.integers(N))
        bit = int(rng.integers(0, 32))
        mask = (1 << bit) | ((1 << int(rng.integers(0, 32))) if n % 3 == 0 else 0)
        faults.append(dict(row=row, col=col, site=site, k_step=int(rng.integers(K)),
                           xor_mask=mask, add=float(rng.normal()) * 8.0))
    # at most one fault per element (the oracle applies one per element)
    seen, uniq = set(), []
    for f in faults:
        if (f["row"], f["col"]) not in seen:
            seen.add((f["row"], f["col"]))
            uniq.append(f)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float32, bs=bs, p=2)
    dA, dB = to_dev(A), to_dev(B)
    plan.encode(dA, dB)
    fb = P.make_faults(uniq, dA.device)
    plan.gemm(dA, dB, fb, len(uniq))
    torch.cuda.synchronize()
    enc = orc.encode(A, B, bs, 2)
    Cm, Ccol, Crow = orc.gemm(A, B), orc.gemm(enc["Acs"], B), orc.gemm(A, enc["Bcs"])
    orc.apply_faults(A, B, enc, Cm, Ccol, Crow, uniq)
    g = [host(plan.C), host(plan.Ccol), host(plan.Crow)]
    for G, O in zip(g, (Cm, Ccol, Crow)):
        same = (G.view(np.uint32) == O.view(np.uint32)) | (np.isnan(G) & np.isnan(O))
        assert same.all(), np.argwhere(~same)[:5]
