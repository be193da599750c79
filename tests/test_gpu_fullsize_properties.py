"""Full-size properties at BASELINE configs[1] and [2] (top-p lists, Eq 1 / Eq 2 checksums, Eq 3 product).

Alg 1 selects, per row of A / column of B and per checksum row / column, the p
largest |values|; reading R13 fixes the order (value descending, ties to the lowest index).  At
full size the sequential oracle is too slow to run over every vector, but the selection has a
plain definition: the first p entries of a STABLE descending sort of |vector|.  torch.sort (a
library primitive, independent of this repo's kernels) gives that permutation, so every index,
every value and the tie order are compared for every vector -- data and checksum vectors -- and
the indices of each list are distinct by construction of the comparison.
"""
import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def P():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_dsn_braunhw14_b200 import api
    return api


def first_p_stable(X, p):
    """(values, indices) of the first p entries of a stable descending sort of |X| per row."""
    v, i = torch.sort(X.abs().to(torch.float64), dim=1, descending=True, stable=True)
    return v[:, :p], i[:, :p].to(torch.int32)


@pytest.mark.parametrize("case", [
    ("f64", 4096, 4096, 4096, 64, 2, "uniform"),     # configs[1]
    ("f32", 8192, 8192, 8192, 64, 2, "wide"),        # configs[2]
    ("f64", 4096, 4096, 4096, 64, 2, "integer"),     # many exact ties
])
def test_topp_full_size_equals_stable_sort(P, case):
    dt, M, N, K, bs, p, recipe = case
    npdt = np.float64 if dt == "f64" else np.float32
    tdt = torch.float64 if dt == "f64" else torch.float32
    kw = dict(q=3) if recipe == "integer" else {}
    A = torch.from_numpy(synth.generate(recipe, M, K, seed=31, matrix_id=0, dtype=npdt, **kw)).cuda()
    B = torch.from_numpy(synth.generate(recipe, K, N, seed=31, matrix_id=1, dtype=npdt, **kw)).cuda()
    plan = P.ProtectedGemm(M, N, K, dtype=tdt, bs=bs, p=p)
    plan.encode(A, B)
    torch.cuda.synchronize()
    rowsA = torch.cat([A, plan.Acs], dim=0)          # data rows, then checksum rows
    colsB = torch.cat([B.t(), plan.Bcs.t()], dim=0)  # data columns, then checksum columns
    for X, val, idx, name in ((rowsA, plan.topA_val, plan.topA_idx, "A"),
                              (colsB, plan.topB_val, plan.topB_idx, "B")):
        ev, ei = first_p_stable(X, p)
        assert torch.equal(idx, ei), name
        assert torch.equal(val, ev), name


@pytest.mark.parametrize("case", [
    ("f64", 4096, 4096, 4096, 64),     # configs[1]
    ("f32", 8192, 8192, 8192, 64),     # configs[2]
])
def test_checksums_full_size_sequential_definition(P, case):
    """Eq 1 / Eq 2 at full size, bit for bit: Acs[I] = (((A[I*bs] + A[I*bs+1]) + ...) summed in
    ascending order in the working precision (reading R11), written out as bs elementwise
    library adds over all blocks at once (IEEE adds, no contraction); Bcs likewise over j."""
    dt, M, N, K, bs = case
    npdt = np.float64 if dt == "f64" else np.float32
    tdt = torch.float64 if dt == "f64" else torch.float32
    rec = "uniform" if dt == "f64" else "wide"
    A = torch.from_numpy(synth.generate(rec, M, K, seed=32, matrix_id=0, dtype=npdt)).cuda()
    B = torch.from_numpy(synth.generate(rec, K, N, seed=32, matrix_id=1, dtype=npdt)).cuda()
    plan = P.ProtectedGemm(M, N, K, dtype=tdt, bs=bs, p=2)
    plan.encode(A, B)
    torch.cuda.synchronize()
    Ab = A.view(M // bs, bs, K)
    acs = Ab[:, 0].clone()
    for r in range(1, bs):
        acs = acs + Ab[:, r]
    Bb = B.view(K, N // bs, bs)
    bcs = Bb[:, :, 0].clone()
    for c in range(1, bs):
        bcs = bcs + Bb[:, :, c]
    assert torch.equal(plan.Acs, acs)
    assert torch.equal(plan.Bcs, bcs)


@pytest.mark.parametrize("case", [
    ("f64", 4096, 4096, 4096, 64, 1e-13),   # configs[1]: north_star's FP64 bar
    ("f32", 8192, 8192, 8192, 64, 1e-5),    # configs[2]: north_star's FP32 bar
])
def test_product_full_size_every_element(P, case):
    """Eq 3 at full size, EVERY element of C, Ccol = Acs.B and Crow = A.Bcs against an FP64
    library product of the same operands (cuBLAS via torch.matmul -- an independent
    implementation of the plain definition), normalised by |A||B| as north_star states."""
    dt, M, N, K, bs, tol = case
    npdt = np.float64 if dt == "f64" else np.float32
    tdt = torch.float64 if dt == "f64" else torch.float32
    rec = "uniform" if dt == "f64" else "wide"
    A = torch.from_numpy(synth.generate(rec, M, K, seed=33, matrix_id=0, dtype=npdt)).cuda()
    B = torch.from_numpy(synth.generate(rec, K, N, seed=33, matrix_id=1, dtype=npdt)).cuda()
    plan = P.ProtectedGemm(M, N, K, dtype=tdt, bs=bs, p=2)
    res = plan.run(A, B)
    torch.cuda.synchronize()
    assert res.counts()["checks_critical"] == 0
    A64, B64 = A.double(), B.double()
    Acs64, Bcs64 = plan.Acs.double(), plan.Bcs.double()
    for got, ref, den in ((res.C, A64 @ B64, A64.abs() @ B64.abs()),
                          (res.Ccol, Acs64 @ B64, Acs64.abs() @ B64.abs()),
                          (res.Crow, A64 @ Bcs64, A64.abs() @ Bcs64.abs())):
        err = ((got.double() - ref).abs() / den.clamp_min(1e-300)).max().item()
        assert err <= tol, err
