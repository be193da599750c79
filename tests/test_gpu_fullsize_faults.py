"""Fault-verdict parity at the bench configurations (paper §VI-C).

The paper injects one fault per GEMM at n up to 8192.  Here every faulted BS x BS
block is an independent trial (partitioned encoding): one GEMM in the bench's launch
configuration carries one fault in each of a few hundred blocks -- chosen to include both the
data-parallel waves and the stream-K tail tiles of the persistent FP64 schedule -- swept over
magnitudes 2^-6 .. 2^6 x eps (additive, at the final value = site 2 and in the accumulator
mid-k = site 3, Alg 3 errorVecAdd2 / errorVecAdd1) and over every bit of the final value
(site 0, XOR).  The oracle recomputes each faulted block from scratch -- the BS rows of A and
BS columns of B over the full K give exactly that block's C, carried checksums, top-p tables
and bounds -- applies the same fault with its own arithmetic, and checks / corrects it.
Outside the 2x band (reading R22) the verdicts must be identical: status, critical row and
column counts, located element; 'must detect' faults are corrected and 'must be silent' ones
leave the block CLEAN on both sides.
"""
import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

CFG = {
    # name: M, N, K, bs, dtype, recipe, faulted blocks
    "c2": (4096, 4096, 4096, 64, np.float64, "uniform", 256),
    "c3": (8192, 8192, 8192, 64, np.float32, "wide", 256),
    "c5": (8192, 8192, 65536, 64, np.float64, "uniform", 48),
}


@pytest.fixture(scope="module")
def P():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_dsn_braunhw14_b200 import api
    return api


def to_device(recipe, rows, cols, seed, mid, dtype, chunk=1024):
    """Full matrix on the device, generated in row chunks (bounded host memory)."""
    td = torch.float64 if dtype == np.float64 else torch.float32
    X = torch.empty(rows, cols, dtype=td, device="cuda")
    for r0 in range(0, rows, chunk):
        n = min(chunk, rows - r0)
        X[r0:r0 + n] = torch.from_numpy(synth.generate(recipe, n, cols, seed=seed, matrix_id=mid,
                                                       dtype=dtype, row0=r0, full_cols=cols)).cuda()
    return X


def xor_value(v, bit, dtype):
    ut = np.uint64 if dtype == np.float64 else np.uint32
    a = np.array([v], dtype=dtype).view(ut) ^ ut(1 << bit)
    with np.errstate(all="ignore"):
        return float(a.view(dtype)[0])


def pick_blocks(nI, nJ, n, rng):
    """n distinct blocks: a quarter from the last block-columns (the stream-K tail tiles of the
    grouped raster sit at the end of the last group) and the rest uniformly."""
    tail = [(I, J) for I in range(nI) for J in range(max(0, nJ - 6), nJ)]
    pick = {tail[k] for k in rng.choice(len(tail), n // 4, replace=False)}
    while len(pick) < n:
        pick.add((int(rng.integers(nI)), int(rng.integers(nJ))))
    return sorted(pick)


@pytest.mark.parametrize("name", list(CFG))
def test_fault_verdicts_full_size(P, orc, name):
    M, N, K, bs, dt, recipe, nblk = CFG[name]
    td = torch.float64 if dt == np.float64 else torch.float32
    nbits = 64 if dt == np.float64 else 32
    rng = np.random.default_rng({"c2": 11, "c3": 12, "c5": 13}[name])
    A = to_device(recipe, M, K, 1, 0, dt)
    B = to_device(recipe, K, N, 2, 1, dt)
    plan = P.ProtectedGemm(M, N, K, dtype=td, bs=bs, p=2)
    res = plan.run(A, B)
    torch.cuda.synchronize()
    assert res.counts()["clean"] == (M // bs) * (N // bs)
    C0 = res.C.detach().cpu().numpy().copy()
    bnd = plan.bound()
    eps_col = bnd["eps_col"].cpu().numpy()
    eps_row = bnd["eps_row"].cpu().numpy()
    blocks = pick_blocks(M // bs, N // bs, nblk, rng)
    faults, labels = [], []
    for n, (I, J) in enumerate(blocks):
        i = I * bs + int(rng.integers(bs))
        j = J * bs + int(rng.integers(bs))
        lo = min(eps_col[I, j], eps_row[i, J])
        hi = max(eps_col[I, j], eps_row[i, J])
        kind = n % 3
        if kind < 2:  # magnitude sweep, site 2 (final value) / site 3 (accumulator mid-k)
            r = 2.0 ** (int(rng.integers(-12, 13)) / 2) * (1 if rng.integers(2) else -1)
            f = dict(row=i, col=j, site=2 if kind == 0 else 3, k_step=K // 2, add=float(r * hi))
            e = abs(r * hi)
        else:  # bit sweep of the final value (site 0)
            bit = int(rng.integers(nbits))
            f = dict(row=i, col=j, site=0, xor_mask=1 << bit)
            e = abs(xor_value(C0[i, j], bit, dt) - float(C0[i, j]))
        lab = "detect" if (not np.isfinite(e) or e > 2 * hi) else ("silent" if e < 0.5 * lo else "band")
        faults.append(f)
        labels.append(lab)
    assert labels.count("detect") > nblk // 5 and labels.count("silent") > nblk // 10
    res = plan.run(A, B, faults=faults)
    torch.cuda.synchronize()
    rep = res.reports()
    C1 = res.C.detach().cpu().numpy()
    faulted = np.zeros(rep.shape, bool)
    nchk = 0
    for (I, J), f, lab in zip(blocks, faults, labels):
        faulted[I, J] = True
        Ab = synth.generate(recipe, bs, K, seed=1, matrix_id=0, dtype=dt, row0=I * bs, full_cols=K)
        Bb = synth.generate(recipe, K, bs, seed=2, matrix_id=1, dtype=dt, col0=J * bs, full_cols=N)
        lf = dict(f, row=f["row"] - I * bs, col=f["col"] - J * bs)
        o = orc.protected_matmul(Ab, Bb, bs=bs, p=2, faults=[lf])
        och = o["check"]
        g = rep[I, J]
        if lab == "band":
            continue
        nchk += 1
        want = 1 if lab == "detect" else 0
        assert g["status"] == want == och.status[0, 0], (name, f, lab, g, och.status)
        assert (g["n_bad_rows"], g["n_bad_cols"]) == (och.nrows[0, 0], och.ncols[0, 0]), (f, g)
        assert (g["row"], g["col"]) == (och.row[0, 0] + I * bs if och.row[0, 0] >= 0 else -1,
                                        och.col[0, 0] + J * bs if och.col[0, 0] >= 0 else -1)
        if lab == "detect":
            # recomputed from the carried column checksum: off by at most that checksum's own
            # rounding error (bounded by eps_col) plus the final rounding
            i, j = f["row"], f["col"]
            c0 = float(C0[i, j])
            tol = eps_col[I, j] + 2 * float(np.spacing(dt(abs(c0))))
            assert abs(float(C1[i, j]) - c0) <= tol, (name, f, C1[i, j], c0, tol)
            assert abs(float(o["C"][i - I * bs, j - J * bs]) - c0) <= tol
    assert nchk >= nblk // 2
    # every block without a fault is CLEAN, every element outside the faulted ones untouched
    assert np.all(rep["status"][~faulted] == 0)
    mask = np.ones(C0.shape, bool)
    for f in faults:
        mask[f["row"], f["col"]] = False
    assert np.array_equal(C1[mask], C0[mask])
    del plan, res, A, B
    torch.cuda.empty_cache()
