"""AABFT_FLAG_CHECK_CORRECTS and the memset-free check counters.

Alg 2 classifies and corrects per block; with the flag aabft_check corrects every
SINGLE block in the same kernel.  The result must equal check() followed by correct() -- C,
every report field and every counter -- for both check kernels (fused: reference sums from the
GEMM epilogue; unfused: re-sum of C) and both dtypes.  The counters no longer need a memset:
aabft_gemm zeroes the workspace accumulator and the check's last CTA re-arms it, so repeated
checks report the same totals and a garbage-filled workspace gives correct totals.
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


def host(t):
    return t.detach().cpu().numpy()


def faults_for(M, N, bs, n, seed):
    rng = np.random.default_rng(seed)
    nI, nJ = M // bs, N // bs
    out = []
    # blocks other than (0, 0) and (0, nJ - 1), which get the multi-fault cases below
    cand = [b for b in range(nI * nJ) if b not in (0, nJ - 1)]
    for b in rng.choice(cand, size=min(n, len(cand)), replace=False):
        I, J = divmod(int(b), nJ)
        out.append(dict(row=I * bs + int(rng.integers(bs)), col=J * bs + int(rng.integers(bs)),
                        site=2, add=float(rng.choice([1.0, -64.0, 1e3]))))
    # two faults in one block (uncorrectable) and one in a carried checksum (checksum only)
    out.append(dict(row=1, col=2, site=2, add=5.0))
    out.append(dict(row=2, col=3, site=2, add=7.0))
    out.append(dict(row=M, col=N - 1, site=2, add=9.0))
    return out


CASES = [
    (torch.float64, 512, 640, 300, 64, 2, True),
    (torch.float64, 512, 640, 300, 64, 2, False),
    (torch.float64, 256, 256, 130, 32, 3, True),
    (torch.float64, 256, 512, 200, 128, 2, False),   # bs > 64: the streaming check
    (torch.float32, 512, 512, 256, 64, 2, True),
    (torch.float32, 768, 768, 300, 256, 2, False),   # 3 x 3 blocks of 256
]


@pytest.mark.parametrize("case", CASES)
def test_check_corrects_equals_check_then_correct(P, case):
    dt, M, N, K, bs, p, fused = case
    npdt = np.float64 if dt == torch.float64 else np.float32
    A = torch.from_numpy(synth.generate("uniform", M, K, seed=21, matrix_id=0, dtype=npdt)).cuda()
    B = torch.from_numpy(synth.generate("uniform", K, N, seed=21, matrix_id=1, dtype=npdt)).cuda()
    fl = P.make_faults(faults_for(M, N, bs, 6, 21), "cuda")
    nf = fl.numel() // 48
    outs = []
    for fusedcorr in (True, False):
        plan = P.ProtectedGemm(M, N, K, dtype=dt, bs=bs, p=p, fused=fused)
        plan.encode(A, B)
        plan.gemm(A, B, fl, nf)
        if fusedcorr:
            plan.check(correct=True)
        else:
            plan.check()
            plan.correct()
        torch.cuda.synchronize()
        res = plan.result()
        outs.append((host(res.C).copy(), host(res.report_buf).copy(), res.counts()))
    (C1, R1, n1), (C2, R2, n2) = outs
    assert np.array_equal(C1, C2)
    assert np.array_equal(R1, R2)
    assert n1 == n2
    assert n1["corrected"] >= 6 and n1["uncorrectable"] >= 1 and n1["checksum_only"] >= 1


@pytest.mark.parametrize("fused", [True, False])
def test_repeated_check_counts_rearmed(P, fused):
    """The accumulator is re-armed by the last CTA: a second check reports the same totals."""
    M = N = K = 512
    A = torch.from_numpy(synth.generate("uniform", M, K, seed=22, matrix_id=0)).cuda()
    B = torch.from_numpy(synth.generate("uniform", K, N, seed=22, matrix_id=1)).cuda()
    plan = P.ProtectedGemm(M, N, K, bs=64, p=2, fused=fused)
    plan.run(A, B, faults=[dict(row=5, col=7, site=2, add=3.0)], correct=False)
    torch.cuda.synchronize()
    c1 = plan.result().counts()
    for _ in range(3):
        plan.check()
    torch.cuda.synchronize()
    assert plan.result().counts() == c1
    assert c1["blocks"] == 64 and c1["clean"] == 63


def test_garbage_workspace_counts(P):
    """A workspace full of garbage still gives exact totals (the GEMM zeroes the accumulator)."""
    M = N = K = 256
    A = torch.from_numpy(synth.generate("uniform", M, K, seed=23, matrix_id=0)).cuda()
    B = torch.from_numpy(synth.generate("uniform", K, N, seed=23, matrix_id=1)).cuda()
    plan = P.ProtectedGemm(M, N, K, bs=32, p=2)
    plan.ws.fill_(0xA5)  # not zero: the check must not depend on a pre-zeroed workspace
    plan.counts.fill_(-1)
    plan.run(A, B)
    torch.cuda.synchronize()
    c = plan.result().counts()
    assert c["blocks"] == 64 and c["clean"] == 64 and c["checks_rounding"] == 2 * 64 * 32
    assert c["checks_critical"] == 0 and c["corrected"] == 0
