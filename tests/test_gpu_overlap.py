"""AABFT_FLAG_OVERLAP_ENCODE: the encode grid running concurrently with the GEMM.

The flagged path (one 64-thread CTA per SM, complete-vector units, programmatic dependent launch
of the GEMM) must give the oracle's encoding bit for bit (Alg 1: the
sequential sums of Eq 1 / Eq 2 and the sequential top-p scan), and the whole protected product
must equal the unflagged run bit for bit (same GEMM kernel; only the launch overlap differs).
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


def to_dev(X):
    X = np.ascontiguousarray(X)
    r, c = X.shape
    ld = (c + 1) // 2 * 2
    buf = torch.zeros(r, ld, dtype=torch.float64, device="cuda")
    buf[:, :c] = torch.from_numpy(X).cuda()
    return buf[:, :c]


def host(t):
    return t.detach().cpu().numpy()


OVERLAP_SHAPES = [
    # M, N, K, bs, p -- every unit kind, ragged edges, more units than SMs
    (128, 128, 128, 32, 2),     # c1-like
    (192, 320, 200, 64, 2),     # N not a multiple of 64 (last B unit ragged), K % 16 = 8
    (64, 96, 37, 16, 3),        # K < 64 (one ragged A chunk), bs = 16 (4 blocks per B unit)
    (48, 80, 5, 16, 4),         # K < 16: one ragged tile per unit, p = 4
    (256, 256, 4099, 32, 3),    # odd K, many chunks
    (9600, 64, 48, 64, 1),      # 150 A units + 1 B unit: more units than SMs (2nd round)
    (64, 12800, 300, 64, 2),    # 200 B units
    (1024, 1024, 2048, 64, 4),  # stream-K GEMM tail; bigger units
]


@pytest.mark.parametrize("overlap", [True, False])
@pytest.mark.parametrize("shape", OVERLAP_SHAPES)
def test_overlap_encode_bit_exact(P, orc, shape, overlap):
    """overlap=True: the co-resident encode grid; overlap=False: the default chunked kernels
    (encode_ab + topp_reduce) at the same ragged shapes."""
    M, N, K, bs, p = shape
    A = synth.generate("uniform", M, K, seed=11, matrix_id=0)
    B = synth.generate("wide", K, N, seed=11, matrix_id=1)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p, overlap=overlap)
    assert plan.overlap == overlap
    plan.topA_val.fill_(-7.0)
    plan.topB_idx.fill_(-7)
    plan.encode(to_dev(A), to_dev(B))
    torch.cuda.synchronize()
    enc = orc.encode(A, B, bs, p)
    assert np.array_equal(host(plan.Acs), enc["Acs"])
    assert np.array_equal(host(plan.Bcs), enc["Bcs"])
    assert np.array_equal(host(plan.topA_val), enc["topA"][0])
    assert np.array_equal(host(plan.topA_idx), enc["topA"][1])
    assert np.array_equal(host(plan.topB_val), enc["topB"][0])
    assert np.array_equal(host(plan.topB_idx), enc["topB"][1])


@pytest.mark.parametrize("overlap", [True, False])
@pytest.mark.parametrize("bs", [16, 32, 64])
def test_overlap_encode_ties_integer_data(P, orc, bs, overlap):
    """Many equal |values|: lowest index wins in every merge of the complete-vector units."""
    M, N, K, p = 128, 192, 333, 4
    A = synth.generate("integer", M, K, seed=12, matrix_id=0, q=2)
    B = synth.generate("integer", K, N, seed=12, matrix_id=1, q=2)
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p, overlap=overlap)
    plan.encode(to_dev(A), to_dev(B))
    torch.cuda.synchronize()
    enc = orc.encode(A, B, bs, p)
    for name, o in (("topA", enc["topA"]), ("topB", enc["topB"])):
        assert np.array_equal(host(getattr(plan, name + "_idx")), o[1]), name
        assert np.array_equal(host(getattr(plan, name + "_val")), o[0]), name
    assert np.array_equal(host(plan.Acs), enc["Acs"])
    assert np.array_equal(host(plan.Bcs), enc["Bcs"])


@pytest.mark.parametrize("shape", [(128, 128, 128, 32, 2), (1024, 1024, 2048, 64, 2),
                                   (2048, 1536, 1000, 64, 3)])
@pytest.mark.parametrize("faults", [False, True])
def test_overlap_run_equals_serial_run(P, shape, faults):
    """encode -> gemm (PDL) -> check -> correct: C, carried checksums, reports and counters
    identical to the serial launches, also with the fault-injection GEMM instantiation."""
    M, N, K, bs, p = shape
    A = to_dev(synth.generate("uniform", M, K, seed=13, matrix_id=0))
    B = to_dev(synth.generate("uniform", K, N, seed=13, matrix_id=1))
    fl = [dict(row=3, col=5, site=2, add=1.0), dict(row=M - 1, col=N - 2, site=0, xor_mask=1 << 62)] \
        if faults else None
    out = []
    for ov in (True, False):
        plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p, overlap=ov)
        for _ in range(2):  # a second run re-uses the re-armed split-K flags
            res = plan.run(A, B, faults=fl)
        torch.cuda.synchronize()
        out.append((host(res.C).copy(), host(res.Ccol).copy(), host(res.Crow).copy(),
                    host(res.report_buf).copy(), res.counts(), host(res.topA_idx).copy()))
    a, b = out
    for x, y in zip(a, b):
        if isinstance(x, dict):
            assert x == y
        else:
            assert np.array_equal(x, y)
    if faults:
        assert a[4]["corrected"] == 2
    else:
        assert a[4]["clean"] == a[4]["blocks"]


def test_overlap_graph_capture(P):
    """The overlapped launches record into a CUDA graph and replay bit-identically."""
    M, N, K, bs, p = 512, 512, 512, 64, 2
    A = to_dev(synth.generate("uniform", M, K, seed=14, matrix_id=0))
    B = to_dev(synth.generate("uniform", K, N, seed=14, matrix_id=1))
    plan = P.ProtectedGemm(M, N, K, dtype=torch.float64, bs=bs, p=p, overlap=True)
    plan.run(A, B)
    torch.cuda.synchronize()
    C0 = host(plan.C).copy()
    g = plan.capture(A, B)
    plan.C.fill_(0.0)
    g.replay()
    torch.cuda.synchronize()
    assert np.array_equal(host(plan.C), C0)
    assert plan.result().counts()["clean"] == (M // bs) * (N // bs)
