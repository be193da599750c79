"""Protected-step time with and without AABFT_FLAG_OVERLAP_ENCODE (CUDA events, device time).

    python tools/time_overlap.py [M N K bs p steps]

Prints one JSON line: ms per protected step (encode -> gemm -> check -> correct) for the
overlapped and the serial launches, the unprotected GEMM, and the encode alone.
"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
import synth  # noqa: E402
from paper_conf_dsn_braunhw14_b200 import api  # noqa: E402


def timed(fn, steps):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / steps


def main():
    a = [int(x) for x in sys.argv[1:]]
    M, N, K, bs, p, steps = (a + [4096, 4096, 4096, 64, 2, 20][len(a):])[:6]
    A = torch.from_numpy(synth.generate("uniform", M, K, seed=1, matrix_id=0)).cuda()
    B = torch.from_numpy(synth.generate("uniform", K, N, seed=1, matrix_id=1)).cuda()
    C = torch.empty(M, N, dtype=torch.float64, device="cuda")
    out = {"shape": [M, N, K, bs, p]}
    for ov in (True, False):
        plan = api.ProtectedGemm(M, N, K, bs=bs, p=p, overlap=ov)
        out["step_ms_overlap" if ov else "step_ms_serial"] = timed(lambda: plan.run(A, B), steps)
        out["encode_ms_" + ("overlap_kernel" if ov else "serial_kernels")] = timed(
            lambda: plan.encode(A, B), steps)
        if not os.environ.get("NOASSERT"):
            assert plan.result().counts()["clean"] == (M // bs) * (N // bs)
    out["plain_ms"] = timed(lambda: api.gemm_plain(A, B, out=C), steps)
    fl = 2.0 * M * N * K
    out["tflops_overlap"] = fl / out["step_ms_overlap"] / 1e9
    out["tflops_serial"] = fl / out["step_ms_serial"] / 1e9
    out["tflops_plain"] = fl / out["plain_ms"] / 1e9
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
