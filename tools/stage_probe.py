"""Device time of each protected-path stage alone (CUDA events around R back-to-back calls of
one stage, so launch gaps are hidden behind queued work) -- for tuning encode / check."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
from paper_conf_dsn_braunhw14_b200 import api

n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
dt = sys.argv[2] if len(sys.argv) > 2 else "f64"
bs = int(sys.argv[3]) if len(sys.argv) > 3 else 64
tdt, ndt = (torch.float64, np.float64) if dt == "f64" else (torch.float32, np.float32)
A = torch.from_numpy(synth.generate("uniform", n, n, seed=1, matrix_id=0, dtype=ndt)).cuda()
B = torch.from_numpy(synth.generate("uniform", n, n, seed=2, matrix_id=1, dtype=ndt)).cuda()
plan = api.ProtectedGemm(n, n, n, dtype=tdt, bs=bs, p=2)
plan.run(A, B)
torch.cuda.synchronize()


def t(fn, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3  # us


es = 8 if dt == "f64" else 4
out = {"n": n, "dtype": dt, "bs": bs}
out["encode_us"] = t(lambda: plan.encode(A, B))
out["encode_A_us"] = t(lambda: plan.encode(A, None))
out["encode_B_us"] = t(lambda: plan.encode(None, B))
out["encode_cs_only_us"] = t(lambda: plan.encode(A, B, topp=False))
out["encode_GBps_A+B"] = 2 * n * n * es / (out["encode_us"] * 1e3)
out["check_us"] = t(plan.check)
out["correct_us"] = t(plan.correct)
out["gemm_us"] = t(lambda: plan.gemm(A, B), reps=5)
out["step_us"] = t(lambda: plan.run(A, B), reps=5)
print(json.dumps(out))
