"""Device time of the check stage alone (and check + correct) at a config, CUDA events.

    python tools/time_check.py [M N K bs p dtype]
"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
import synth  # noqa: E402
from paper_conf_dsn_braunhw14_b200 import api  # noqa: E402


def timed(fn, steps=50):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / steps * 1e3


a = sys.argv[1:]
M, N, K, bs, p = [int(x) for x in (a + ["4096", "4096", "4096", "64", "2"][len(a):])[:5]]
dt = torch.float64 if (a[5:] or ["f64"])[0] == "f64" else torch.float32
A = torch.from_numpy(synth.generate("uniform", M, K, seed=1, matrix_id=0)).to(dt).cuda()
B = torch.from_numpy(synth.generate("uniform", K, N, seed=1, matrix_id=1)).to(dt).cuda()
plan = api.ProtectedGemm(M, N, K, dtype=dt, bs=bs, p=p)
plan.run(A, B)
torch.cuda.synchronize()
out = {"shape": [M, N, K, bs, p, str(dt)]}
out["check_us"] = timed(lambda: plan.check())
out["check_then_correct_us"] = timed(lambda: (plan.check(), plan.correct()))
try:
    out["check_correcting_us"] = timed(lambda: plan.check(correct=True))
except TypeError:
    pass
out["counts"] = plan.result().counts()
print(json.dumps(out))
