"""Minimal driver for ncu: c2-shaped protected GEMM (encode, gemm, check, correct) x N."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, numpy as np, synth
from paper_conf_dsn_braunhw14_b200 import api
n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
dt = sys.argv[3] if len(sys.argv) > 3 else "f64"
tdt, ndt = (torch.float64, np.float64) if dt == "f64" else (torch.float32, np.float32)
A = torch.from_numpy(synth.generate("uniform", n, n, seed=1, matrix_id=0, dtype=ndt)).cuda()
B = torch.from_numpy(synth.generate("uniform", n, n, seed=2, matrix_id=1, dtype=ndt)).cuda()
plan = api.ProtectedGemm(n, n, n, dtype=tdt, bs=64, p=2)
for _ in range(reps):
    plan.run(A, B)
    api.gemm_plain(A, B)
torch.cuda.synchronize()
print("ok", plan.counts.cpu().tolist())
