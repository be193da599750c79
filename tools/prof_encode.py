"""Driver for ncu: encode variants at c2 shape (full top-p, checksums only)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, numpy as np, synth
from paper_conf_dsn_braunhw14_b200 import api
n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
A = torch.from_numpy(synth.generate("uniform", n, n, seed=1, matrix_id=0)).cuda()
B = torch.from_numpy(synth.generate("uniform", n, n, seed=2, matrix_id=1)).cuda()
plan = api.ProtectedGemm(n, n, n, dtype=torch.float64, bs=64, p=2)
for _ in range(2):
    plan.encode(A, B, topp=False)
    plan.encode(A, B)
torch.cuda.synchronize()
print("ok")
