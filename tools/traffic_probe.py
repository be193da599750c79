"""One protected step of a bench workload, for `ncu --metrics dram__bytes_*` (bench.py's
roofline.traffic): runs encode -> gemm -> check -> correct twice; the second GEMM launch is
the measured one (the first warms up one-time setup)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
from paper_conf_dsn_braunhw14_b200 import api
M, N, K, bs, dt, recipe = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), sys.argv[5], sys.argv[6]
ndt, tdt = (np.float64, torch.float64) if dt == "f64" else (np.float32, torch.float32)
A = torch.empty(M, K, dtype=tdt, device="cuda")
for r0 in range(0, M, 2048):
    n = min(2048, M - r0)
    A[r0:r0 + n] = torch.from_numpy(synth.generate(recipe, n, K, seed=1, matrix_id=0, dtype=ndt, row0=r0, full_cols=K)).cuda()
B = torch.from_numpy(synth.generate(recipe, K, N, seed=2, matrix_id=1, dtype=ndt)).cuda()
plan = api.ProtectedGemm(M, N, K, dtype=tdt, bs=bs, p=2)
for _ in range(2):
    plan.run(A, B)
torch.cuda.synchronize()
print("ok")
