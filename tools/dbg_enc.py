import sys, numpy as np, torch
sys.path.insert(0, '.')
sys.path.insert(0, 'tests')
import synth
from oracle import oracle as orc
from paper_conf_dsn_braunhw14_b200 import api
from test_gpu_parity import to_dev, host
M, N, K, bs, p = 192, 320, 200, 64, 2
for dt in (np.float64, np.float32):
    A = synth.generate("uniform", M, K, seed=3, matrix_id=0, dtype=dt)
    B = synth.generate("wide", K, N, seed=3, matrix_id=1, dtype=dt)
    plan = api.ProtectedGemm(M, N, K, dtype=torch.float64 if dt == np.float64 else torch.float32, bs=bs, p=p)
    plan.encode(to_dev(A), to_dev(B)); torch.cuda.synchronize()
    enc = orc.encode(A, B, bs, p)
    g, o = host(plan.topA_val), enc["topA"][0]
    bad = np.argwhere(g != o)
    print(dt, "bad A", len(bad), bad[:5], [ (g[i,j], o[i,j]) for i,j in bad[:5]], host(plan.topA_idx)[bad[:3,0]] if len(bad) else '', enc["topA"][1][bad[:3,0]] if len(bad) else '')
    g, o = host(plan.topB_val), enc["topB"][0]
    print(dt, "bad B", len(np.argwhere(g != o)))
