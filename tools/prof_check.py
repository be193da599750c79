"""ncu driver: c2 protected step x2 (the check kernel's launches are the ones to capture)."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import synth  # noqa: E402
from paper_conf_dsn_braunhw14_b200 import api  # noqa: E402
n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
dt = torch.float64 if (sys.argv[2:] or ["f64"])[0] == "f64" else torch.float32
A = torch.from_numpy(synth.generate("uniform", n, n, seed=1, matrix_id=0)).to(dt).cuda()
B = torch.from_numpy(synth.generate("uniform", n, n, seed=2, matrix_id=1)).to(dt).cuda()
plan = api.ProtectedGemm(n, n, n, dtype=dt, bs=64, p=2)
for _ in range(3):
    plan.run(A, B)
torch.cuda.synchronize()
print("ok", plan.result().counts())
