"""Small protected GEMMs for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
BASELINE configs[0] (128^3 FP64, BS 32) and a shape whose persistent schedule has a stream-K
tail (split tiles: partial slots, flags, the owner's spin-wait), fused and unfused checks, a
fault list, the FP32 path and the opt-in top-p selection inside the GEMM."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
from paper_conf_dsn_braunhw14_b200 import api

def run(M, N, K, bs, dt=np.float64, fused=True, topp_in_gemm=False, faults=None, overlap=False):
    A = torch.from_numpy(synth.generate("uniform", M, K, seed=1, matrix_id=0, dtype=dt)).cuda()
    B = torch.from_numpy(synth.generate("uniform", K, N, seed=2, matrix_id=1, dtype=dt)).cuda()
    td = torch.float64 if dt == np.float64 else torch.float32
    plan = api.ProtectedGemm(M, N, K, dtype=td, bs=bs, p=2, fused=fused, topp_in_gemm=topp_in_gemm,
                             overlap=overlap)
    r = plan.run(A, B, faults=faults)
    torch.cuda.synchronize()
    c = r.counts()
    print(M, N, K, bs, dt.__name__, fused, topp_in_gemm, c["blocks"], c["clean"], c["corrected"], flush=True)

run(128, 128, 128, 32)                                   # c1
f = [dict(row=3, col=200, site=2, add=1.0), dict(row=700, col=40, site=1, k_step=100, xor_mask=1 << 62)]
run(1024, 1088, 520, 64, faults=f)                       # stream-K tail, faults, fused
run(1024, 1088, 520, 64, fused=False, faults=f)          # unfused streaming check
run(1024, 1088, 520, 64, topp_in_gemm=True)              # top-p in the GEMM (stream-K partial lists)
run(512, 384, 300, 64, dt=np.float32, faults=f[:1])     # FP32 FFMA path
run(1024, 1088, 520, 64, overlap=True, faults=f)         # encode overlapped with the GEMM (PDL)
run(2048, 256, 96, 32, faults=f)                         # many check units per CTA (one-wave grid loop)
api.gemm_plain(torch.rand(512, 256, dtype=torch.float64, device="cuda"),
               torch.rand(256, 384, dtype=torch.float64, device="cuda"))
torch.cuda.synchronize()
print("done")
