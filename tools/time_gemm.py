"""Time the augmented GEMM and the plain GEMM alone (CUDA events, median) for tuning."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, numpy as np, synth
from paper_conf_dsn_braunhw14_b200 import api
n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
dt = sys.argv[2] if len(sys.argv) > 2 else "f64"
tdt, ndt = (torch.float64, np.float64) if dt == "f64" else (torch.float32, np.float32)
A = torch.from_numpy(synth.generate("uniform", n, n, seed=1, matrix_id=0, dtype=ndt)).cuda()
B = torch.from_numpy(synth.generate("uniform", n, n, seed=2, matrix_id=1, dtype=ndt)).cuda()
plan = api.ProtectedGemm(n, n, n, dtype=tdt, bs=64, p=2)
plan.encode(A, B)
Cp = torch.empty(n, n, dtype=tdt, device="cuda")
def t(fn, reps=10):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))
tg = t(lambda: plan.gemm(A, B))
def gemm_tp():
    plan._topp_pending = True  # AABFT_FLAG_TOPP_IN_GEMM: the GEMM selects the top-p
    plan.gemm(A, B)
ttp = t(gemm_tp)
tp = t(lambda: api.gemm_plain(A, B, out=Cp))
tc = t(lambda: torch.matmul(A, B))
fl = 2.0 * n ** 3
aug = 2.0 * n * (n * n + 2 * (n // 64) * n)
print(json.dumps({"lib": os.environ.get("AABFT_LIB", "default"), "n": n, "dtype": dt,
                  "gemm_ms": tg, "gemm_topp_ms": ttp, "gemm_topp_aug_tflops": aug / ttp / 1e9, "gemm_aug_tflops": aug / tg / 1e9, "gemm_useful_tflops": fl / tg / 1e9,
                  "plain_ms": tp, "plain_tflops": fl / tp / 1e9, "cublas_tflops": fl / tc / 1e9}))
