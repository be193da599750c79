"""Plain FP64 GEMM rate at shapes whose tile count is an exact multiple of the persistent grid
(no stream-K tail) vs the c2 shape: separates steady-state losses from tail / fix-up losses."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_dsn_braunhw14_b200 import api
def t(fn, reps=10):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))
SHAPES = [(4096, 4096, 4096), (9472, 3072, 4096), (9472, 3072, 1024), (9472, 6144, 4096), (4736, 3072, 8192)]
if len(sys.argv) > 1:
    SHAPES = [tuple(int(x) for x in a.split('x')) for a in sys.argv[1:]]
for M, N, K in SHAPES:
    A = torch.rand(M, K, dtype=torch.float64, device="cuda"); B = torch.rand(K, N, dtype=torch.float64, device="cuda")
    C = torch.empty(M, N, dtype=torch.float64, device="cuda")
    ms = t(lambda: api.gemm_plain(A, B, out=C))
    mc = t(lambda: torch.matmul(A, B))
    print(json.dumps({"lib": os.environ.get("AABFT_LIB", "default"), "M": M, "N": N, "K": K, "tiles": (M // 64) * (N // 64),
                      "plain_tflops": 2 * M * N * K / ms / 1e9, "cublas_tflops": 2 * M * N * K / mc / 1e9}))
