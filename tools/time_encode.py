"""Time aabft_encode (with and without top-p) and aabft_check at c2 / c3 shapes (CUDA events)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
from paper_conf_dsn_braunhw14_b200 import api
n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
dt = sys.argv[2] if len(sys.argv) > 2 else "f64"
tdt, ndt = (torch.float64, np.float64) if dt == "f64" else (torch.float32, np.float32)
rec = "uniform" if dt == "f64" else "wide"
A = torch.from_numpy(synth.generate(rec, n, n, seed=1, matrix_id=0, dtype=ndt)).cuda()
B = torch.from_numpy(synth.generate(rec, n, n, seed=2, matrix_id=1, dtype=ndt)).cuda()
plan = api.ProtectedGemm(n, n, n, dtype=tdt, bs=64, p=2)
plan.run(A, B)
def t(fn, reps=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        # keep the GPU busy while the host enqueues, so the events bracket device time only
        # (on an idle stream e0 completes at once and the host's launch latency is counted)
        torch.cuda._sleep(2_000_000)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    return float(np.median(ts)) * 1e3
out = {"lib": os.environ.get("AABFT_LIB", "default"), "n": n, "dtype": dt,
       "encode_us": t(lambda: plan.encode(A, B)),
       "encode_cs_only_us": t(lambda: plan.encode(A, B, topp=False)),
       "encode_A_us": t(lambda: plan.encode(A, None)),
       "encode_B_us": t(lambda: plan.encode(None, B)),
       "check_us": t(plan.check)}
out["encode_GBps"] = 2 * n * n * A.element_size() / (out["encode_us"] * 1e-6) / 1e9
print(json.dumps(out))
