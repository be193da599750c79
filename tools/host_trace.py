"""One aabft_protected_gemm_host call at a bench workload with AABFT_HOST_TRACE=1 (event timeline
on stderr): where the end-to-end step's time goes."""
import ctypes as C, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["AABFT_HOST_TRACE"] = "1"
import numpy as np, torch, synth
from paper_conf_dsn_braunhw14_b200 import _abi
n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
A = torch.from_numpy(synth.generate("uniform", n, n, seed=1, matrix_id=0)).pin_memory()
B = torch.from_numpy(synth.generate("uniform", n, n, seed=2, matrix_id=1)).pin_memory()
Ch = torch.empty(n, n, dtype=torch.float64).pin_memory()
cfg = _abi.Config(0, 64, n, n, n, 2, 0, 3.0, 1, 0)
L = _abi.lib()
nb = L.aabft_host_arena_bytes(C.byref(cfg))
arena = torch.empty(nb, dtype=torch.uint8, device="cuda")
cnt = _abi.Counts()
st = torch.cuda.current_stream().cuda_stream
for _ in range(3):
    _abi.ok(L.aabft_protected_gemm_host(C.byref(cfg), A.data_ptr(), B.data_ptr(), Ch.data_ptr(),
                                        C.addressof(cnt), arena.data_ptr(), nb, st), "host")
