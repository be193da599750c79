"""Timeline of one overlapped protected step (build with -DAABFT_OV_PROBE; AABFT_LIB=that .so):
encode grid start/end and GEMM first-CTA start / encode-wait return / end, in us."""
import ctypes as C
import os
import sys

import torch

sys.path.insert(0, os.path.join(os.path.dirname(__file__), ".."))
import synth  # noqa: E402
from paper_conf_dsn_braunhw14_b200 import api, _abi  # noqa: E402

a = [int(x) for x in sys.argv[1:]]
M, N, K, bs, p = (a + [4096, 4096, 4096, 64, 2][len(a):])[:5]
A = torch.from_numpy(synth.generate("uniform", M, K, seed=1, matrix_id=0)).cuda()
B = torch.from_numpy(synth.generate("uniform", K, N, seed=1, matrix_id=1)).cuda()
L = _abi.lib()
plan = api.ProtectedGemm(M, N, K, bs=bs, p=p, overlap=True)
for it in range(4):
    e = (C.c_ulonglong * 2)()
    g = (C.c_ulonglong * 3)()
    torch.cuda.synchronize()
    L.aabft_debug_ov_probe(e)
    L.aabft_debug_gemm_probe(g)
    plan.run(A, B)
    torch.cuda.synchronize()
    L.aabft_debug_ov_probe(e)
    L.aabft_debug_gemm_probe(g)
    t0 = e[0]
    print(f"encode {0:.1f}..{(e[1]-t0)/1e3:.1f} us; gemm start {(g[0]-t0)/1e3:.1f}, "
          f"latest encode-wait return {(g[2]-t0)/1e3:.1f}, end {(g[1]-t0)/1e3:.1f} us")
