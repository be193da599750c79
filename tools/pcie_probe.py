"""PCIe facts for the end-to-end entry: pinned H2D / D2H rates alone and concurrently."""
import json
import torch
MiB = 1 << 20
a = torch.empty(256 * MiB, dtype=torch.uint8).pin_memory()
c = torch.empty(128 * MiB, dtype=torch.uint8).pin_memory()
da = torch.empty(256 * MiB, dtype=torch.uint8, device="cuda")
dc = torch.empty(128 * MiB, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def t(fn, reps=5):
    fn(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps
out = {}
ms = t(lambda: da.copy_(a, non_blocking=True)); out["h2d_GBps"] = 256 * MiB / ms / 1e6
ms = t(lambda: c.copy_(dc, non_blocking=True)); out["d2h_GBps"] = 128 * MiB / ms / 1e6
def both():
    with torch.cuda.stream(s1):
        da.copy_(a, non_blocking=True)
    with torch.cuda.stream(s2):
        c.copy_(dc, non_blocking=True)
ms = t(both); out["both_ms"] = ms; out["both_h2d_only_ms"] = 256 * MiB / out["h2d_GBps"] / 1e6
# strided 2D (B panel: 4096 rows x 8 KiB of a 32 KiB pitch)
import ctypes, glob, os
rt = ctypes.CDLL(glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia",
                                        "cuda_runtime", "lib", "libcudart.so.*"))[0])
H2D = 1
def panels():
    st = ctypes.c_void_p(torch.cuda.current_stream().cuda_stream)
    for j in range(4):  # B (4096 x 4096 f64) as 4 column panels of 1024 columns
        rc = rt.cudaMemcpy2DAsync(ctypes.c_void_p(da.data_ptr() + j * 8192), ctypes.c_size_t(32768),
                                  ctypes.c_void_p(a.data_ptr() + j * 8192), ctypes.c_size_t(32768),
                                  ctypes.c_size_t(8192), ctypes.c_size_t(4096 * 2), H2D, st)
        assert rc == 0, rc
ms = t(panels); out["h2d_2d_panels_GBps"] = 256 * MiB / ms / 1e6
def panels_both():
    with torch.cuda.stream(s2):
        c.copy_(dc, non_blocking=True)
    with torch.cuda.stream(s1):
        panels()
ms = t(panels_both); out["panels_plus_d2h_ms"] = ms
print(json.dumps(out))
