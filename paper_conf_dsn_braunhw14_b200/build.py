"""Build the sm_100a C-ABI library ``libaabft.so`` in-tree with nvcc (no JIT cache).

``python -m paper_conf_dsn_braunhw14_b200.build`` or ``__graft_entry__.build()``.
"""
from __future__ import annotations

import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
OUT = os.environ.get("AABFT_BUILD_OUT", os.path.join(HERE, "libaabft.so"))
OBJ = os.environ.get("AABFT_BUILD_OBJ", os.path.join(HERE, "build"))
SOURCES = ["api.cu", "encode.cu", "check.cu", "gemm_f64.cu", "gemm_f32.cu", "study.cu", "sea.cu"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC,-ffp-contract=off", "-Xptxas", "-v", "-I", os.path.join(HERE, "..", "include"),
         *os.environ.get("AABFT_EXTRA_FLAGS", "").split()]


def _stale(obj: str, deps) -> bool:
    if not os.path.exists(obj):
        return True
    t = os.path.getmtime(obj)
    return any(os.path.getmtime(d) > t for d in deps)


def build(verbose: bool = False, force: bool = False) -> str:
    os.makedirs(OBJ, exist_ok=True)
    headers = [os.path.join(CSRC, "common.cuh"), os.path.join(HERE, "..", "include", "aabft.h")]
    jobs = []
    for src in SOURCES:
        s = os.path.join(CSRC, src)
        o = os.path.join(OBJ, src.replace(".cu", ".o"))
        if force or _stale(o, [s, *headers]):
            jobs.append((s, o))

    def compile_one(job):
        s, o = job
        r = subprocess.run([NVCC, *FLAGS, "-c", s, "-o", o], capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {s}:\n{r.stdout}\n{r.stderr}")
        with open(o + ".ptxas.txt", "w") as f:
            f.write(r.stderr)
        return s

    with ThreadPoolExecutor(max_workers=len(jobs) or 1) as ex:
        for s in ex.map(compile_one, jobs):
            if verbose:
                print("compiled", os.path.basename(s))
    objs = [os.path.join(OBJ, s.replace(".cu", ".o")) for s in SOURCES]
    if force or jobs or _stale(OUT, objs):
        subprocess.check_call([NVCC, "-shared", "-cudart", "static", "-o", OUT, *objs,
                               "-gencode", "arch=compute_100a,code=sm_100a"])
    return OUT


if __name__ == "__main__":
    print(build(verbose=True, force="--force" in sys.argv))
