#!/usr/bin/env python3
"""SASS mnemonic counts per kernel of the built libaabft.so (cuobjdump -sass): the evidence
that the FP64 GEMM issues DMMA fed by TMA (UTMALDG) and mbarrier waits (SYNCS), the FP32 GEMM
FFMA2, and that the encode top-p runs on the integer ALU (ISETP/SEL, no DSETP).

    python tools/sass_counts.py [lib] > profiles/r02_sass_counts.md
"""
import collections
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "paper_conf_dsn_braunhw14_b200", "libaabft.so")
KEEP = ["DMMA", "UTMALDG", "SYNCS", "FFMA2", "FFMA", "DFMA", "DADD", "DMUL", "DSETP", "ISETP",
        "SEL", "LDS", "LDG", "STG", "STS", "SHFL", "ATOMG", "RED", "BAR", "LDL", "STL"]


def main():
    sass = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True).stdout
    kern, counts = None, collections.OrderedDict()
    for line in sass.splitlines():
        m = re.match(r"\s+Function : (\S+)", line)
        if m:
            kern = m.group(1)
            counts[kern] = collections.Counter()
            continue
        m = re.match(r"\s+/\*[0-9a-f]+\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9]*)", line)
        if m and kern:
            counts[kern][m.group(1)] += 1
    demangled = {}
    try:
        out = subprocess.run(["c++filt"], input="\n".join(counts), capture_output=True, text=True).stdout
        demangled = dict(zip(counts, out.splitlines()))
    except Exception:
        pass
    print(f"# SASS mnemonic counts (static, per kernel) of `{os.path.relpath(LIB, ROOT)}`\n")
    print("Produced by `tools/sass_counts.py` (cuobjdump -sass).  Static instruction counts per "
          "kernel body, not executed counts.\n")
    print("| kernel | " + " | ".join(KEEP) + " |")
    print("|---|" + "---|" * len(KEEP))
    for k, c in counts.items():
        name = demangled.get(k, k)
        name = name.replace("aabft::(anonymous namespace)::", "").replace("void ", "")
        name = re.sub(r">\(.*", ">", name)
        print(f"| `{name}` | " + " | ".join(str(c.get(op, 0)) for op in KEEP) + " |")


if __name__ == "__main__":
    main()
