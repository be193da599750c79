#!/usr/bin/env python3
"""Mutation check of the oracle pins: apply one plausible mistake at a time to
oracle/aabft_oracle.c (in a scratch copy), rebuild, run the CPU pin suite, and require it to
go red.  The oracle source in the tree is never modified.

    python tools/oracle_mutations.py          # prints one line per mutation, exit 1 if any survives
"""
import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

MUTATIONS = [
    # (name, original text, mutated text)
    ("classify: sigma edge -> eps (drops TOLERABLE)", "if (a <= sig) return 0;", "if (a <= eps) return 0;"),
    ("classify: eps edge -> 2 eps", "if (a <= eps) return 1;", "if (a <= 2.0 * eps) return 1;"),
    ("EV term doubled (Eq 43)", "e = e + ((double)n / 3.0) * ldexp(y, -2 * t);",
     "e = e + 2.0 * ((double)n / 3.0) * ldexp(y, -2 * t);"),
    ("EV term dropped", "if (!fma_model) e = e + ((double)n / 3.0) * ldexp(y, -2 * t);", ""),
    ("site 3 sign (f64)", "if (site == 3 && k == k_step) c = c + add;",
     "if (site == 3 && k == k_step) c = c - add;"),
    ("site 3 sign (f32)", "if (site == 3 && k == k_step) c = (float)((double)c + add);",
     "if (site == 3 && k == k_step) c = (float)((double)c - add);"),
    ("site 1 at k_step+1", "if (site == 1 && k == k_step) c = of_bits(bits_of(c) ^ xor_mask);",
     "if (site == 1 && k == k_step + 1) c = of_bits(bits_of(c) ^ xor_mask);"),
    ("y: case 2 uses bmax", "double case2 = amax * bmin;", "double case2 = amax * bmax;"),
    ("sigma coeff /24 instead of /48", "F = ((dn * (dn + 1.0)) * (2.0 * dn + 1.0)) / 48.0;",
     "F = ((dn * (dn + 1.0)) * (2.0 * dn + 1.0)) / 24.0;"),
    ("encode: skip last row", "for (int64_t i = I * bs; i < I * bs + bs; ++i) s = s + ((const double *)A)[i * lda + k];",
     "for (int64_t i = I * bs; i < I * bs + bs - 1; ++i) s = s + ((const double *)A)[i * lda + k];"),
    ("top-p tie -> highest index", "if (v > best) { best = v; best_k = k; }",
     "if (v >= best) { best = v; best_k = k; }"),
    ("check: row ref uses Ccol", "double d = ref - ld(dtype, Crow, i * ld_crow + J);",
     "double d = ref - ld(dtype, Ccol, (i / bs) * ld_ccol + J);"),
    ("verdict: (1,1) not single", "else if (nr == 1 && nc == 1) status = 4;",
     "else if (nr == 1 && nc == 1) status = 3;"),
    ("correct: keep faulty element in sum", "if (ii != i) v = v - ld(dtype, C, ii * ldc + j);",
     "v = v - ld(dtype, C, ii * ldc + j);"),
]


def main():
    src = os.path.join(ROOT, "oracle", "aabft_oracle.c")
    text = open(src).read()
    survivors = 0
    for name, a, b in MUTATIONS:
        if a not in text:
            print(f"SKIP   {name}: pattern not found")
            survivors += 1
            continue
        with tempfile.TemporaryDirectory() as tmp:
            shutil.copytree(ROOT, os.path.join(tmp, "r"),
                            ignore=shutil.ignore_patterns(".git", "gpurun_out", "*.so", "build",
                                                          "profiles", "__pycache__"))
            r = os.path.join(tmp, "r")
            with open(os.path.join(r, "oracle", "aabft_oracle.c"), "w") as f:
                f.write(text.replace(a, b, 1))
            p = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "not gpu",
                                "tests/test_oracle_pins.py", "tests/test_oracle_classes.py",
                                "tests/test_oracle_comparators.py", "tests/test_oracle_hdr.py"],
                               cwd=r, capture_output=True, text=True)
            killed = p.returncode != 0
            survivors += not killed
            tail = p.stdout.strip().splitlines()[-1] if p.stdout.strip() else p.stderr[-200:]
            print(f"{'KILLED' if killed else 'SURVIVED'} {name}: {tail}")
    print(f"{len(MUTATIONS) - survivors}/{len(MUTATIONS)} mutations killed")
    return 1 if survivors else 0


if __name__ == "__main__":
    sys.exit(main())
