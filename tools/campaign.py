#!/usr/bin/env python3
"""Fault-injection campaign on the sm_100a path (paper §VI-C).

One fault per BS x BS block per GEMM (each block is an independent trial: the partitioned
encoding makes blocks independent), through the C ABI's fault hooks (Alg 3):

* magnitude sweep: additive e = r * max(eps_col, eps_row), r = 2^(x/2), x = -12..12, both
  signs, at the final value (site 2, Alg 3 errorVecAdd2) and in the accumulator after
  k = K/2 (site 3, errorVecAdd1);
* bit sweep (Fig 4 style): single-bit XOR of every bit 0..63 of the final value (site 0) and
  of the accumulator after k = K/2 (site 1).

Labels: north_star contract -- "must detect" |e| > 2 max(eps_col, eps_row), "must be silent"
|e| < min(eps)/2 (R22); paper -- "critical" |e| > 3 sigma_ij of the element (sigma_ij
from aabft_bound_elements).  Realised e is measured (faulty run without correction minus the
clean run).  Writes JSON (and a markdown summary) to profiles/.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
from paper_conf_dsn_braunhw14_b200 import api  # noqa: E402

WL = {"c2": (4096, 4096, 4096, 64, "f64", "uniform"), "c1": (128, 128, 128, 32, "f64", "uniform"),
      "c3": (8192, 8192, 8192, 64, "f32", "wide"), "c2u100": (4096, 4096, 4096, 64, "f64", "uniform100"),
      # Eq 47 (Table IV / Fig 4's third workload): alpha = 0, kappa = 65536
      "c2hdr": (4096, 4096, 4096, 64, "f64", "hdr65536")}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c2", choices=sorted(WL))
    ap.add_argument("--seed", type=int, default=7)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r01_campaign"))
    ap.add_argument("--bits", default="all", help="'all' or comma list")
    args = ap.parse_args()
    M, N, K, bs, dts, recipe = WL[args.workload]
    ndt = np.float64 if dts == "f64" else np.float32
    tdt = torch.float64 if dts == "f64" else torch.float32
    ut = np.uint64 if dts == "f64" else np.uint32
    nbits = 64 if dts == "f64" else 32
    mant_bits = 52 if dts == "f64" else 23

    from fig4 import make_input  # seeded recipes, or Eq 47 assembled on the device
    A = make_input(recipe, M, K, 1, 0, ndt)
    B = make_input(recipe, K, N, 2, 1, ndt)
    plan = api.ProtectedGemm(M, N, K, dtype=tdt, bs=bs, p=2)
    res = plan.run(A, B)
    torch.cuda.synchronize()
    clean_counts = res.counts()
    C0 = res.C.detach().cpu().numpy().copy()
    b = plan.bound()
    eps_col = b["eps_col"].cpu().numpy()
    eps_row = b["eps_row"].cpu().numpy()
    nI, nJ = M // bs, N // bs
    rng = np.random.default_rng(args.seed)

    def positions():
        I, J = np.meshgrid(np.arange(nI), np.arange(nJ), indexing="ij")
        i = (I * bs + rng.integers(0, bs, I.shape)).ravel()
        j = (J * bs + rng.integers(0, bs, J.shape)).ravel()
        return i, j

    def inject(faults, correct):
        fb = api.make_faults(faults, "cuda")
        r = plan.run(A, B, faults=fb, correct=correct)
        torch.cuda.synchronize()
        return r.reports()["status"].ravel().copy(), r.C.detach().cpu().numpy()

    def sigma_of(i, j):
        sig, _ = plan.bound_elements(torch.from_numpy(i), torch.from_numpy(j))
        return sig.cpu().numpy()

    out = {"workload": args.workload, "M": M, "N": N, "K": K, "bs": bs, "dtype": dts,
           "recipe": recipe, "blocks": nI * nJ, "clean": clean_counts, "magnitude": [], "bits": []}
    t0 = time.time()
    # ------------------------------------------------------------------ magnitude sweep
    for site in (2, 3):
        for x in range(-12, 13):
            r = 2.0 ** (x / 2)
            for sign in (1, -1):
                i, j = positions()
                I, J = i // bs, j // bs
                hi = np.maximum(eps_col[I, j], eps_row[i, J])
                lo = np.minimum(eps_col[I, j], eps_row[i, J])
                add = sign * r * hi
                faults = [dict(row=int(a), col=int(c), site=site, k_step=K // 2, add=float(e))
                          for a, c, e in zip(i, j, add)]
                st_nc, C1 = inject(faults, correct=False)
                e_real = C1[i, j].astype(np.float64) - C0[i, j].astype(np.float64)
                st, C2 = inject(faults, correct=True)
                must = np.abs(e_real) > 2 * hi
                silent = np.abs(e_real) < 0.5 * lo
                det = st != 0
                corr = st == 1
                restored = np.abs(C2[i, j] - C0[i, j]) <= eps_col[I, j]
                out["magnitude"].append(dict(
                    site=site, r=r, sign=sign, faults=len(faults),
                    must_detect=int(must.sum()), detected_of_must=int((det & must).sum()),
                    corrected_of_must=int((corr & must & restored).sum()),
                    must_silent=int(silent.sum()), silent_ok=int((~det & silent).sum()),
                    band=int((~must & ~silent).sum()), detected_in_band=int((det & ~must & ~silent).sum())))
    # ------------------------------------------------------------------ bit sweep (Fig 4)
    bits = range(nbits) if args.bits == "all" else [int(v) for v in args.bits.split(",")]
    for site in (0, 1):
        for bit in bits:
            i, j = positions()
            faults = [dict(row=int(a), col=int(c), site=site, k_step=K // 2, xor_mask=1 << bit)
                      for a, c in zip(i, j)]
            _, C1 = inject(faults, correct=False)
            st, C2 = inject(faults, correct=True)
            I, J = i // bs, j // bs
            with np.errstate(all="ignore"):
                e_real = C1[i, j].astype(np.float64) - C0[i, j].astype(np.float64)
            hi = np.maximum(eps_col[I, j], eps_row[i, J])
            sig = sigma_of(i, j)
            finite = np.isfinite(e_real)
            crit = ~finite | (np.abs(e_real) > 3 * sig)              # paper
            must = ~finite | (np.abs(e_real) > 2 * hi)                # contract (north_star)
            det = st != 0
            field = "sign" if bit == nbits - 1 else ("exponent" if bit >= mant_bits else "mantissa")
            out["bits"].append(dict(
                site=site, bit=bit, field=field, faults=len(faults),
                critical=int(crit.sum()), detected_of_critical=int((det & crit).sum()),
                must_detect=int(must.sum()), detected_of_must=int((det & must).sum()),
                corrected=int((st == 1).sum()), detected=int(det.sum())))
    out["seconds"] = time.time() - t0

    # ------------------------------------------------------------------ summary
    def rate(rows, num, den):
        d = sum(r[den] for r in rows)
        return (sum(r[num] for r in rows) / d) if d else None

    mag, bit = out["magnitude"], out["bits"]
    summ = {
        "contract_detection_rate": rate(mag + bit, "detected_of_must", "must_detect"),
        "contract_must_detect": sum(r["must_detect"] for r in mag + bit),
        "contract_correction_rate_magnitude": rate(mag, "corrected_of_must", "must_detect"),
        "silent_ok_rate": rate(mag, "silent_ok", "must_silent"),
        "false_positives_clean": clean_counts["checks_critical"],
    }
    for site in (0, 1):
        for fld in ("sign", "exponent", "mantissa"):
            rows = [r for r in bit if r["site"] == site and r["field"] == fld]
            summ[f"paper_detected_of_critical_site{site}_{fld}"] = rate(rows, "detected_of_critical", "critical")
            summ[f"critical_fraction_site{site}_{fld}"] = (sum(r["critical"] for r in rows) /
                                                          max(1, sum(r["faults"] for r in rows)))
    out["summary"] = summ
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out + f"_{args.workload}.json", "w") as f:
        json.dump(out, f, indent=1)
    lines = [f"# Fault campaign {args.workload}: {M}x{N}x{K} {dts} BS {bs}, {recipe}, one fault per block "
             f"({nI * nJ} trials per GEMM), {out['seconds']:.0f} s", "",
             "| quantity | value |", "|---|---|"]
    for k, v in summ.items():
        lines.append(f"| {k} | {v if v is None or isinstance(v, int) else round(v, 5)} |")
    lines += ["", "Bit sweep (paper metric: detected among |e| > 3 sigma_ij; contract: among |e| > 2 eps):", "",
              "| site | bit | field | critical | detected/critical | must | detected/must |", "|---|---|---|---|---|---|---|"]
    for r in bit:
        dc = r["detected_of_critical"] / r["critical"] if r["critical"] else float("nan")
        dm = r["detected_of_must"] / r["must_detect"] if r["must_detect"] else float("nan")
        lines.append(f"| {r['site']} | {r['bit']} | {r['field']} | {r['critical']} | {dc:.4f} | {r['must_detect']} | {dm:.4f} |")
    with open(args.out + f"_{args.workload}.md", "w") as f:
        f.write("\n".join(lines) + "\n")
    print(json.dumps(summ))


if __name__ == "__main__":
    main()
