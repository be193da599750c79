#!/usr/bin/env python3
"""Fig 4 experiment on the sm_100a path (NEXT-2 + NEXT-3; paper §VI-C).

Per-operation fault injection (Alg 3) into the protected GEMM and the detection rate of
A-ABFT next to SEA-ABFT over the SAME faulty products:

* operations: final-sum addition (site 0, "errorVecAdd2"), inner-loop addition (site 1,
  "errorVecAdd1") and -- on the FP32 FFMA path, where products are separate instructions --
  inner-loop multiplication (site 4, "errorVecMul");  FP64 runs on the DMMA tensor pipe, whose
  products are not addressable, and its site 1 acts after the 16-step k-tile (R23);
* single-bit flips and 3- / 5-bit flips with the paper's neighbourhood rule (two
  random positions, the remaining flips at random positions between them; reading R27), in
  the mantissa (Fig 4 shows mantissa flips; sign / exponent flips are reported separately --
  "A-ABFT, as well as SEA-ABFT detected all faults ... injected into the sign bit or the
  exponent");
* one fault per BS x BS block per GEMM (each block an independent trial), k_step
  uniform in [0, K);
* "critical" = |e| > 3 sigma_ij of the affected element (with "smaller" read as
  "larger", reading R19), sigma_ij from the A-ABFT bound of row a_i and column b_j
  (aabft_bound_elements); e is the realised error (faulty minus clean, on the device);
* detected = the block's verdict is not CLEAN under the scheme's bound: A-ABFT (aabft_check)
  or SEA-ABFT (aabft_sea_bound + aabft_check_ext) on the same product (no correction).

Writes profiles/<out>_<dtype>.json and .md.
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


def flip_masks(rng, n, nflips, lo_bit, hi_bit):
    """n XOR masks with `nflips` bits in [lo_bit, hi_bit): single bit uniform; multi-bit: two
    distinct random end positions at least nflips-1 apart, the other nflips-2 flips at distinct
    random positions strictly between them (reading R27)."""
    width = hi_bit - lo_bit
    if nflips == 1:
        return np.uint64(1) << (lo_bit + rng.integers(0, width, n)).astype(np.uint64)
    a = np.empty(n, np.int64)
    b = np.empty(n, np.int64)
    todo = np.arange(n)
    while todo.size:  # rejection: distinct ends with room for the middle flips
        x = rng.integers(0, width, todo.size)
        y = rng.integers(0, width, todo.size)
        lo, hi = np.minimum(x, y), np.maximum(x, y)
        okm = hi - lo - 1 >= nflips - 2
        a[todo[okm]], b[todo[okm]] = lo[okm], hi[okm]
        todo = todo[~okm]
    pos = np.arange(width)[None, :]
    keys = rng.random((n, width))
    keys[(pos <= a[:, None]) | (pos >= b[:, None])] = np.inf  # only strictly between the ends
    mid = np.argsort(keys, axis=1)[:, : nflips - 2]
    m = (np.uint64(1) << (lo_bit + a).astype(np.uint64)) | (np.uint64(1) << (lo_bit + b).astype(np.uint64))
    for c in range(nflips - 2):
        m |= np.uint64(1) << (lo_bit + mid[:, c]).astype(np.uint64)
    return m


def make_input(recipe, rows, cols, seed, mid, ndt):
    """Seeded inputs on the device.  'hdr<kappa>' is Eq 47 (Table IV; the paper's
    third Fig 4 workload: alpha = 0, kappa = 65536), A = 10^alpha U D_kappa V^T
    (reading R28) assembled on the device from the seeded host factors (input generation,
    not the protected path)."""
    if recipe.startswith("hdr"):
        Ud, V = synth.hdr_factors(rows, cols, seed=seed, matrix_id=mid, kappa=float(recipe[3:]),
                                  alpha=0.0)
        X = torch.from_numpy(Ud).cuda() @ torch.from_numpy(V).cuda().T
        return X.to(torch.float64 if ndt == np.float64 else torch.float32).contiguous()
    return torch.from_numpy(synth.generate(recipe, rows, cols, seed=seed, matrix_id=mid,
                                           dtype=ndt)).cuda()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--sizes", default="512,1024,2048,4096,8192")
    ap.add_argument("--recipes", default="uniform,uniform100,hdr65536",
                    help="synth recipes, or hdr<kappa> for Eq 47 with alpha = 0")
    ap.add_argument("--bs", type=int, default=32)
    ap.add_argument("--reps", type=int, default=4, help="GEMMs per (size, site, flips) cell")
    ap.add_argument("--seed", type=int, default=11)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r01_fig4"))
    args = ap.parse_args()
    f64 = args.dtype == "f64"
    ndt, tdt = (np.float64, torch.float64) if f64 else (np.float32, torch.float32)
    mant = 52 if f64 else 23
    nbits = 64 if f64 else 32
    sites = (0, 1) if f64 else (0, 1, 4)
    rng = np.random.default_rng(args.seed)
    rows = []
    t0 = time.time()
    for recipe in args.recipes.split(","):
        for n in [int(v) for v in args.sizes.split(",")]:
            M = N = K = n
            bs = args.bs
            A = make_input(recipe, M, K, 1, 0, ndt)
            B = make_input(recipe, K, N, 2, 1, ndt)
            plan = api.ProtectedGemm(M, N, K, dtype=tdt, bs=bs, p=2)
            res = plan.run(A, B)
            torch.cuda.synchronize()
            clean = res.counts()
            C0 = plan.C.clone()
            sea = plan.sea_bound(A, B)
            sea_col, sea_row = sea["eps_col"].clone(), sea["eps_row"].clone()
            plan.check_ext(eps_col=sea_col, eps_row=sea_row)
            clean_sea = api.counts_dict(plan.counts)
            nI, nJ = M // bs, N // bs
            cells = [(s, f, "mantissa") for s in sites for f in (1, 3, 5)]
            cells += [(s, 1, "sign_exponent") for s in sites]
            for site, nflips, field in cells:
                crit = det_a = det_s = tot = crit_det_a = crit_det_s = 0
                for _ in range(args.reps):
                    I, J = np.meshgrid(np.arange(nI), np.arange(nJ), indexing="ij")
                    i = (I * bs + rng.integers(0, bs, I.shape)).ravel()
                    j = (J * bs + rng.integers(0, bs, J.shape)).ravel()
                    if field == "mantissa":
                        masks = flip_masks(rng, i.size, nflips, 0, mant)
                    else:
                        masks = (np.uint64(1) << rng.integers(mant, nbits, i.size).astype(np.uint64))
                    ks = rng.integers(0, K, i.size)
                    fb = api.make_faults_arrays(i, j, site, ks, masks)
                    plan.gemm(A, B, fb, i.size)
                    plan.check()
                    st_a = torch.from_numpy(plan.result().reports()["status"].ravel().copy())
                    plan.check_ext(eps_col=sea_col, eps_row=sea_row)
                    st_s = torch.from_numpy(plan.result().reports()["status"].ravel().copy())
                    ti, tj = torch.from_numpy(i).cuda(), torch.from_numpy(j).cuda()
                    e = (plan.C[ti, tj].double() - C0[ti, tj].double()).cpu().numpy()
                    sig, _ = plan.bound_elements(ti, tj)
                    sig = sig.cpu().numpy()
                    with np.errstate(invalid="ignore"):
                        c = ~np.isfinite(e) | (np.abs(e) > 3 * sig)
                    blk = (i // bs) * nJ + (j // bs)
                    da = st_a.numpy()[blk] != 0
                    ds = st_s.numpy()[blk] != 0
                    tot += i.size
                    crit += int(c.sum())
                    det_a += int(da.sum())
                    det_s += int(ds.sum())
                    crit_det_a += int((c & da).sum())
                    crit_det_s += int((c & ds).sum())
                rows.append(dict(recipe=recipe, n=n, site=site, flips=nflips, field=field,
                                 faults=tot, critical=crit,
                                 aabft_detected_of_critical=crit_det_a / crit if crit else None,
                                 sea_detected_of_critical=crit_det_s / crit if crit else None,
                                 aabft_detected=det_a, sea_detected=det_s))
                print(json.dumps(rows[-1]), flush=True)
            rows.append(dict(recipe=recipe, n=n, clean_false_positives_aabft=clean["checks_critical"],
                             clean_false_positives_sea=clean_sea["checks_critical"]))
            del plan, A, B, C0
            torch.cuda.empty_cache()
    out = {"dtype": args.dtype, "bs": args.bs, "reps": args.reps, "seconds": time.time() - t0,
           "rows": rows}
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(f"{args.out}_{args.dtype}.json", "w") as f:
        json.dump(out, f, indent=1)
    op = {0: "final add (site 0)", 1: "inner add (site 1)", 4: "inner mul (site 4)"}
    lines = [f"# Fig 4 on B200 ({args.dtype}, BS {args.bs}, one fault per block, {args.reps} GEMMs "
             f"per cell, {out['seconds']:.0f} s)", "",
             "Detected among critical faults (|e| > 3 sigma_ij, P:L543), A-ABFT vs SEA-ABFT on the "
             "same faulty products.", "",
             "| inputs | n | operation | flips | field | faults | critical | A-ABFT | SEA-ABFT |",
             "|---|---|---|---|---|---|---|---|---|"]
    for r in rows:
        if "site" not in r:
            continue
        fa = "-" if r["aabft_detected_of_critical"] is None else f"{r['aabft_detected_of_critical']:.4f}"
        fs = "-" if r["sea_detected_of_critical"] is None else f"{r['sea_detected_of_critical']:.4f}"
        lines.append(f"| {r['recipe']} | {r['n']} | {op[r['site']]} | {r['flips']} | {r['field']} | "
                     f"{r['faults']} | {r['critical']} | {fa} | {fs} |")
    lines += ["", "Clean runs (false positives): " + ", ".join(
        f"{r['recipe']} n={r['n']}: A-ABFT {r['clean_false_positives_aabft']}, SEA {r['clean_false_positives_sea']}"
        for r in rows if "site" not in r)]
    with open(f"{args.out}_{args.dtype}.md", "w") as f:
        f.write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
