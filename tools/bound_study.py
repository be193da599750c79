#!/usr/bin/env python3
"""NEXT-1 / NEXT-3 / NEXT-4: the paper's bound-quality experiment (§VI-B, Tables II/III/IV,
P:L414-464) at GPU scale.

For n = 512 ... 8192 (square, FP64, BS = 32, p = 2, 3 sigma; readings R1/R2), the two uniform
input ranges of Tables II/III and the Eq 47 high-dynamic-range inputs of Table IV (alpha = 0,
kappa = 2, reading R28; generated once on the device from the seeded host factors), on the
sm_100a path:
  * AVG. A-ABFT  = mean eps over all carried checksum elements (aabft_bound)      -> pinned
  * AVG. Rnd. Error = mean |carried - exact| of the column checksums, exact in double-double
    on the GPU (aabft_checksum_errors); our DMMA GEMM accumulates in a different order than
    the paper's sequential Kepler kernel, so this column is reported, not pinned.
  * AVG. SEA-ABFT = mean SEA bound over column, row and corner checksums (aabft_sea_bound,
    reading R25)                                                             -> pinned (II/III)
Table IV's absolute scale depends on the unstated scale of U, V in Eq 47 (parity unpinned);
its growth with n is pinned by tests/test_oracle_hdr.py.
Writes profiles/r01_bound_study.{json,md}.
"""
from __future__ import annotations

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

SIZES = [int(v) for v in os.environ.get("SIZES", "512,1024,2048,3072,4096,5120,6144,7168,8192").split(",")]
OUT = os.environ.get("OUT", os.path.join(ROOT, "profiles", "r01_bound_study"))
TABLES = os.environ.get("TABLES", "table2_uniform1.json,table3_uniform100.json,table4_hdr.json").split(",")


def make(g, n, seed, matrix_id):
    """Inputs of one table row on the device: the seeded recipes of Tables II/III, or Eq 47
    (Table IV) assembled on the device from the seeded host factors."""
    if g["recipe"] == "hdr":
        Ud, V = synth.hdr_factors(n, n, seed=seed, matrix_id=matrix_id, kappa=g["kappa"],
                                  alpha=g["alpha"])
        return torch.from_numpy(Ud).cuda() @ torch.from_numpy(V).cuda().T
    return torch.from_numpy(synth.generate(g["recipe"], n, n, seed=seed, matrix_id=matrix_id)).cuda()


def main():
    rows = []
    for table in TABLES:
        g = json.load(open(os.path.join(ROOT, "tests", "golden", table)))
        for n in SIZES:
            t0 = time.time()
            A = make(g, n, 1, 0)
            B = make(g, n, 2, 1)
            plan = api.ProtectedGemm(n, n, n, dtype=torch.float64, bs=32, p=2)
            res = plan.run(A, B)
            b = plan.bound()
            ec, er = plan.checksum_errors(A, B)
            sea = plan.sea_bound(A, B, corner=True)
            torch.cuda.synchronize()
            sea_all = torch.cat([sea["eps_col"].ravel(), sea["eps_row"].ravel(),
                                 sea["eps_corner"].ravel()])
            eps_all = torch.cat([b["eps_col"].ravel(), b["eps_row"].ravel()])
            err_col = ec.abs()
            err_all = torch.cat([ec.abs().ravel(), er.abs().ravel()])
            ref = g["rows"][str(n)]
            r = dict(table=table.split("_")[0], recipe=g["recipe"], n=n,
                     mean_eps=float(eps_all.mean()), paper_mean_eps=ref["avg_aabft"],
                     mean_err_col=float(err_col.mean()), mean_err_all=float(err_all.mean()),
                     paper_mean_err=ref["avg_rnd_error"],
                     max_err_over_eps=float((torch.cat([ec.ravel().abs() / b["eps_col"].ravel(),
                                                        er.ravel().abs() / b["eps_row"].ravel()])).max()),
                     critical_checks=res.counts()["checks_critical"],
                     mean_sea=float(sea_all.mean()), paper_mean_sea=ref["avg_sea_abft"],
                     seconds=time.time() - t0)
            r["sea_ratio_to_paper"] = r["mean_sea"] / r["paper_mean_sea"]
            r["sea_over_aabft"] = r["mean_sea"] / r["mean_eps"]
            r["eps_ratio_to_paper"] = r["mean_eps"] / r["paper_mean_eps"]
            r["err_ratio_to_paper"] = r["mean_err_col"] / r["paper_mean_err"]
            r["bound_over_actual"] = r["mean_eps"] / r["mean_err_col"]
            rows.append(r)
            print(json.dumps(r), flush=True)
            del A, B, plan, res, b, ec, er, sea, sea_all
            torch.cuda.empty_cache()
    json.dump(rows, open(OUT + ".json", "w"), indent=1)
    lines = ["# Bound-quality study on B200 (Tables II/III/IV, P:L414-464)", "",
             "FP64, BS 32, p 2, 3 sigma, t 52, seeds A=1 B=2.  `mean eps` = mean bound over all carried "
             "checksum elements (pinned to the paper within 5%, tests/test_gpu_parity.py); `mean err` = "
             "mean |carried - exact| of the column checksums, exact in double-double on the GPU; the "
             "paper's Kepler GEMM accumulated sequentially in k, our DMMA GEMM does not, so its actual "
             "errors differ (reported, not pinned).  `SEA` = mean SEA-ABFT bound over column, row and "
             "corner checksums (reading R25; pinned within 5% for Tables II/III).  Table IV (`hdr`, Eq 47, "
             "alpha 0, kappa 2, reading R28): the scale of U, V is not stated, so its absolute ratios are "
             "unpinned; the growth with n is pinned (tests/test_oracle_hdr.py).", "",
             "| table | range | n | mean eps | paper | ratio | mean err (ours) | paper err | ratio | bound/actual | max |err|/eps | critical | SEA | paper SEA | ratio | SEA/A-ABFT |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for r in rows:
        lines.append(f"| {r['table']} | {r['recipe']} | {r['n']} | {r['mean_eps']:.3e} | {r['paper_mean_eps']:.2e} | "
                     f"{r['eps_ratio_to_paper']:.3f} | {r['mean_err_col']:.3e} | {r['paper_mean_err']:.2e} | "
                     f"{r['err_ratio_to_paper']:.3f} | {r['bound_over_actual']:.0f} | {r['max_err_over_eps']:.4f} | {r['critical_checks']} | "
                     f"{r['mean_sea']:.3e} | {r['paper_mean_sea']:.2e} | {r['sea_ratio_to_paper']:.3f} | {r['sea_over_aabft']:.0f} |")
    open(OUT + ".md", "w").write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
