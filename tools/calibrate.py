#!/usr/bin/env python
"""Fit the B200 performance model (§V, L1402-1419 method re-done):
one linear model per kernel over the planner's features (model.cpp), fitted by
non-negative least squares on relative error, with a random 80/20 split of the
configurations (L1311-1313) and the paper's precision metric
mean(|actual - predicted| / actual) x 100 (L1414-1416).

Also reports the model's *regret*: for every case, the measured time of the
candidate the fitted model would pick vs the best measured candidate.

  python tools/calibrate.py gpurun_out/calib8_*.jsonl [--write]
"""
from __future__ import annotations

import argparse
import collections
import json
import os
import random
import sys

import numpy as np
from scipy.optimize import nnls

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
COEFF_H = os.path.join(ROOT, "paper_conf_ipps_veduradasskhpkn18_b200", "csrc", "model_coeffs.h")
KINDS = ["direct", "tile", "pipe", "quad", "bulkq", "bulkg", "vec"]


def fit(rows):
    X = np.array([r["features"] for r in rows])
    y = np.array([r["meas"] for r in rows])
    c, _ = nnls(X / y[:, None], np.ones(len(y)))
    return c


def err_pct(rows, c):
    if not rows:
        return float("nan")
    X = np.array([r["features"] for r in rows])
    y = np.array([r["meas"] for r in rows])
    return float(np.mean(np.abs(X @ c - y) / y) * 100)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("files", nargs="+")
    ap.add_argument("--write", action="store_true")
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--rel-max", type=float, default=1.5,
                    help="fit only candidates within this factor of their case's best "
                         "(the model's job is ranking the good region)")
    args = ap.parse_args()
    rows = [json.loads(l) for f in args.files for l in open(f) if l.startswith("{")]
    best = collections.defaultdict(lambda: float("inf"))
    for r in rows:
        best[r["case"]] = min(best[r["case"]], r["meas"])
    for r in rows:
        r["rel"] = r["meas"] / best[r["case"]]
    cases = sorted({r["case"] for r in rows})
    rng = random.Random(args.seed)
    test_cases = set(rng.sample(cases, max(1, len(cases) // 5)))
    coefs, report = {}, {}
    for k in KINDS:
        rk = [r for r in rows if r["kernel"] == k]
        tr = [r for r in rk if r["case"] not in test_cases and r["rel"] <= args.rel_max]
        te = [r for r in rk if r["case"] in test_cases and r["rel"] <= args.rel_max]
        if not tr:
            continue
        c = fit(tr)
        coefs[k] = c
        report[k] = {"n_train": len(tr), "n_test": len(te), "err_train": err_pct(tr, c),
                     "err_test": err_pct(te, c)}
        print(f"{k:6s} n={len(rk):5d} coef={np.array2string(c, precision=3)} "
              f"train {report[k]['err_train']:.2f}% test {report[k]['err_test']:.2f}%")
    # regret of the argmin-predicted choice, per case
    by = collections.defaultdict(list)
    for r in rows:
        if r["kernel"] in coefs:
            r["fit"] = float(np.dot(coefs[r["kernel"]], r["features"]))
            by[r["case"]].append(r)
    reg, gb_choice, gb_best, gb_auto = [], [], [], []
    for c, rs in by.items():
        best = min(rs, key=lambda r: r["meas"])
        pick = min(rs, key=lambda r: r["fit"])
        reg.append(pick["meas"] / best["meas"] - 1)
        gb_choice.append(pick["gbs"])
        gb_best.append(best["gbs"])
        auto = [r for r in rs if r.get("is_auto")]
        if auto:
            gb_auto.append(auto[0]["gbs"])
    print(f"cases {len(by)}: mean regret {100 * np.mean(reg):.1f}%  "
          f"GB/s picked {np.mean(gb_choice):.0f} best {np.mean(gb_best):.0f} "
          f"(current auto {np.mean(gb_auto) if gb_auto else float('nan'):.0f})")
    if args.write:
        with open(COEFF_H) as f:
            src = f.read()
        lines = []
        for k, name in (("direct", "kCoefDirect"), ("tile", "kCoefTile"), ("pipe", "kCoefPipe"),
                        ("quad", "kCoefQuad"), ("bulkq", "kCoefBulkQ"), ("bulkg", "kCoefBulkG"),
                        ("vec", "kCoefVec")):
            if k in coefs:
                vals = ", ".join(f"{v:.6e}" for v in coefs[k])
                lines.append(f"constexpr double {name}[kModelNumFeatures] = {{{vals}}};")
        out = []
        for line in src.splitlines():
            if line.startswith("constexpr double kCoef"):
                nm = line.split()[2].split("[")[0]
                rep = [l for l in lines if l.split()[2].split("[")[0] == nm]
                out.append(rep[0] if rep else line)
            elif line.startswith("constexpr const char *kModelSource"):
                tag = "; ".join(f"{k}: train {v['err_train']:.1f}% test {v['err_test']:.1f}% "
                                f"(n={v['n_train']}+{v['n_test']})" for k, v in report.items())
                out.append(f'constexpr const char *kModelSource = "B200 fit ({len(cases)} cases, '
                           f'{len(rows)} points, rel<={args.rel_max}): {tag}; '
                           f'regret {100 * np.mean(reg):.1f}%";')
            else:
                out.append(line)
        with open(COEFF_H, "w") as f:
            f.write("\n".join(out) + "\n")
        print("wrote", COEFF_H)
    print(json.dumps(report))


if __name__ == "__main__":
    main()
