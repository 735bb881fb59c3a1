#!/usr/bin/env python
"""Fit the ranking stage of the B200 performance model: gradient-boosted
regression trees on the log of (measured time / ideal one-pass time) over
plan descriptors (model.cpp model_descriptor), trained on tools/calib_sweep.py
data (§V's per-kernel linear regression re-derived for B200: the
linear model screens candidates, the trees rank the short list).

Reports, on a random 80/20 split of configurations (L1311-1313), the paper's
precision metric mean(|a-p|/a) (L1414-1416) and the selection regret; then
refits on everything and writes paper_conf_ipps_veduradasskhpkn18_b200/csrc/model_gbt.h.

  python tools/calibrate_gbt.py gpurun_out/calib16_*.jsonl [--write]
"""
from __future__ import annotations

import argparse
import collections
import gzip
import json
import math
import os
import random
import re

import numpy as np
from sklearn.ensemble import GradientBoostingRegressor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_ipps_veduradasskhpkn18_b200", "csrc")
KID = {"direct": 0, "tile": 1, "pipe": 2, "quad": 3, "bulkq": 5, "bulkg": 6, "vec": 7}
HBM = 6555.5e9
SMS = 148
TOPK = int(os.environ.get("TTLG_GBT_TOPK", "16"))


def desc(r):
    """Must match model.cpp model_descriptor() exactly."""
    W, V = r["W"], r["V"]
    occ, th = max(1, r["occ"]), r["threads"]
    LAb = (V if r["kernel"] == "direct" else r["LA"]) * W
    f = r["features"]
    N = r["bytes"] / (2.0 * W)
    RA = V / (V if r["kernel"] == "direct" else r["LA"])
    RB = V / r["LB"]
    return [KID[r["kernel"]], math.log2(W), math.log2(LAb), math.log2(r["LB"] * W),
            math.log2(V * W), th / 256.0, float(occ), occ * th / 2048.0,
            math.log2(r["tiles"]), f[2] / max(f[1], 1e-12), f[8] / max(1.0, r["bytes"] / 1e9),
            r["tiles"] / (SMS * occ),
            math.log2(V / th), (RA + RB + r["LB"]) / th, N / (r["tiles"] * V),
            math.ceil(r["tiles"] / r["grid"]), math.log2(r["bytes"]), float(r.get("nstage", 0))]


def ideal(r):
    return r["bytes"] / HBM


def linear_coefs():
    src = open(os.path.join(CSRC, "model_coeffs.h")).read()
    co = {}
    for name, k in (("kCoefDirect", "direct"), ("kCoefTile", "tile"), ("kCoefPipe", "pipe"),
                    ("kCoefQuad", "quad"), ("kCoefBulkQ", "bulkq"), ("kCoefBulkG", "bulkg"),
                    ("kCoefVec", "vec")):
        m = re.search(name + r"\[kModelNumFeatures\] = \{([^}]*)\}", src)
        co[k] = np.array([float(x) for x in m.group(1).split(",")])
    return co


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("files", nargs="+")
    ap.add_argument("--write", action="store_true")
    ap.add_argument("--trees", type=int, default=100)
    ap.add_argument("--depth", type=int, default=5)
    ap.add_argument("--lr", type=float, default=0.2)
    ap.add_argument("--sym", default="kGbt", help="C symbol prefix of the tree set")
    ap.add_argument("--out", default="model_gbt.h", help="header name under csrc/")
    args = ap.parse_args()
    def lines(f):
        return gzip.open(f, "rt") if f.endswith(".gz") else open(f)
    rows = [json.loads(l) for f in args.files for l in lines(f) if l.startswith("{")]
    # k_deint is not ranked by the trees (its time is a measured factor, model.h)
    rows = [r for r in rows if r["kernel"] in KID]
    co = linear_coefs()
    by = collections.defaultdict(list)
    for r in rows:
        r["lin"] = float(co[r["kernel"]] @ np.array(r["features"]))
        by[r["case"]].append(r)
    cases = sorted(by)
    rng = random.Random(0)
    test = set(rng.sample(cases, len(cases) // 5))

    def fit(rs):
        X = np.array([desc(r) for r in rs])
        y = np.array([math.log(r["meas"] / ideal(r)) for r in rs])
        return GradientBoostingRegressor(n_estimators=args.trees, max_depth=args.depth,
                                         learning_rate=args.lr, subsample=0.8,
                                         random_state=0).fit(X, y)

    def per_schema(m, cs):
        """Held-out mean |a-p|/a (L1414-1416) of every measured candidate, by
        schema and by kernel; plus the error of each case's chosen plan."""
        out = collections.defaultdict(list)
        for c in cs:
            rs = by[c]
            P = m.predict(np.array([desc(r) for r in rs]))
            for r, p in zip(rs, P):
                e = abs(math.exp(p) * ideal(r) - r["meas"]) / r["meas"]
                out["schema:" + r["schema"]].append(e)
                out["kernel:" + r["kernel"]].append(e)
                out["size:" + ("<16MB" if r["bytes"] < 16e6 else ">=16MB")].append(e)
        return {k: (round(100 * float(np.mean(v)), 1), len(v)) for k, v in sorted(out.items())}

    def evaluate(m, cs):
        reg, err, gp, gb = [], [], [], []
        for c in cs:
            # the planner's short list holds one entry per (tile box, kernel, block size)
            uniq = {}
            for r in sorted(by[c], key=lambda r: r["lin"]):
                uniq.setdefault((tuple(r["tile"]), r["kernel"], r["threads"]), r)
            rs = list(uniq.values())[:TOPK]
            P = m.predict(np.array([desc(r) for r in rs]))
            best = min(by[c], key=lambda r: r["meas"])
            pick = rs[int(np.argmin(P))]
            reg.append(pick["meas"] / best["meas"] - 1)
            gp.append(pick["gbs"])
            gb.append(best["gbs"])
            for r, p in zip(rs, P):
                err.append(abs(math.exp(p) * ideal(r) - r["meas"]) / r["meas"])
        return 100 * np.mean(reg), 100 * np.mean(err), np.mean(gp), np.mean(gb)

    m = fit([r for r in rows if r["case"] not in test])
    tr = evaluate(m, [c for c in cases if c not in test])
    te = evaluate(m, list(test))
    print(f"train: regret {tr[0]:.1f}% err(top{TOPK}) {tr[1]:.1f}% picked {tr[2]:.0f} best {tr[3]:.0f}")
    print(f"test : regret {te[0]:.1f}% err(top{TOPK}) {te[1]:.1f}% picked {te[2]:.0f} best {te[3]:.0f}")
    print("held-out error by schema / kernel / size (mean |a-p|/a %, n):")
    print(json.dumps(per_schema(m, list(test))))
    if not args.write:
        return
    m = fit(rows)  # final model on all configurations
    # complete binary trees of depth D in implicit layout (node i -> children
    # 2i+1, 2i+2): shallower sklearn leaves are padded with always-left dummy
    # splits (feature 0, threshold +inf) so traversal is D branch-free steps
    D = args.depth
    NI, NL = 2 ** D - 1, 2 ** D
    F, T, V = [], [], []
    for est in m.estimators_[:, 0]:
        t = est.tree_
        f_ = [0] * NI
        t_ = [float("inf")] * NI
        v_ = [0.0] * NL

        def fill(i, pos, depth):
            if t.children_left[i] == -1:
                val = float(t.value[i][0][0]) * m.learning_rate
                lo, hi = pos, pos  # leaves of the complete subtree under pos
                while lo < NI:
                    lo, hi = 2 * lo + 1, 2 * hi + 2
                for q in range(lo, hi + 1):
                    v_[q - NI] = val
                return
            assert depth < D
            f_[pos] = int(t.feature[i])
            t_[pos] = float(t.threshold[i])
            fill(t.children_left[i], 2 * pos + 1, depth + 1)
            fill(t.children_right[i], 2 * pos + 2, depth + 1)

        fill(0, 0, 0)
        F.append(f_)
        T.append(t_)
        V.append(v_)
    init = float(m.init_.constant_[0][0]) if hasattr(m.init_, "constant_") else float(
        np.mean([math.log(r["meas"] / ideal(r)) for r in rows]))

    def flt(x):
        return "INFINITY" if x == float("inf") else f"{x!r}f"

    P = args.sym
    with open(os.path.join(CSRC, args.out), "w") as f:
        f.write(f"// {args.out} -- GENERATED by tools/calibrate_gbt.py: boosted regression trees\n"
                "// predicting log(time / one-pass ideal) from model_descriptor() (model.cpp).\n"
                f"// Fitted on {len(rows)} B200 measurements ({len(cases)} configurations); held-out\n"
                f"// 20%: selection regret {te[0]:.1f}%, mean |a-p|/a {te[1]:.1f}% (top-{TOPK} lists).\n"
                f"// Complete trees of depth {D}: node i has children 2i+1 (x <= t) and 2i+2.\n"
                "#pragma once\n#include <math.h>\n#include <stdint.h>\nnamespace ttlg {\n")
        f.write(f"constexpr int {P}Trees = {len(F)};\nconstexpr int {P}Depth = {D};\n"
                + (f"constexpr int {P}TopK = {TOPK};\n" if P == "kGbt" else ""))
        f.write(f"constexpr double {P}Init = {init!r};\n")
        f.write(f'constexpr const char *{P}Source = "GBT {len(F)} trees depth {D}, '
                f'{len(rows)} points / {len(cases)} cases; test regret {te[0]:.1f}%, '
                f'err {te[1]:.1f}%";\n')
        f.write(f"constexpr int8_t {P}F[{len(F)}][{NI}] = {{\n" +
                ",\n".join("{" + ",".join(map(str, r)) + "}" for r in F) + "};\n")
        f.write(f"constexpr float {P}T[{len(F)}][{NI}] = {{\n" +
                ",\n".join("{" + ",".join(flt(x) for x in r) + "}" for r in T) + "};\n")
        f.write(f"constexpr float {P}V[{len(F)}][{NL}] = {{\n" +
                ",\n".join("{" + ",".join(flt(x) for x in r) + "}" for r in V) + "};\n")
        f.write("}  // namespace ttlg\n")
    feats = F
    print("wrote", os.path.join(CSRC, args.out), len(feats), "trees")


if __name__ == "__main__":
    main()
