#!/usr/bin/env python
"""SURVEY N3 report: the paper's second workloads on B200, grouped as the paper
plots them.

- Figs. 6/8/10 (repeated use) and 7/9/11 (single use, plan cost included): the
  720 permutations of 15^6 / 16^6 / 17^6 fp64, grouped by scaled rank (the
  rank after index fusion: the red "staircase");
- Fig. 12: bandwidth vs number of repeated calls (tools/fig12.cpp output).

  python tools/n3_report.py --dir gpurun_out/r2eN --out profiles/r2_n3.json
Inputs in --dir: cases_720-{15,16,17}.json (tools/cases.py), singleuse_720-{e}.txt
(tools/singleuse.cpp), fig12.jsonl (tools/fig12.cpp).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics


def scaled_rank(perm):
    """Fused rank (all extents > 1): maximal runs perm[i+1] = perm[i] + 1 (L666-685)."""
    return 1 + sum(1 for i in range(1, len(perm)) if perm[i] != perm[i - 1] + 1)


def read_single(path):
    out = {}
    if not os.path.exists(path):
        return out
    for line in open(path):
        if line.startswith("#") or "|" not in line:
            continue
        head, mid, tail = line.split("|")
        f = head.split()
        d = int(f[1])
        perm = tuple(int(x) for x in f[2 + d:2 + 2 * d])
        rep, sgl, ratio = (float(x) for x in mid.split())
        pmin, pmed = (float(x) for x in tail.split())
        out[perm] = {"repeated_us": rep, "single_us": sgl, "ratio": ratio,
                     "plan_min_us": pmin, "plan_med_us": pmed}
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--dir", required=True)
    ap.add_argument("--out", required=True)
    args = ap.parse_args()
    rep = {"source": args.dir, "sweeps": {}, "fig12": None}
    for e in (15, 16, 17):
        p = os.path.join(args.dir, f"cases_720-{e}.json")
        if not os.path.exists(p):
            continue
        d = json.load(open(p))
        single = read_single(os.path.join(args.dir, f"singleuse_720-{e}.txt"))
        groups = {}
        for r in d["cases"]:
            perm = tuple(int(c) for c in r["case"].split(":")[2])
            sr = scaled_rank(perm)
            g = groups.setdefault(sr, {"n": 0, "gbs": [], "frac_d2d": [], "single_gbs": [],
                                       "ratio": [], "kernels": {}})
            g["n"] += 1
            g["gbs"].append(r["gbs"])
            g["frac_d2d"].append(r["frac_d2d"])
            g["kernels"][r["kernel"]] = g["kernels"].get(r["kernel"], 0) + 1
            s = single.get(perm)
            if s:
                nbytes = 2 * e ** 6 * 8
                g["single_gbs"].append(nbytes / (s["single_us"] * 1e-6) / 1e9)
                g["ratio"].append(s["ratio"])
        summ = {}
        for sr, g in sorted(groups.items()):
            summ[str(sr)] = {
                "perms": g["n"], "kernels": g["kernels"],
                "repeated_gbs": {"mean": statistics.mean(g["gbs"]), "min": min(g["gbs"]),
                                 "max": max(g["gbs"])},
                "frac_d2d": {"mean": statistics.mean(g["frac_d2d"]), "min": min(g["frac_d2d"])},
                "single_gbs": ({"mean": statistics.mean(g["single_gbs"]),
                                "min": min(g["single_gbs"])} if g["single_gbs"] else None),
                "single_over_repeated": ({"mean": statistics.mean(g["ratio"]),
                                          "max": max(g["ratio"])} if g["ratio"] else None)}
        rep["sweeps"][f"{e}^6"] = {"aggregate_gbs": d["aggregate_gbs"],
                                   "min_frac_d2d": d["min_frac_d2d"],
                                   "d2d_gbs": d["cases"][0]["d2d_gbs"],
                                   "by_scaled_rank": summ}
    p = os.path.join(args.dir, "fig12.jsonl")
    if os.path.exists(p):
        curves = {}
        for line in open(p):
            r = json.loads(line)
            curves.setdefault(r["perm"], {}).setdefault(r["mode"], []).append(
                [r["calls"], round(r["gbs"], 1)])
        rep["fig12"] = curves
    with open(args.out, "w") as f:
        json.dump(rep, f, indent=1)
    print(json.dumps(rep)[:2000])


if __name__ == "__main__":
    main()
