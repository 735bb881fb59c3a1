#!/usr/bin/env python
"""Offline regret of a compiled tree set (model_gbt.h / model_gbt2.h) on
calibration data: per case, the measured time of the candidate the trees pick
among the linear screen's top 16 (as the planner ranks) vs the best measured
candidate of the case.

  python tools/gbt_eval.py --header model_gbt.h --sym kGbt f1.jsonl [f2.jsonl ...]
"""
from __future__ import annotations

import argparse
import collections
import gzip
import json
import math
import os
import re
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
import calibrate_gbt as cg  # noqa: E402


def load_trees(path, sym):
    src = open(path).read()

    def arr(name, conv):
        m = re.search(name + r"\[\d+\]\[\d+\] = \{\n(.*?)\};", src, re.S)
        rows = re.findall(r"\{([^}]*)\}", m.group(1))
        return [[conv(x) for x in r.split(",")] for r in rows]

    def flt(x):
        x = x.strip()
        return float("inf") if x == "INFINITY" else float(x.rstrip("f"))
    F = arr(sym + "F", lambda x: int(x))
    T = arr(sym + "T", flt)
    V = arr(sym + "V", flt)
    init = float(re.search(sym + r"Init = ([^;]*);", src).group(1))
    depth = int(re.search(sym + r"Depth = (\d+);", src).group(1))
    return F, T, V, init, depth


def predict(trees, d):
    F, T, V, init, D = trees
    NI = 2 ** D - 1
    s = init
    x = np.float32(d)
    for f, t, v in zip(F, T, V):
        i = 0
        for _ in range(D):
            i = 2 * i + 1 + (1 if x[f[i]] > np.float32(t[i]) else 0)
        s += v[i - NI]
    return s


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("files", nargs="+")
    ap.add_argument("--header", default="model_gbt.h")
    ap.add_argument("--sym", default="kGbt")
    ap.add_argument("--topk", type=int, default=16)
    ap.add_argument("--exclude", default="", help="comma list of kernels the trees do not rank")
    args = ap.parse_args()
    trees = load_trees(os.path.join(cg.CSRC, args.header), args.sym)
    rows = [json.loads(l) for f in args.files for l in (gzip.open(f, "rt") if f.endswith(".gz") else open(f)) if l.startswith("{")]
    rows = [r for r in rows if r["kernel"] in cg.KID
            and r["kernel"] not in args.exclude.split(",")]
    co = cg.linear_coefs()
    by = collections.defaultdict(list)
    for r in rows:
        r["lin"] = float(co[r["kernel"]] @ np.array(r["features"]))
        by[r["case"]].append(r)
    reg, out = [], []
    for c, rs in sorted(by.items()):
        uniq = {}
        for r in sorted(rs, key=lambda r: r["lin"]):
            uniq.setdefault((tuple(r["tile"]), r["kernel"], r["threads"]), r)
        cand = list(uniq.values())[:args.topk]
        P = [predict(trees, np.array(cg.desc(r), dtype=np.float32)) for r in cand]
        pick = cand[int(np.argmin(P))]
        best = min(rs, key=lambda r: r["meas"])
        reg.append(pick["meas"] / best["meas"] - 1)
        out.append((c, pick["kernel"], pick["gbs"], best["kernel"], best["gbs"]))
    print(f"{args.header}: {len(by)} cases, mean regret {100 * np.mean(reg):.1f}%, "
          f"picked {np.mean([o[2] for o in out]):.0f} best {np.mean([o[4] for o in out]):.0f} GB/s")
    for o in sorted(out, key=lambda o: o[2] / o[4])[:8]:
        print("   %-34s pick %-6s %6.0f  best %-6s %6.0f" % o)


if __name__ == "__main__":
    main()
