#!/usr/bin/env python
"""Add the single- vs repeated-use ratio and the plan time (tools/singleuse.cpp
output) to a per-case table (tools/cases.py output), matching cases by extents
and permutation.

  python tools/merge_single.py profiles/r2_cases_c3.json profiles/r2_singleuse_c3.txt
"""
import json
import sys


def main(cases_path, single_path):
    single = {}
    for line in open(single_path):
        if line.startswith("#") or "|" not in line:
            continue
        head, mid, tail = line.split("|")
        f = head.split()
        d = int(f[1])
        key = (tuple(int(x) for x in f[2:2 + d]), tuple(int(x) for x in f[2 + d:2 + 2 * d]))
        rep, sgl, ratio = (float(x) for x in mid.split())
        pmin, pmed = (float(x) for x in tail.split())
        single[key] = {"repeated_us_host": rep, "single_us_host": sgl,
                       "single_over_repeated": ratio, "plan_us_median": pmed}
    doc = json.load(open(cases_path))
    n = 0
    for r in doc["cases"]:
        _, ext, perm = r["case"].split(":")
        key = (tuple(int(x) for x in ext.split("x")), tuple(int(c) for c in perm))
        if key in single:
            r.update(single[key])
            n += 1
    ratios = [r["single_over_repeated"] for r in doc["cases"] if "single_over_repeated" in r]
    if ratios:
        doc["single_over_repeated"] = {"mean": sum(ratios) / len(ratios), "max": max(ratios),
                                       "over_1.10": sum(1 for x in ratios if x > 1.10),
                                       "source": single_path,
                                       "timing": "K back-to-back ttlg_transpose vs K ttlg_execute "
                                                 "of a pre-built plan, host wall clock to stream "
                                                 "sync, median of trials (tools/singleuse.cpp)"}
    json.dump(doc, open(cases_path, "w"), indent=1)
    print(f"{cases_path}: {n} cases merged", doc.get("single_over_repeated"))


if __name__ == "__main__":
    main(*sys.argv[1:])
