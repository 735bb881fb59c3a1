#!/usr/bin/env python
"""Summarise a calibration sweep: per case auto vs best candidate GB/s."""
import collections
import json
import statistics
import sys


def main():
    rows = [json.loads(l) for f in sys.argv[1:] for l in open(f) if l.startswith("{")]
    by = collections.defaultdict(list)
    for r in rows:
        by[r["case"]].append(r)
    A, Bst = [], []
    for c, rs in by.items():
        best = max(rs, key=lambda r: r["gbs"])
        auto = [r for r in rs if r["is_auto"]]
        a = auto[0]["gbs"] if auto else float("nan")
        A.append(a)
        Bst.append(best["gbs"])
        print(f"{c[:34]:34s} auto {a:5.0f} best {best['gbs']:5.0f} {best['schema']:4s} W{best['W']:<2d} "
              f"tile {best['tile']} LA {best['LA']} LB {best['LB']} grid {best['grid']} occ {best['occ']}")
    print("mean auto", statistics.mean(x for x in A if x == x), "mean best", statistics.mean(Bst))


if __name__ == "__main__":
    main()
