#!/usr/bin/env python
"""Summarise one evidence run (gpurun_out/<tag>/ written by tools/experiments/r2e38.sh)
into the markdown tables of DESIGN.md §6b and copy its files to profiles/ under
the round-2 names.

  python tools/r2_report.py gpurun_out/r2e38 [--copy]
"""
import glob
import json
import os
import shutil
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BENCH = [("bench.json", "config 2 TTC-57 fp64", "ttc57"), ("bench_ccsdt.json", "config 3 CCSD(T) fp64", "ccsdt"),
         ("bench_smallfvi.json", "config 4 small-FVI fp32", "smallfvi"),
         ("bench_sharded.json", "config 5 at N = 1 (local perms)", "sharded"),
         ("bench_720-16.json", "720 perms of 16^6 fp64", "720-16"),
         ("bench_720-15.json", "720 perms of 15^6 fp64", "720-15"),
         ("bench_720-17.json", "720 perms of 17^6 fp64", "720-17"),
         ("bench_fig13.json", "Fig. 13 sizes (15^4 ... 128^4)", "fig13"),
         ("bench_c1.json", "config 1 (16^4, 512 KiB, launch-bound)", "c1")]


def last_json(p):
    with open(p) as f:
        return json.loads(f.read().strip().splitlines()[-1])


def main():
    d = sys.argv[1]
    print("| workload | GB/s | fraction of peak | same-run D2D | dominant kernel (frac of peak) | model error | SM MHz / reasons |")
    print("|---|---|---|---|---|---|---|")
    for f, name, _ in BENCH:
        p = os.path.join(d, f)
        if not os.path.exists(p):
            continue
        try:
            b = last_json(p)
        except Exception as e:  # noqa: BLE001
            print(f"| {name} | ERR {e} |")
            continue
        r = b.get("roofline") or {}
        clk = b.get("clocks") or {}
        err = b.get("model_err_pct")
        print(f"| {name} | {b['value']:.0f} | {b.get('frac_of_peak') or 0:.3f} | "
              f"{b.get('d2d_gbs') or 0:.0f} | {r.get('kernel')} {r.get('achieved', 0):.0f} "
              f"({r.get('frac', 0):.3f}) | {'' if err is None else f'{err:.1f} %'} | "
              f"{clk.get('sm_mhz')} {','.join(clk.get('reasons') or [])} |")
    print()
    print("| workload | cases | aggregate GB/s | median / min fraction of HBM peak | cases < 0.9 of same-size D2D | min of D2D |")
    print("|---|---|---|---|---|---|")
    for w in ("c2", "c3", "c4", "720-16", "720-15", "720-17", "fig13", "c1"):
        p = os.path.join(d, f"cases_{w}.json")
        if not os.path.exists(p):
            continue
        c = json.load(open(p))
        fr = [x["frac_peak"] for x in c["cases"]]
        print(f"| {w} | {len(c['cases'])} | {c['aggregate_gbs']:.0f} | {statistics.median(fr):.3f} / "
              f"{min(fr):.3f} | {len(c['below_0.9_d2d'])} | {c['min_frac_d2d']:.3f} |")
    print()
    for f in sorted(glob.glob(os.path.join(d, "singleuse_*.txt"))):
        rows = [ln.split("|") for ln in open(f) if not ln.startswith("#") and "|" in ln]
        rat = [float(x[1].split()[2]) for x in rows if len(x) > 2]
        if rat:
            print(f"{os.path.basename(f)}: n={len(rat)} single/repeated mean {statistics.mean(rat):.3f} "
                  f"max {max(rat):.3f} (> 1.10: {sum(x > 1.10 for x in rat)})")
    if "--copy" in sys.argv:
        prof = os.path.join(ROOT, "profiles")
        for f, _, w in BENCH:
            if os.path.exists(os.path.join(d, f)):
                shutil.copy(os.path.join(d, f), os.path.join(prof, f"r2_bench_{w}.json"))
        pairs = [("bench_ref.json", "r2_bench_reference.json"), ("launches.csv", "r2_launches.csv"),
                 ("ncu_k_quad_summary.txt", "r2_ncu_k_quad_bench_summary.txt"),
                 ("fig12.jsonl", "r2_fig12.jsonl")]
        pairs += [(os.path.basename(x), "r2_" + os.path.basename(x))
                  for x in glob.glob(os.path.join(d, "cases_*.json"))]
        pairs += [(os.path.basename(x), "r2_" + os.path.basename(x))
                  for x in glob.glob(os.path.join(d, "singleuse_*.txt"))]
        pairs += [(os.path.basename(x), "r2_" + os.path.basename(x))
                  for x in glob.glob(os.path.join(d, "ncu_k_*_summary.txt"))
                  if "k_quad_summary" not in x]
        for a, b in pairs:
            if os.path.exists(os.path.join(d, a)):
                shutil.copy(os.path.join(d, a), os.path.join(prof, b))
        print("copied", len(pairs), "files to profiles/")


if __name__ == "__main__":
    main()
