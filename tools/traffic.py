#!/usr/bin/env python
"""Per-kernel DRAM traffic per launch from the ncu launch list of one bench
step (tools/round_bench.sh) -> profiles/ncu_traffic.json, read by bench.py for
roofline.traffic.  Launch i of the step is case i of the workload (bench.py
launches the cases in order), so each launch is attributed to its case's kernel."""
import collections
import csv
import json
import sys


def main(launches="gpurun_out/launches.csv", bench="gpurun_out/bench.json",
         out="profiles/ncu_traffic.json", workload="ttc57"):
    rows = list(csv.reader(l for l in open(launches) if l.startswith('"')))
    hdr = rows[0]
    ix = {h: i for i, h in enumerate(hdr)}
    per = collections.OrderedDict()
    for r in rows[1:]:
        d = per.setdefault(int(r[ix["ID"]]), {})
        d[r[ix["Metric Name"]]] = float(r[ix["Metric Value"]].replace(",", ""))
    cases = json.load(open(bench))["cases"]
    assert len(per) == len(cases), (len(per), len(cases))
    acc = collections.defaultdict(lambda: [0.0, 0, 0.0, 0.0])
    for (lid, m), c in zip(per.items(), cases):
        a = acc[c["kernel"]]
        a[0] += m["dram__bytes_read.sum"] + m["dram__bytes_write.sum"]
        a[1] += 1
        a[2] += m["gpu__time_duration.sum"]
    tot = sum(a[2] for a in acc.values())
    res = {k: a[0] / a[1] for k, a in acc.items()}
    share = {k: a[2] / tot for k, a in acc.items()}
    import os
    doc = json.load(open(out)) if os.path.exists(out) else {}
    doc[workload] = res
    doc.setdefault("ncu_time_share", {})
    if not isinstance(doc["ncu_time_share"], dict) or "k_quad" in doc["ncu_time_share"]:
        doc["ncu_time_share"] = {}
    doc["ncu_time_share"][workload] = share
    doc["source"] = ("ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,"
                     "dram__bytes_write.sum, one bench step per workload (profiles/*launches*.csv)")
    json.dump(doc, open(out, "w"), indent=1)
    print(res, share)


if __name__ == "__main__":
    main(*sys.argv[1:])
