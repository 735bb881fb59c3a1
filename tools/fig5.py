#!/usr/bin/env python
"""Fig. 5-style model check: 27^5 fp64, perm 4 1 2 0 3,
output slice fixed to the output FVI (o0 = i4, 27 elements), input slice
varied over every (input dim, block) the planner enumerates.  For each input
slice the model picks kernel and block size (ttlg_plan_ex with the slice
forced), predicts its time (the ranked prediction ttlg_plan_describe reports)
and the slice is timed (CUDA events, median of reps).  The paper's claim is
qualitative -- "the predictions follow the trend" of the measured times
(L1433-1434) -- so the report gives both series, the rank correlation and
whether the fastest measured slice is the model's pick.

  python tools/fig5.py [--reps 20] > fig5.jsonl
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def spearman(x, y):
    def ranks(v):
        order = sorted(range(len(v)), key=lambda i: v[i])
        r = [0.0] * len(v)
        for k, i in enumerate(order):
            r[i] = float(k)
        return r
    rx, ry = ranks(x), ranks(y)
    mx, my = sum(rx) / len(rx), sum(ry) / len(ry)
    num = sum((a - mx) * (b - my) for a, b in zip(rx, ry))
    den = (sum((a - mx) ** 2 for a in rx) * sum((b - my) ** 2 for b in ry)) ** 0.5
    return num / den if den else 0.0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=20)
    args = ap.parse_args()
    import torch
    import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
    from synth import configs, gen_tensor_torch, case_seed

    c = configs.fig5_case()
    ext, perm = list(c.extents), list(c.perm)
    auto = ttlg.plan("f64", ext, perm).describe()
    slices = set()
    for d in ttlg.plan_candidates("f64", ext, perm):
        if d["kernel"] == "direct" or d["out_dim"] != 0:
            continue
        fp = d["fused_perm"]
        if d["tile_extents"][fp[0]] != d["fused_extents"][fp[0]]:
            continue  # output slice = the whole output FVI (27), as in Fig. 5
        slices.add((d["in_dim"], d["tile_extents"][d["in_dim"]]))
    # the paper's x-axis: input slice 27 x b (i0 whole, the fused i1 i2 blocked by b)
    slices |= {(1, b) for b in range(1, 11)}
    A = gen_tensor_torch(case_seed(c.case_id), c.n_elems, 8, device="cuda")
    B = torch.empty_like(A)
    s = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    rows = []
    for a, ta in sorted(slices):
        try:
            p = ttlg.plan("f64", ext, perm, in_dim=a, in_block=ta, out_dim=0)
        except ttlg.TtlgError:
            continue
        info = p.describe()
        for _ in range(3):
            p.execute(A.data_ptr(), B.data_ptr(), s.cuda_stream)
        ts = []
        for _ in range(args.reps):
            e0.record()
            p.execute(A.data_ptr(), B.data_ptr(), s.cuda_stream)
            e1.record()
            e1.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e-3)
        t = statistics.median(ts)
        in_vol = 1
        for k in range(a + 1):
            in_vol *= info["tile_extents"][k]
        row = {"in_dim": a, "in_block": ta, "in_slice": in_vol, "kernel": info["kernel"],
               "threads": info["threads"], "pred_us": info["predicted_seconds"] * 1e6,
               "meas_us": t * 1e6, "gbs": c.alg_bytes / t / 1e9,
               "is_auto": info["tile_extents"] == auto["tile_extents"]}
        rows.append(row)
        print(json.dumps(row), flush=True)
    best = min(rows, key=lambda r: r["meas_us"])
    pick = min(rows, key=lambda r: r["pred_us"])
    print(json.dumps({"summary": True, "slices": len(rows),
                      "spearman_pred_vs_meas": spearman([r["pred_us"] for r in rows],
                                                        [r["meas_us"] for r in rows]),
                      "mean_abs_err_pct": 100 * statistics.mean(
                          abs(r["pred_us"] - r["meas_us"]) / r["meas_us"] for r in rows),
                      "best_measured": best, "model_pick": pick,
                      "pick_regret_pct": 100 * (pick["meas_us"] / best["meas_us"] - 1)}),
          flush=True)


if __name__ == "__main__":
    main()
