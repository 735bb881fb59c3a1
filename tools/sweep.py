#!/usr/bin/env python
"""Time individual transposition cases (CUDA events, median of reps) under the
auto plan or forced hints; prints one JSON line per (case, hints).

  python tools/sweep.py --group c2 [--hints '{"schema":"OD"}'] [--reps 20] [--check]
  python tools/sweep.py --case 5120,5120:1,0:8
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def parse_case(s):
    from synth.configs import Case
    e, p, b = s.split(":")
    return Case(0, tuple(int(x) for x in e.split(",")), tuple(int(x) for x in p.split(",")),
                int(b), "cli")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--group", default=None)
    ap.add_argument("--case", action="append", default=[])
    ap.add_argument("--hints", action="append", default=[])
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--limit", type=int, default=0)
    ap.add_argument("--stride", type=int, default=1)
    ap.add_argument("--d2d", action="store_true")
    args = ap.parse_args()

    import torch
    import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
    from synth import configs, gen_tensor_torch, case_seed

    cases = []
    if args.group:
        cases = configs.all_configs()[args.group] if args.group in configs.all_configs() else {
            "720-16": lambda: configs.sweep720(16), "720-15": lambda: configs.sweep720(15),
            "720-17": lambda: configs.sweep720(17), "fig13": configs.fig13,
            "fig5": lambda: [configs.fig5_case()]}[args.group]()
    cases += [parse_case(s) for s in args.case]
    cases = cases[::args.stride]
    if args.limit:
        cases = cases[:args.limit]
    hint_sets = [json.loads(h) for h in args.hints] or [{}]
    dev = torch.device("cuda:0")
    stream = torch.cuda.current_stream()
    for c in cases:
        A = gen_tensor_torch(case_seed(c.case_id), c.n_elems, c.elem_bytes, device=dev)
        B = torch.empty_like(A)
        if args.d2d:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            for _ in range(3):
                B.copy_(A)
            ts = []
            for _ in range(args.reps):
                e0.record()
                B.copy_(A)
                e1.record()
                e1.synchronize()
                ts.append(e0.elapsed_time(e1))
            print(json.dumps({"case": c.label(), "d2d_gbs": c.alg_bytes / statistics.median(ts)
                              / 1e6}), flush=True)
        for h in hint_sets:
            try:
                p = ttlg.plan("f64" if c.elem_bytes == 8 else "f32", c.extents, c.perm, **h)
            except ttlg.TtlgError as ex:
                print(json.dumps({"case": c.label(), "hints": h, "error": str(ex)}), flush=True)
                continue
            info = p.describe()
            for _ in range(3):
                p.execute(A.data_ptr(), B.data_ptr(), stream.cuda_stream)
            ts = []
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            for _ in range(args.reps):
                e0.record()
                p.execute(A.data_ptr(), B.data_ptr(), stream.cuda_stream)
                e1.record()
                e1.synchronize()
                ts.append(e0.elapsed_time(e1))
            med = statistics.median(ts)
            print(json.dumps({
                "case": c.label(), "hints": h, "schema": info["schema"],
                "gbs": c.alg_bytes / med / 1e6, "ms": med,
                "pred_ms": info["predicted_seconds"] * 1e3,
                "W": info["access_bytes"], "fused": info["fused_extents"],
                "fperm": info["fused_perm"], "tile": info["tile_extents"],
                "LA": info["in_run"], "LB": info["out_run"], "tiles": info["num_tiles"],
                "grid": info["grid"], "smem": info["smem_bytes"]}), flush=True)
        del A, B
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
