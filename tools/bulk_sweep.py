#!/usr/bin/env python
"""k_bulk exploration: per case, every k_bulk candidate slice (forced variant
5 = quad consumers, 6 = gather consumers; ttlg_plan_candidates) timed as a CUDA
graph of R launches, beside the auto plan.  One JSON line per candidate
(calibration data) and a per-case summary line.

  python tools/bulk_sweep.py --workload c2 [--reps 5] [--max-cand 120]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c2")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--max-cand", type=int, default=120)
    ap.add_argument("--stride", type=int, default=1)
    ap.add_argument("--variants", default="5,6",
                    help="comma list of forced kernel variants to enumerate (0 = every "
                         "non-bulk candidate)")
    ap.add_argument("--only", default=None, help="comma-separated case ids")
    args = ap.parse_args()

    import torch
    import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
    from synth import gen_tensor_torch, case_seed
    from cases import workload

    s = torch.cuda.Stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    def gtime(p, A, B):
        with torch.cuda.stream(s):
            p.execute(A.data_ptr(), B.data_ptr(), s.cuda_stream)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(args.reps):
                p.execute(A.data_ptr(), B.data_ptr(), s.cuda_stream)
        ts = []
        with torch.cuda.stream(s):
            g.replay()
            for _ in range(3):
                e0.record(s)
                g.replay()
                e1.record(s)
                e1.synchronize()
                ts.append(e0.elapsed_time(e1) * 1e-3 / args.reps)
        return statistics.median(ts)

    cases = workload(args.workload)[::args.stride]
    if args.only:
        keep = {int(x) for x in args.only.split(",")}
        cases = [c for c in cases if c.case_id in keep]
    variants = [int(v) for v in args.variants.split(",")]
    for c in cases:
        dt = "f64" if c.elem_bytes == 8 else "f32"
        A = gen_tensor_torch(case_seed(c.case_id), c.n_elems, c.elem_bytes, device="cuda:0")
        B = torch.empty_like(A)
        auto = ttlg.plan(dt, c.extents, c.perm)
        ai = auto.describe()
        ta = gtime(auto, A, B)
        best = None
        for v in variants:
            try:
                cands = ttlg.plan_candidates(dt, c.extents, c.perm,
                                             **({"variant": v} if v else {}))
            except ttlg.TtlgError:
                continue
            if len(cands) > args.max_cand:
                cands.sort(key=lambda d: d["predicted_seconds"])
                step = len(cands) / args.max_cand
                cands = [cands[int(i * step)] for i in range(args.max_cand)]
            for cd in cands:
                h = dict(cd["hints"])
                try:
                    p = ttlg.plan(dt, c.extents, c.perm, **h)
                except ttlg.TtlgError:
                    continue
                info = p.describe()
                t = gtime(p, A, B)
                row = {"case": c.label(), "kernel": info["kernel"], "hints": h,
                       "threads": info["threads"], "tile": info["tile_extents"][:info["fused_rank"]],
                       "LA_bytes": info["in_run"] * info["access_bytes"],
                       "LB_bytes": info["out_run"] * info["access_bytes"],
                       "V_bytes": info["tile_volume"] * info["access_bytes"],
                       "tiles": info["num_tiles"], "smem": info["smem_bytes"],
                       "features": info["features"], "pred": info["predicted_seconds"],
                       "meas": t, "gbs": c.alg_bytes / t / 1e9}
                print(json.dumps(row), flush=True)
                if best is None or t < best["meas"]:
                    best = row
        print(json.dumps({"summary": c.label(), "auto_kernel": ai["kernel"],
                          "auto_gbs": c.alg_bytes / ta / 1e9,
                          "best": None if best is None else
                          {k: best[k] for k in ("kernel", "gbs", "tile", "threads", "LA_bytes",
                                                "LB_bytes", "V_bytes")}}), flush=True)
        del A, B
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
