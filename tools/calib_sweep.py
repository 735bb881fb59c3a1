#!/usr/bin/env python
"""Calibration / measure-mode sweep (§V "DataSet" L1298-1313 and
"Model" L1402-1419, re-done on B200): for each case, enumerate the planner's
candidates (ttlg_plan_candidates), execute up to --max-cand of them and record
(features, predicted, measured) per candidate as JSON lines.

  python tools/calib_sweep.py --group c2 --max-cand 40 > calib_c2.jsonl
  python tools/calib_sweep.py --recipe 60 --seed 1   (random A17-recipe cases)
"""
from __future__ import annotations

import argparse
import itertools
import json
import math
import os
import random
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def recipe_cases(n, seed, lo_mb=32, hi_mb=512, log_size=False):
    """Paper dataset recipe (L1298-1313): ranks 3-6, any permutation, five extent
    orderings (equal, increasing, decreasing, up-down, down-up), volume range."""
    from synth.configs import Case
    rng = random.Random(seed)
    out = []
    for k in range(n):
        d = rng.randint(3, 6)
        eb = rng.choice([4, 8])
        if log_size:
            target = math.exp(rng.uniform(math.log(lo_mb), math.log(hi_mb))) * 2 ** 20 / eb
        else:
            target = rng.uniform(lo_mb, hi_mb) * 2 ** 20 / eb
        base = target ** (1.0 / d)
        kind = rng.choice(["eq", "inc", "dec", "updown", "downup"])
        f = [1.0] * d
        for i in range(d):
            t = i / max(1, d - 1)
            f[i] = {"eq": 1.0, "inc": 0.5 + t, "dec": 1.5 - t,
                    "updown": 0.6 + 0.8 * (1 - abs(2 * t - 1)),
                    "downup": 0.6 + 0.8 * abs(2 * t - 1)}[kind]
        g = (1.0 / (1e-9 + float(math.prod(f)))) ** (1.0 / d)
        ext = [max(2, int(round(base * fi * g * rng.uniform(0.9, 1.1)))) for fi in f]
        perm = list(range(d))
        while perm == list(range(d)):
            rng.shuffle(perm)
        out.append(Case(8000 + k, tuple(ext), tuple(perm), eb, f"recipe-{kind}"))
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--group", default=None)
    ap.add_argument("--recipe", type=int, default=0)
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--lo-mb", type=float, default=32.0)
    ap.add_argument("--hi-mb", type=float, default=512.0)
    ap.add_argument("--log-size", action="store_true", help="tensor sizes log-uniform")
    ap.add_argument("--max-cand", type=int, default=40)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--graph", type=int, default=0,
                    help="time R back-to-back launches captured as one CUDA graph (per-launch "
                         "time = replay / R) instead of an event pair around one launch")
    ap.add_argument("--stride", type=int, default=1)
    ap.add_argument("--ids", default="", help="comma list of case ids to keep")
    ap.add_argument("--threads", default="", help="comma list of block sizes to try per candidate")
    ap.add_argument("--top", action="store_true",
                    help="measure the linear screen's best candidates instead of a spread")
    args = ap.parse_args()

    import torch
    import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
    from synth import configs, gen_tensor_torch, case_seed

    cases = []
    if args.group:
        cases += configs.all_configs()[args.group][::args.stride]
    if args.recipe:
        cases += recipe_cases(args.recipe, args.seed, args.lo_mb, args.hi_mb, args.log_size)
    if args.ids:
        keep = {int(x) for x in args.ids.split(",")}
        cases = [c for c in cases if c.case_id in keep]
    dev = torch.device("cuda:0")
    stream = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    gs = torch.cuda.Stream()
    for c in cases:
        dt = "f64" if c.elem_bytes == 8 else "f32"
        cands = ttlg.plan_candidates(dt, c.extents, c.perm)
        auto = ttlg.plan(dt, c.extents, c.perm).describe()
        if len(cands) > args.max_cand:
            cands.sort(key=lambda d: d["predicted_seconds"])
            if args.top:
                # the linear screen's best: the region the ranking stage must order
                cands = cands[:args.max_cand]
            else:
                # an even spread over the whole predicted range
                step = len(cands) / args.max_cand
                cands = [cands[int(i * step)] for i in range(args.max_cand)]
        A = gen_tensor_torch(case_seed(c.case_id), c.n_elems, c.elem_bytes, device=dev)
        B = torch.empty_like(A)
        thr = [int(x) for x in args.threads.split(",") if x] or [0]
        for cd, th in [(cd, th) for cd in cands for th in thr]:
            h = dict(cd["hints"])
            if th:
                h["threads"] = th
            try:
                p = ttlg.plan(dt, c.extents, c.perm, **h)
            except ttlg.TtlgError:
                continue
            info = p.describe()
            for _ in range(2):
                p.execute(A.data_ptr(), B.data_ptr(), stream.cuda_stream)
            ts = []
            if args.graph:
                # back-to-back launches as one CUDA graph (no launch gaps: the
                # kernel time a bench step sees; an event pair around ONE launch
                # after a sync also times the host's launch latency, which
                # dominates tensors below a few MB)
                torch.cuda.synchronize()
                g = torch.cuda.CUDAGraph()
                with torch.cuda.graph(g, stream=gs):
                    for _ in range(args.graph):
                        p.execute(A.data_ptr(), B.data_ptr(), gs.cuda_stream)
                with torch.cuda.stream(gs):
                    g.replay()
                    for _ in range(args.reps):
                        e0.record(gs)
                        g.replay()
                        e1.record(gs)
                        e1.synchronize()
                        ts.append(e0.elapsed_time(e1) * 1e-3 / args.graph)
                del g
            else:
                for _ in range(args.reps):
                    e0.record()
                    p.execute(A.data_ptr(), B.data_ptr(), stream.cuda_stream)
                    e1.record()
                    e1.synchronize()
                    ts.append(e0.elapsed_time(e1) * 1e-3)
            t = statistics.median(ts)
            print(json.dumps({
                "case": c.label(), "group": c.group, "bytes": c.alg_bytes, "W": info["access_bytes"],
                "schema": info["schema"], "kernel": info["kernel"], "hints": h,
                "threads": info["threads"], "kernel_hint": h.get("variant", 0),
                "tile": info["tile_extents"], "LA": info["in_run"], "LB": info["out_run"],
                "V": info["tile_volume"], "tiles": info["num_tiles"], "grid": info["grid"],
                "occ": info["occupancy"], "nstage": info["stages"], "features": info["features"],
                "pred": info["predicted_seconds"], "meas": t, "gbs": c.alg_bytes / t / 1e9,
                "timing": f"graph{args.graph}" if args.graph else "event",
                "is_auto": info["tile_extents"] == auto["tile_extents"]
                and info["schema"] == auto["schema"]}), flush=True)
        del A, B
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
