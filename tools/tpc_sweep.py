#!/usr/bin/env python
"""Tiles per CTA (tpc) for the model's own tile choice: time the auto plan's
tile box / kernel / block size with grid = ceil(tiles / tpc), tpc = 1..4,
back to back (R launches between two events), per case of a workload.

  python tools/tpc_sweep.py --workload ttc57 --stride 3
"""
import argparse
import json
import math
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="ttc57")
    ap.add_argument("--stride", type=int, default=1)
    ap.add_argument("--reps", type=int, default=20)
    args = ap.parse_args()
    import torch
    import bench
    import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
    from synth import gen_tensor_torch, case_seed
    _, cases = bench._workload(args.workload)
    s = torch.cuda.Stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for c in cases[::args.stride]:
        dt = "f64" if c.elem_bytes == 8 else "f32"
        A = gen_tensor_torch(case_seed(c.case_id), c.n_elems, c.elem_bytes, device="cuda")
        B = torch.empty_like(A)
        torch.cuda.synchronize()  # A is generated on the default stream
        d = ttlg.plan(dt, c.extents, c.perm).describe()
        if d["kernel"] not in ("quad", "tile"):
            continue
        h = ttlg.candidate_hints(d)
        out = {"case": c.label(), "kernel": d["kernel"], "tiles": d["num_tiles"],
               "auto_grid": d["grid"]}
        for tpc in (1, 2, 3, 4):
            p = ttlg.plan(dt, c.extents, c.perm, grid=math.ceil(d["num_tiles"] / tpc), **h)
            with torch.cuda.stream(s):
                for _ in range(3):
                    p.execute(A.data_ptr(), B.data_ptr(), s.cuda_stream)
                e0.record(s)
                for _ in range(args.reps):
                    p.execute(A.data_ptr(), B.data_ptr(), s.cuda_stream)
                e1.record(s)
            e1.synchronize()
            out[f"tpc{tpc}"] = round(c.alg_bytes * args.reps / (e0.elapsed_time(e1) / 1e3) / 1e9)
        print(json.dumps(out), flush=True)
        del A, B


if __name__ == "__main__":
    main()
