#!/usr/bin/env python
"""Model pick vs measure-mode pick, each timed back to back (R launches between
CUDA events, the bench's steady state), per case of a workload.

  python tools/regret_b2b.py --workload ttc57 --reps 20 --cands 16
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="ttc57")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--cands", type=int, default=16)
    args = ap.parse_args()
    import torch
    import bench
    import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
    from synth import gen_tensor_torch, case_seed
    _, cases = bench._workload(args.workload)
    s = torch.cuda.Stream()
    sp = s.cuda_stream
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    def b2b(p, A, B):
        with torch.cuda.stream(s):
            for _ in range(3):
                p.execute(A.data_ptr(), B.data_ptr(), sp)
            e0.record(s)
            for _ in range(args.reps):
                p.execute(A.data_ptr(), B.data_ptr(), sp)
            e1.record(s)
        e1.synchronize()
        return e0.elapsed_time(e1) / 1e3 / args.reps

    for c in cases:
        dt = "f64" if c.elem_bytes == 8 else "f32"
        A = gen_tensor_torch(case_seed(c.case_id), c.n_elems, c.elem_bytes, device="cuda")
        B = torch.empty_like(A)
        torch.cuda.synchronize()  # A is generated on the default stream
        pm = ttlg.plan(dt, c.extents, c.perm)
        pt = ttlg.plan(dt, c.extents, c.perm)
        pt.tune(A.data_ptr(), B.data_ptr(), sp, args.cands)
        tm1, tt1 = b2b(pm, A, B), b2b(pt, A, B)
        tt2, tm2 = b2b(pt, A, B), b2b(pm, A, B)
        tm, tt = min(tm1, tm2), min(tt1, tt2)
        dm, dtn = pm.describe(), pt.describe()
        print(json.dumps({"case": c.label(), "model_gbs": c.alg_bytes / tm / 1e9,
                          "tuned_gbs": c.alg_bytes / tt / 1e9, "gain": tm / tt - 1,
                          "model": [dm["kernel"], dm["tile_extents"], dm["threads"]],
                          "tuned": [dtn["kernel"], dtn["tile_extents"], dtn["threads"]]}),
              flush=True)
        del A, B


if __name__ == "__main__":
    main()
