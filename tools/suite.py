#!/usr/bin/env python
"""Per-configuration results table (BASELINE configs 1-5 and the paper's
workloads): model-chosen plan, measured GB/s (CUDA events, median of reps),
fraction of the same-size device-to-device copy and of the measured HBM peak,
model-predicted vs measured time, and -- for config 3 -- single-use
(ttlg_transpose per call, plan cost included) vs repeated-use (ttlg_execute of
a pre-built plan) time, K back-to-back calls each, host wall clock to sync.

  python tools/suite.py --groups c1,c2,c3,c4,c5 [--out gpurun_out/suite.jsonl]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--groups", default="c1,c2,c3,c4,c5")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--single-k", type=int, default=50)
    ap.add_argument("--out", default=None)
    ap.add_argument("--check", action="store_true", help="sampled parity vs the oracle")
    args = ap.parse_args()

    import torch
    import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
    from synth import configs, gen_tensor_torch, case_seed

    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] \
        if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    groups = {"c1": configs.config1, "c2": configs.config2, "c3": configs.config3,
              "c4": configs.config4, "c5": configs.config5,
              "720-16": lambda: configs.sweep720(16), "720-15": lambda: configs.sweep720(15),
              "720-17": lambda: configs.sweep720(17), "fig13": configs.fig13,
              "fig5": lambda: [configs.fig5_case()]}
    out = open(args.out, "w") if args.out else sys.stdout
    dev = torch.device("cuda:0")
    st = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    def timed(fn, reps):
        for _ in range(3):
            fn()
        ts = []
        for _ in range(reps):
            e0.record()
            fn()
            e1.record()
            e1.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e-3)
        return statistics.median(ts)

    for g in args.groups.split(","):
        for c in groups[g]():
            dt = "f64" if c.elem_bytes == 8 else "f32"
            A = gen_tensor_torch(case_seed(c.case_id), c.n_elems, c.elem_bytes, device=dev)
            B = torch.empty_like(A)
            p = ttlg.plan(dt, c.extents, c.perm)
            info = p.describe()
            t = timed(lambda: p.execute(A.data_ptr(), B.data_ptr(), st.cuda_stream), args.reps)
            check = None
            if args.check:
                # sampled parity against the oracle's definition (lin_B -> lin_A)
                import numpy as np
                import oracle
                from synth import gen_at_np
                rng = np.random.default_rng(c.case_id)
                linB = np.unique(np.concatenate([rng.integers(0, c.n_elems, 4096),
                                                 [0, c.n_elems - 1]]))
                iv = torch.int64 if c.elem_bytes == 8 else torch.int32
                got = B.view(iv)[torch.from_numpy(linB).to(dev)].cpu().numpy()
                got = got.view(np.uint64 if c.elem_bytes == 8 else np.uint32)
                exp = gen_at_np(case_seed(c.case_id),
                                oracle.source_index(c.extents, c.perm, linB), c.elem_bytes)
                check = bool(np.array_equal(got, exp))
            td = timed(lambda: B.copy_(A), args.reps)
            rec = {"group": g, "case": c.label(), "schema": info["schema"], "kernel": info["kernel"],
                   "bytes": c.alg_bytes, "ms": t * 1e3, "gbs": c.alg_bytes / t / 1e9,
                   "d2d_gbs": c.alg_bytes / td / 1e9, "frac_d2d": td / t, "frac_peak":
                   c.alg_bytes / t / 1e9 / peak, "pred_ms": info["predicted_seconds"] * 1e3,
                   "model_err": abs(info["predicted_seconds"] - t) / t,
                   "fused_rank": info["fused_rank"], "tile": info["tile_extents"],
                   "parity_sampled": check}
            if g == "c3":
                K = args.single_k
                ext, perm = list(c.extents), list(c.perm)
                torch.cuda.synchronize()
                w0 = time.perf_counter()
                for _ in range(K):
                    p.execute(A.data_ptr(), B.data_ptr(), st.cuda_stream)
                torch.cuda.synchronize()
                rep_t = (time.perf_counter() - w0) / K
                w0 = time.perf_counter()
                for _ in range(K):
                    ttlg.transpose(dt, ext, perm, A.data_ptr(), B.data_ptr(), st.cuda_stream)
                torch.cuda.synchronize()
                single_t = (time.perf_counter() - w0) / K
                rec.update({"repeated_ms": rep_t * 1e3, "single_ms": single_t * 1e3,
                            "single_over_repeated": single_t / rep_t})
            out.write(json.dumps(rec) + "\n")
            out.flush()
            del A, B
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
