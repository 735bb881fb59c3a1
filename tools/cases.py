#!/usr/bin/env python
"""Per-case floor table (VERDICT r1 "Next round" 2): every case of a workload
timed on its own as ONE CUDA graph of R back-to-back `ttlg_execute` launches
of its pre-built plan (no event pairs between launches), beside a graph of R
same-size cudaMemcpyAsync device-to-device copies (the case-size-matched D2D
denominator of the north star's ">= 90 % of D2D").

  python tools/cases.py --workload c2 [--reps 20] [--trials 5] [--out f.json]

Per case: GB/s = R * 2*N*s / t, the D2D GB/s of the same
byte count, their ratio, the fraction of the measured HBM peak, the plan
(schema, kernel, tile), predicted vs measured seconds (model error), and the
strict Alg. 1 label is NOT used here (that is test infrastructure).
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


def workload(name):
    from synth import configs
    table = {"c1": configs.config1, "c2": configs.config2, "c3": configs.config3,
             "c4": configs.config4, "c5": configs.config5, "fig13": configs.fig13,
             "720-15": lambda: configs.sweep720(15), "720-16": lambda: configs.sweep720(16),
             "720-17": lambda: configs.sweep720(17)}
    if name == "fmlrows":
        return fml_rows()
    return table[name]()


def fml_rows():
    """FML rows that are not 16-byte multiples, 64-2048+ bytes long: [n0, m, k]
    `0 2 1` (fp64 odd n0, fp32 n0 = 4j+-1), ~256 MB per tensor (k_direct vs k_rows)."""
    from synth.configs import Case
    out = []
    shapes = [(8, n0) for n0 in (15, 31, 47, 63, 95, 127, 191, 255, 383, 511, 1023, 2047)] + \
             [(4, n0) for n0 in (63, 127, 255, 511, 1023, 2047)]
    for i, (s, n0) in enumerate(shapes):
        m = max(3, int(round((256 * 2 ** 20 / (s * n0)) ** 0.5))) | 1
        # all-odd extents: every row keeps its 16-byte phase (as 127^4)
        out.append(Case(9000 + i, (n0, m, m + 2), (0, 2, 1), s, "fmlrows"))
        if s == 8 and n0 in (127, 255, 1023):  # half the rows change phase
            out.append(Case(9100 + i, (n0, m + 1, m + 2), (0, 2, 1), s, "fmlrows"))
    return out


_cudart = None


def memcpy_d2d(dst: int, src: int, nbytes: int, stream: int):
    """cudaMemcpyAsync(dst, src, nbytes, cudaMemcpyDeviceToDevice, stream) -- the
    north star's D2D denominator (torch's copy_ falls back to an unvectorised
    kernel for odd element counts: 3 TB/s on 17^6 fp64)."""
    import ctypes
    global _cudart
    if _cudart is None:
        import paper_conf_ipps_veduradasskhpkn18_b200  # noqa: F401  (loads libcudart.so.12)
        _cudart = ctypes.CDLL("libcudart.so.12")
        _cudart.cudaMemcpyAsync.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t,
                                            ctypes.c_int, ctypes.c_void_p]
    rc = _cudart.cudaMemcpyAsync(dst, src, nbytes, 3, stream)
    if rc != 0:
        raise RuntimeError(f"cudaMemcpyAsync failed: {rc}")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="c2")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--trials", type=int, default=5)
    ap.add_argument("--out", default=None)
    ap.add_argument("--only", default=None, help="comma-separated case ids")
    ap.add_argument("--hints", default=None, help="json dict of plan hints for every case")
    ap.add_argument("--bulk", action="store_true",
                    help="per case: the auto plan's slice with the k_bulk kernel (quad "
                         "consumers for k_quad plans, else gather); the model's own k_bulk "
                         "slice when the auto slice does not apply")
    args = ap.parse_args()

    import torch
    import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
    from synth import gen_tensor_torch, case_seed

    peak = 6552.6
    pp = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(pp):
        peak = json.load(open(pp))["hbm_gbs"]
    cases = workload(args.workload)
    if args.only:
        keep = {int(x) for x in args.only.split(",")}
        cases = [c for c in cases if c.case_id in keep]
    hints = json.loads(args.hints) if args.hints else {}
    dev = torch.device("cuda:0")
    s = torch.cuda.Stream(device=dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    def time_graph(g):
        with torch.cuda.stream(s):
            for _ in range(2):
                g.replay()
            ts = []
            for _ in range(args.trials):
                e0.record(s)
                g.replay()
                e1.record(s)
                e1.synchronize()
                ts.append(e0.elapsed_time(e1) * 1e-3)
        return statistics.median(ts)

    rows, bufs = [], {}
    d2d_cache = {}
    t_start = time.time()
    for c in cases:
        key = (c.n_elems, c.elem_bytes)
        if key not in bufs:
            bufs.clear()
            torch.cuda.empty_cache()
            A = gen_tensor_torch(case_seed(c.case_id), c.n_elems, c.elem_bytes, device=dev)
            bufs[key] = (A, torch.empty_like(A))
        A, B = bufs[key]
        dt = "f64" if c.elem_bytes == 8 else "f32"
        if args.bulk:
            a = ttlg.plan(dt, c.extents, c.perm).describe()
            h = ttlg.candidate_hints(a)
            h.pop("threads", None)
            h["variant"] = 5 if a["kernel"] == "quad" else 6
            p = None
            for hh in (h, {"variant": h["variant"]}, {"variant": 6}):
                try:
                    p = ttlg.plan(dt, c.extents, c.perm, **hh)
                    break
                except ttlg.TtlgError:
                    continue
            if p is None:
                p = ttlg.plan(dt, c.extents, c.perm)
        else:
            p = ttlg.plan(dt, c.extents, c.perm, **hints)
        info = p.describe()
        with torch.cuda.stream(s):
            p.execute(A.data_ptr(), B.data_ptr(), s.cuda_stream)  # warm (function attributes)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(args.reps):
                p.execute(A.data_ptr(), B.data_ptr(), s.cuda_stream)
        t = time_graph(g) / args.reps
        del g
        nbytes = c.alg_bytes
        if nbytes not in d2d_cache:
            gd = torch.cuda.CUDAGraph()
            with torch.cuda.graph(gd, stream=s):
                for _ in range(args.reps):
                    memcpy_d2d(B.data_ptr(), A.data_ptr(), c.n_elems * c.elem_bytes, s.cuda_stream)
            d2d_cache[nbytes] = nbytes / (time_graph(gd) / args.reps) / 1e9
            del gd
        gbs = nbytes / t / 1e9
        d2d = d2d_cache[nbytes]
        rows.append({"case": c.label(), "schema": info["schema"], "kernel": info["kernel"],
                     "access_bytes": info["access_bytes"], "threads": info["threads"],
                     "tile": info["tile_extents"][:info["fused_rank"]],
                     "fused": info["fused_extents"][:info["fused_rank"]],
                     "fperm": info["fused_perm"][:info["fused_rank"]],
                     "us": t * 1e6, "gbs": gbs, "d2d_gbs": d2d, "frac_d2d": gbs / d2d,
                     "frac_peak": gbs / peak, "pred_us": info["predicted_seconds"] * 1e6,
                     "model_err": abs(info["predicted_seconds"] - t) / t})
        print(json.dumps(rows[-1]), flush=True)
    tot_b = sum(c.alg_bytes for c in cases)
    tot_t = sum(r["us"] for r in rows) * 1e-6
    summ = {"workload": args.workload, "reps": args.reps, "trials": args.trials, "peak": peak,
            "timing": "per case: one CUDA graph of `reps` back-to-back ttlg_execute launches "
                      "(median of `trials` replays); D2D: a graph of `reps` same-size "
                      "device-to-device copies",
            "aggregate_gbs": tot_b / tot_t / 1e9,
            "min_frac_d2d": min(r["frac_d2d"] for r in rows),
            "below_0.9_d2d": [r["case"] for r in rows if r["frac_d2d"] < 0.9],
            "mean_model_err": statistics.mean(r["model_err"] for r in rows),
            "wall_s": time.time() - t_start, "cases": rows}
    print(json.dumps({k: v for k, v in summ.items() if k != "cases"}), flush=True)
    if args.out:
        os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
        with open(args.out, "w") as f:
            json.dump(summ, f, indent=1)


if __name__ == "__main__":
    main()
