#!/usr/bin/env python
"""bench.py -- the driver's benchmark contract for the B200 TTLG library.

Metric (BASELINE.json): effective transpose GB/s = 2*N*sizeof(elem)/time/1e9
(PAPER.md L1501-1505), here summed over one "step" = one pass of the hot path
over the workload: every case of the TTC-like 57-case suite (BASELINE config 2,
SURVEY App. A synthetic re-creation), fp64, 200 MiB per tensor, each case one
`ttlg_execute` of a pre-built plan (repeated-use mode, L1569-1593); the
step's 57 launches are captured once into a CUDA graph and replayed (the same
kernels with the same parameter blocks; direct launches are timed as well and
reported as `direct_launch`, `--no-graph` times only those).

  python bench.py [--gpus N] [--steps K] [--warmup W]
                  [--workload ttc57|ccsdt|smallfvi|c1|sharded|720-15|720-16|720-17|fig13]
  python bench.py --impl reference ...   (the oracle on the host cores)

Inputs are generated on the device by the shared SplitMix64 generator
(synth/), resident in HBM before the timed region; every tensor (200 MiB in +
200 MiB out) exceeds the 126 MB L2, so no flush is needed between launches.
Timing: CUDA events on the launching stream, W warm-up steps, K timed steps,
barrier + synchronize on both sides, max over ranks.  Multi-GPU (torchrun):
each rank transposes the full suite on its own GPU (independent problems, no
data-path collective) -> "scaling": "weak".
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

PEAK_FALLBACK_GBS = 6650.0  # B200_PROFILING.md fallback (only if MEASURED_PEAKS.json absent)


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)", d
    return PEAK_FALLBACK_GBS, "fallback (B200_PROFILING.md)", {}


def _workload(name):
    from synth import configs
    if name == "ttc57":
        return "ttc57-fp64-200MiB (BASELINE config 2, synthetic re-creation)", configs.config2()
    if name == "ccsdt":
        return "ccsdt-rank6-fp64 (BASELINE config 3)", configs.config3()
    if name == "smallfvi":
        return "smallfvi-rank3-fp32 (BASELINE config 4)", configs.config4()
    if name == "c1":
        return "rank4-16^4-fp64 all 24 perms (BASELINE config 1)", configs.config1()
    if name in ("720-15", "720-16", "720-17"):
        e = int(name.split("-")[1])
        return (f"all 720 perms of {e}^6 fp64 (PAPER.md L1484-1493, Fig. 10/11 workload)",
                configs.sweep720(e))
    if name == "fig13":
        return "Fig. 13 sizes n^4 fp64 perm 0 2 1 3 (PAPER.md L1881-1895)", configs.fig13()
    raise SystemExit(f"unknown workload {name}")


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self.proc = None

    def start(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.th = threading.Thread(target=self._read, daemon=True)
            self.th.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.samples.append([x.strip() for x in line.split(",")])

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for s in self.samples:
            try:
                sm.append(float(s[0]))
                mx.append(float(s[1]))
                for nm, v in zip(names, s[4:8]):
                    if v.strip().lower() == "active":
                        reasons.add(nm)
            except (ValueError, IndexError):
                continue
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def cpu_baseline(cases, budget_s=12.0, threads=None):
    """The oracle as it stands (oracle.c d-nested loop, threaded over the
    outermost index) on the host cores, on a bounded sample of the workload."""
    import numpy as np
    import oracle
    from synth import gen_tensor_np, case_seed
    cores = threads or len(os.sched_getaffinity(0))
    done, t_total, nbytes = [], 0.0, 0
    for c in cases:
        A = gen_tensor_np(case_seed(c.case_id), c.n_elems, c.elem_bytes)
        t0 = time.perf_counter()
        oracle.transpose(A, c.extents, c.perm, threads=cores)
        t_total += time.perf_counter() - t0
        nbytes += c.alg_bytes
        done.append(c.label())
        del A
        if t_total >= budget_s:
            break
    out = {"value": nbytes / t_total / 1e9, "unit": "GB/s", "cores": cores, "kind": "oracle",
           "sample": f"{len(done)} of {len(cases)} cases ({', '.join(done[:4])}"
                     f"{', ...' if len(done) > 4 else ''}), {t_total:.1f} s of oracle time"}
    if threads is None and cores > 1:
        # the oracle single-threaded too (a smaller budget, the
        # first cases of the same sample)
        st = cpu_baseline(cases, budget_s=max(2.0, budget_s / 3), threads=1)
        out["single_thread"] = {"value": st["value"], "unit": "GB/s", "cores": 1,
                                "sample": st["sample"]}
    return out


def run_reference(args, rank, world):
    """--impl reference: the oracle on the host cores (rank 0 only)."""
    if rank != 0:
        return
    import oracle
    from synth import gen_tensor_np, case_seed, configs
    if args.workload == "sharded":
        # config 5: one rank's slab at P = 8 ([64, 64, 64, 64, 16] fp32, 1 GiB),
        # each of the five perms as a local transposition (the bounded sample)
        name = "c5-8GiB-rank5-fp32 sharded (BASELINE config 5): one P=8 slab per case"
        cases = [configs.Case(c.case_id, c.extents[:-1] + (c.extents[-1] // 8,), c.perm,
                              c.elem_bytes, c.group) for c in configs.config5()]
    else:
        name, cases = _workload(args.workload)
    cores = len(os.sched_getaffinity(0))
    # each step = a bounded sample of the workload: the next m cases of the
    # suite, round-robin (warm-up steps advance too), so K steps sweep it
    m = max(1, min(len(cases), args.ref_cases_per_step))
    times, nb, seen = [], [], set()
    for step in range(args.warmup + args.steps):
        dt_step, nb_step = 0.0, 0
        for i in range(m):
            c = cases[(step * m + i) % len(cases)]
            A = gen_tensor_np(case_seed(c.case_id), c.n_elems, c.elem_bytes)
            t0 = time.perf_counter()
            oracle.transpose(A, c.extents, c.perm, threads=cores)
            dt_step += time.perf_counter() - t0
            nb_step += c.alg_bytes
            if step >= args.warmup:
                seen.add(c.case_id)
            del A
        if step >= args.warmup:
            times.append(dt_step)
            nb.append(nb_step)
    value = sum(nb) / sum(times) / 1e9
    line = {"impl": "reference", "metric": "effective transpose GB/s (2*N*s/time)",
            "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * sum(times) / len(times),
            "higher_is_better": True,
            "scaling": "strong" if args.workload == "sharded" else "weak", "vs_baseline": None,
            "dtype": "f64" if cases[0].elem_bytes == 8 else "f32",
            "data": "synthetic (SplitMix64 bit patterns)",
            "config": {"workload": name,
                       "step": f"{m} cases of the suite per step, round-robin (bounded sample)"},
            "cpu_baseline": {"value": value, "unit": "GB/s", "cores": cores, "kind": "oracle",
                             "sample": f"{len(times)} steps x {m} cases ({len(seen)} distinct "
                                       f"of {len(cases)})"},
            "e2e": {"value": value, "unit": "GB/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_sharded(args, rank, world, local_rank, dev):  # noqa: C901
    """--workload sharded: BASELINE config 5, the 8 GiB rank-5 fp32 tensor
    [64,64,64,64,128] sharded on A's outermost dim across the ranks (one
    process per GPU; the default workload at N > 1).  No-move perms: one local
    transposition per rank, no communication.  Moved perms: the model-chosen
    exchange -- the fused one (ONE batched launch per rank whose
    sub-transpositions store straight into the peers' B slabs over CUDA IPC /
    NVLink) or local transpose -> NCCL all_to_all_single -> fold.  A step =
    the five perms once.  At N = 1 also: the fused exchange of P = 2/4/8
    emulated on this one GPU (every peer slab local) -- its HBM-side cost."""
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
    from paper_conf_ipps_veduradasskhpkn18_b200.sharded import (
        plan_shards, P2PExchange, map_peer_slabs, unmap_peer_slabs, sharded_transpose,
        choose_exchange, NVLINK_GBS)
    from synth import configs, gen_tensor_torch, case_seed

    cases = configs.config5()
    ext = list(cases[0].extents)
    n = 1
    for e in ext:
        n *= e
    n_local = n // world
    stream = torch.cuda.Stream(device=dev)
    sptr = stream.cuda_stream
    A = gen_tensor_torch(case_seed(5000), n_local, 4, device=dev, start=rank * n_local)
    B = torch.empty_like(A)
    if world > 1:
        peers, opened = map_peer_slabs(B)
        nccl_info = {"backend": dist.get_backend(), "communicator_size": dist.get_world_size()}
    else:
        peers, opened = [B.data_ptr()], []
        nccl_info = None
    work = (torch.empty_like(A), torch.empty_like(A)) if world > 1 else None

    def make_ex(perm, out, ptrs, r, P):
        try:
            return P2PExchange(ext, perm, out, peer_ptrs=ptrs, rank=r, world=P)
        except ttlg.TtlgError:  # no p2p plan (sub-box FVI collapses): all-to-all only
            return None
    exs = [make_ex(c.perm, B, peers, rank, world) for c in cases]
    torch.cuda.synchronize()

    def timed(fn, steps):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(steps):
            fn()
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        if world > 1:  # the step time is the slowest rank's
            t = torch.tensor([ms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
            dist.barrier()
        return ms

    def fns_for(c, ex):
        def f_p2p():
            ex.run(A, sptr)

        def f_a2a():
            with torch.cuda.stream(stream):
                sharded_transpose(A, ext, c.perm, work=work)
        return {"p2p": f_p2p, "local": f_p2p, "alltoall": f_a2a}

    per, other, modes = [], {}, {}
    clocks = ClockSampler(local_rank)
    clocks.start()
    time.sleep(0.3)
    for c, ex in zip(cases, exs):
        key = "".join(map(str, c.perm))
        # model-driven choice between the fused exchange and the all-to-all
        mode = choose_exchange(ext, c.perm, world, "f32")["mode"] if world > 1 else "local"
        modes[key] = mode
        fns = fns_for(c, ex)
        for _ in range(args.warmup):
            fns[mode]()
        per.append(timed(fns[mode], args.steps))
        if world > 1 and ex is not None and ex.sp.moved:  # the path not chosen, for comparison
            alt = "alltoall" if mode == "p2p" else "p2p"
            for _ in range(args.warmup):
                fns[alt]()
            other[f"{alt}:{key}"] = 2 * n * 4 * args.steps / (
                timed(fns[alt], args.steps) / 1e3) / 1e9
    clk = clocks.stop()
    total_ms = sum(per)
    value = 2 * n * 4 * len(cases) * args.steps / (total_ms / 1e3) / 1e9
    per_gbs = {"".join(map(str, c.perm)): 2 * n * 4 * args.steps / (m / 1e3) / 1e9
               for c, m in zip(cases, per)}
    # roofline: the local (no-move) transpositions are HBM-bound -- bytes of one
    # rank / that rank's time vs the measured HBM peak; moved perms are bound
    # by NVLink: bus bandwidth = remote bytes per rank / time vs 770 GB/s
    local_keys = [k for k in per_gbs if modes[k] == "local"]
    hbm_achieved = (sum(2 * n_local * 4 * args.steps for _ in local_keys) /
                    (sum(m for c, m in zip(cases, per) if "".join(map(str, c.perm)) in local_keys)
                     / 1e3) / 1e9) if local_keys else None
    nvlink = {}
    for c, m in zip(cases, per):
        k = "".join(map(str, c.perm))
        if modes[k] != "local":
            remote = n_local * 4 * (world - 1) / world * args.steps
            nvlink[k] = {"mode": modes[k], "busbw_gbs": remote / (m / 1e3) / 1e9,
                         "peak_gbs": NVLINK_GBS,
                         "peak_source": "B200_PROFILING.md measured peer copy per direction"}

    # end to end through the public API: each rank's slab from pinned host memory,
    # the sharded transposition, its B slab back to pinned host memory
    e2e = None
    if args.e2e_steps > 0:
        try:
            hA = torch.empty(n_local, dtype=torch.float32, pin_memory=True)
            hA.copy_(A)
            hB = torch.empty(n_local, dtype=torch.float32, pin_memory=True)
            torch.cuda.synchronize()

            def e2e_step():
                with torch.cuda.stream(stream):
                    for c, ex in zip(cases, exs):
                        mode = modes["".join(map(str, c.perm))]
                        A.copy_(hA, non_blocking=True)
                        fns_for(c, ex)[mode]()
                        if world > 1 and mode == "p2p":
                            # peers store into this rank's B: wait for all of them
                            stream.synchronize()
                            dist.barrier()
                        hB.copy_(work[0] if mode == "alltoall" else B, non_blocking=True)
            ms = timed(e2e_step, args.e2e_steps)
            e2e = {"value": 2 * n * 4 * len(cases) * args.e2e_steps / (ms / 1e3) / 1e9,
                   "unit": "GB/s", "h2d_bytes_per_step": len(cases) * n_local * 4 * world,
                   "d2h_bytes_per_step": len(cases) * n_local * 4 * world,
                   "steps": args.e2e_steps,
                   "api": "per rank: pinned host slab -> H2D -> sharded transposition "
                          "(P2PExchange.run / sharded_transpose) -> D2H of the B slab"}
        except Exception as ex_:  # report, do not hide
            e2e = {"value": None, "unit": "GB/s", "error": str(ex_)[:200]}

    emulated = {}
    if rank == 0 and world == 1 and not args.no_emulate:
        # the fused exchange at P = 2/4/8 with every peer slab on this GPU
        Af = A  # world == 1: A is the whole tensor
        for P in (2, 4, 8):
            slabs = [B[q * (n // P):(q + 1) * (n // P)] for q in range(P)]
            ptrs = [t.data_ptr() for t in slabs]
            for c in cases:
                sp = plan_shards(ext, c.perm, P)
                if not sp.moved:
                    continue
                rexs = [make_ex(c.perm, slabs[p], ptrs, p, P) for p in range(P)]
                if rexs[0] is None:
                    continue

                def f_all(rexs=rexs, P=P):
                    for p, ex in enumerate(rexs):
                        ex.run(Af[p * (n // P):(p + 1) * (n // P)], sptr)
                for _ in range(2):
                    f_all()
                ms = timed(f_all, max(2, args.steps // 2))
                emulated[f"P{P}:{''.join(map(str, c.perm))}"] = \
                    2 * n * 4 * max(2, args.steps // 2) / (ms / 1e3) / 1e9
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline([configs.Case(c.case_id, c.extents[:-1] + (c.extents[-1] // 8,),
                                         c.perm, 4, c.group) for c in cases],
                           budget_s=args.cpu_budget)
        cpu["sample"] = "one P=8 slab [64,64,64,64,16] per perm: " + cpu["sample"]
    for ex in exs:
        if ex is not None:
            ex.close()
    unmap_peer_slabs(opened)
    if rank == 0:
        peak, peak_src, _ = _peaks()
        launches = sum(1 if modes[k] != "alltoall" else 2 for k in modes) * args.steps
        line = {
            "metric": "effective transpose GB/s (2*N*s/time)", "value": value, "unit": "GB/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": total_ms / args.steps, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f32",
            "data": "synthetic (SplitMix64 bit patterns, generated on device)",
            "config": {"workload": "c5-8GiB-rank5-fp32 sharded on A's outermost dim (BASELINE config 5)",
                       "extents": ext, "perms": [list(c.perm) for c in cases],
                       "parallelism": f"shard x{world}",
                       "exchange": "per perm, model-chosen: local (no move) | p2p (fused "
                                   "sub-transpositions, one batched launch per rank storing "
                                   "over CUDA IPC / NVLink) | alltoall (local + NCCL "
                                   "all_to_all_single + fold)",
                       "l2": "no flush: 8 GiB tensors (inputs larger than L2)",
                       "process_group": nccl_info},
            "gpu_launches": launches,
            "per_perm_gbs": per_gbs,
            "modes": modes,
            "roofline": {"bound": "hbm", "kernel": "local transpositions (no-move perms)",
                         "achieved": hbm_achieved, "peak": peak, "peak_source": peak_src,
                         "unit": "GB/s", "frac": hbm_achieved / peak if hbm_achieved else None,
                         "traffic": None},
            "nvlink": nvlink or None,
            "other_path_gbs": other or None,
            "p2p_emulated_one_gpu_gbs": emulated or None,
            "frac_of_peak": value / world / peak,
            "clocks": clk,
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)


def spawn_ranks(n: int) -> int:
    """Re-run this command as n ranks under torch.distributed.run (rendezvous
    on 127.0.0.1); returns the launcher's exit code."""
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={n}", "--master-addr=127.0.0.1", f"--master-port={port}",
           os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ttlg", choices=["ttlg", "reference"])
    ap.add_argument("--workload", default=None,
                    help="default: ttc57 at N = 1 (BASELINE config 2, the headline); "
                         "sharded (config 5, the north star's multi-GPU case) at N > 1")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=12.0)
    ap.add_argument("--ref-cases-per-step", type=int, default=6)
    ap.add_argument("--no-graph", action="store_true",
                    help="time the step as direct launches only (default: the step's launches "
                         "captured once into a CUDA graph and replayed; direct launches are "
                         "timed too and reported as direct_launch)")
    ap.add_argument("--no-emulate", action="store_true",
                    help="sharded workload: skip the one-GPU emulation of P = 2/4/8")
    ap.add_argument("--tune", type=int, default=8,
                    help="measure-mode candidates per case for the 'tuned' key (0 = off)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    if "WORLD_SIZE" not in os.environ and args.gpus > 1 and args.impl != "reference":
        # `bench.py --gpus N` without a launcher: start the N ranks ourselves
        # (one process per GPU, the same command under torch.distributed.run)
        sys.exit(spawn_ranks(args.gpus))
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if "WORLD_SIZE" in os.environ and args.gpus != world:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}")
    if args.workload is None:
        args.workload = "ttc57" if args.gpus == 1 else "sharded"
    if args.impl == "reference":
        run_reference(args, rank, args.gpus)
        return

    import numpy as np
    import torch
    import torch.distributed as dist

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)

    import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
    from synth import gen_tensor_torch, case_seed

    if args.workload == "sharded":
        run_sharded(args, rank, world, local_rank, dev)
        if world > 1:
            dist.destroy_process_group()
        return
    name, cases = _workload(args.workload)
    peak, peak_src, peaks = _peaks()
    stream = torch.cuda.Stream(device=dev)
    sptr = stream.cuda_stream

    # ---- resident inputs + plans (outside the timed region).  Cases of one
    # size share one A/B pair when the suite would not fit otherwise (the 720
    # perms of one shape: the operation is content-agnostic)
    As, Bs, plans, infos = [], [], [], []
    share = sum(2 * c.n_elems * c.elem_bytes for c in cases) > 48 * 2 ** 30
    pool = {}
    for c in cases:
        key = (c.n_elems, c.elem_bytes)
        if share and key in pool:
            A, B = pool[key]
        else:
            A = gen_tensor_torch(case_seed(c.case_id), c.n_elems, c.elem_bytes, device=dev)
            B = torch.empty_like(A)
            pool[key] = (A, B)
        As.append(A)
        Bs.append(B)
        p = ttlg.plan("f64" if c.elem_bytes == 8 else "f32", c.extents, c.perm)
        plans.append(p)
        infos.append(p.describe())
    torch.cuda.synchronize()
    step_bytes = sum(c.alg_bytes for c in cases)

    def kname(info):
        return f"k_{info['kernel']}"

    def one_step(evs=None):
        with torch.cuda.stream(stream):
            for i, p in enumerate(plans):
                if evs is not None:
                    evs[i][0].record(stream)
                p.execute(As[i].data_ptr(), Bs[i].data_ptr(), sptr)
                if evs is not None:
                    evs[i][1].record(stream)

    for _ in range(args.warmup):
        one_step()
    graph = None
    if not args.no_graph:
        # the step captured once into a CUDA graph (kernel nodes with their
        # parameter blocks baked in) and replayed: no per-launch host work
        torch.cuda.synchronize()
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph, stream=stream):
            for i, p in enumerate(plans):
                p.execute(As[i].data_ptr(), Bs[i].data_ptr(), stream.cuda_stream)
        for _ in range(2):
            graph.replay()
        torch.cuda.synchronize()
    torch.cuda.synchronize()

    # ---- timed region (device events on the launching stream)
    evs = [[(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
            for _ in plans] for _ in range(args.steps)]
    clocks = ClockSampler(local_rank)
    clocks.start()
    time.sleep(0.3)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    t_start.record(stream)
    for s in range(args.steps):
        if graph is not None:
            with torch.cuda.stream(stream):
                graph.replay()
        else:
            one_step()
    t_end.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    elapsed_ms = t_start.elapsed_time(t_end)
    if world > 1:
        t = torch.tensor([elapsed_ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        elapsed_ms = float(t.item())
    launches = len(plans) * args.steps
    direct = None
    if graph is not None:
        # the same K steps as direct launches (one ttlg_execute per case)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        d0, d1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        d0.record(stream)
        for _ in range(args.steps):
            one_step()
        d1.record(stream)
        torch.cuda.synchronize()
        dms = d0.elapsed_time(d1)
        if world > 1:
            t = torch.tensor([dms], device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            dms = float(t.item())
        direct = {"value": world * step_bytes * args.steps / (dms / 1e3) / 1e9, "unit": "GB/s",
                  "ms_per_step": dms / args.steps}
    # per-kernel durations: the same K steps again, the launches of each kernel
    # grouped between ONE event pair per kernel and step (an event record
    # between two launches adds a bubble, so per-launch pairs would inflate
    # every duration; the headline step above is timed uninstrumented)
    kinds = sorted({kname(inf) for inf in infos})
    kev = {k: [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
               for _ in range(args.steps)] for k in kinds}
    kgraph = {}
    if graph is not None:  # each kernel's launches as one graph, like the step
        for k in kinds:
            kgraph[k] = torch.cuda.CUDAGraph()
            with torch.cuda.graph(kgraph[k], stream=stream):
                for i, p in enumerate(plans):
                    if kname(infos[i]) == k:
                        p.execute(As[i].data_ptr(), Bs[i].data_ptr(), sptr)
        torch.cuda.synchronize()
    with torch.cuda.stream(stream):
        for s in range(args.steps):
            for k in kinds:
                kev[k][s][0].record(stream)
                if k in kgraph:
                    kgraph[k].replay()
                else:
                    for i, p in enumerate(plans):
                        if kname(infos[i]) == k:
                            p.execute(As[i].data_ptr(), Bs[i].data_ptr(), sptr)
                kev[k][s][1].record(stream)
    # per-case durations (model error, per-case table): an event pair per
    # launch; in graph mode, cases moving < 32 MB (tensors < 16 MB, kernels of a few
    # us: an event pair per launch times the host's launch rate there) as
    # their own graph of K back-to-back launches between one event pair --
    # the two timings the model was calibrated with (cal35 / cal33; the third
    # and second tree sets report the predictions on either side)
    for s in range(args.steps):
        one_step(evs[s])
    torch.cuda.synchronize()
    per_case_ms = [[evs[s][i][0].elapsed_time(evs[s][i][1]) for s in range(args.steps)]
                   for i in range(len(plans))]
    small_case = [c.alg_bytes < 32 * 2 ** 20 for c in cases]  # model.h kSmallTraffic
    if graph is not None and any(small_case):
        for i, p in enumerate(plans):
            if not small_case[i]:
                continue
            cg = torch.cuda.CUDAGraph()
            with torch.cuda.graph(cg, stream=stream):
                for _ in range(args.steps):
                    p.execute(As[i].data_ptr(), Bs[i].data_ptr(), sptr)
            with torch.cuda.stream(stream):
                cg.replay()
                ms = []
                for _ in range(3):
                    evs[0][i][0].record(stream)
                    cg.replay()
                    evs[0][i][1].record(stream)
                    evs[0][i][1].synchronize()
                    ms.append(evs[0][i][0].elapsed_time(evs[0][i][1]) / args.steps)
            per_case_ms[i] = ms
            del cg
    torch.cuda.synchronize()
    clk = clocks.stop()
    groups = {}
    for i, info in enumerate(infos):
        k = kname(info)
        g = groups.setdefault(k, {"ms": 0.0, "bytes": 0, "launches": 0})
        g["bytes"] += cases[i].alg_bytes * args.steps
        g["launches"] += args.steps
    for k, g in groups.items():
        g["ms"] = sum(a.elapsed_time(b) for a, b in kev[k])
    dom = max(groups, key=lambda k: groups[k]["ms"])
    dg = groups[dom]
    achieved = dg["bytes"] / (dg["ms"] / 1e3) / 1e9
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tpath):
        try:
            with open(tpath) as f:
                tr = json.load(f)
            traffic = tr.get(args.workload, {}).get(dom.split("[")[0])
        except Exception:
            traffic = None
    med = [statistics.median(x) for x in per_case_ms]
    errs = [abs(m * 1e-3 - inf["predicted_seconds"]) / (m * 1e-3) for m, inf in zip(med, infos)]

    # same-size device-to-device copy (the north star's "% of D2D" denominator)
    d2d_ms = []
    big = max(range(len(cases)), key=lambda i: cases[i].alg_bytes)
    src, dst = As[big], Bs[big]
    with torch.cuda.stream(stream):
        for _ in range(3):
            dst.copy_(src)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(10):
            dst.copy_(src)
        e1.record(stream)
    torch.cuda.synchronize()
    d2d_gbs = 10 * cases[big].alg_bytes / (e0.elapsed_time(e1) / 1e3) / 1e9

    value = world * step_bytes * args.steps / (elapsed_ms / 1e3) / 1e9

    # ---- measure-mode refinement (N2): tune each plan over the model's short
    # list, re-time the step; reported beside the model-driven headline value
    tuned = None
    if args.tune > 0:
        tplans = []
        for i, c in enumerate(cases):
            q = ttlg.plan("f64" if c.elem_bytes == 8 else "f32", c.extents, c.perm)
            q.tune(As[i].data_ptr(), Bs[i].data_ptr(), sptr, args.tune)
            tplans.append(q)
        torch.cuda.synchronize()
        with torch.cuda.stream(stream):
            for i, q in enumerate(tplans):
                q.execute(As[i].data_ptr(), Bs[i].data_ptr(), sptr)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            for _ in range(args.steps):
                for i, q in enumerate(tplans):
                    q.execute(As[i].data_ptr(), Bs[i].data_ptr(), sptr)
            e1.record(stream)
        torch.cuda.synchronize()
        tv = step_bytes * args.steps / (e0.elapsed_time(e1) / 1e3) / 1e9
        tuned = {"value": tv, "unit": "GB/s", "frac_of_d2d": tv / d2d_gbs,
                 "model_regret_pct": 100.0 * (tv / ((direct["value"] if direct else value) /
                                                    world) - 1.0),
                 "candidates_per_case": args.tune,
                 "api": "ttlg_plan_tune (measure mode over the model's short list)"}
        del tplans

    # ---- end to end: C-ABI call with HOST buffers, H2D + D2H inside the timed region
    e2e = None
    if args.e2e_steps > 0:
        try:
            # one pinned host input per tensor size (the operation is
            # content-agnostic; every case still copies its whole input H2D and
            # its whole output D2H inside the timed region), so N ranks pin
            # ~2 x 200 MiB each rather than the whole suite
            hpool = {}
            for A in As:
                key = (A.numel(), A.dtype)
                if key not in hpool:
                    h = torch.empty(A.numel(), dtype=A.dtype, pin_memory=True)
                    h.copy_(A)
                    hpool[key] = h
            hA = [hpool[(A.numel(), A.dtype)] for A in As]
            hB = torch.empty(max(A.numel() for A in As), dtype=As[0].dtype, pin_memory=True)
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            for _ in range(args.e2e_steps):
                for i, p in enumerate(plans):
                    p.execute_host(hA[i].data_ptr(), hB.data_ptr(), As[i].data_ptr(),
                                   Bs[i].data_ptr(), sptr)
            e1.record(stream)
            torch.cuda.synchronize()
            e2e_ms = e0.elapsed_time(e1)
            if world > 1:
                t = torch.tensor([e2e_ms], device=dev)
                dist.all_reduce(t, op=dist.ReduceOp.MAX)
                e2e_ms = float(t.item())
            h2d = sum(c.n_elems * c.elem_bytes for c in cases)
            e2e = {"value": world * step_bytes * args.e2e_steps / (e2e_ms / 1e3) / 1e9,
                   "unit": "GB/s", "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": h2d,
                   "steps": args.e2e_steps, "api": "ttlg_execute_host (pinned host buffers)",
                   "host_inputs": "one pinned host input per tensor size"}
            del hA, hB, hpool
        except Exception as ex:  # report, do not hide
            e2e = {"value": None, "unit": "GB/s", "error": str(ex)[:200]}

    # L2 label: every case of the TTC / CCSD(T) / small-FVI suites moves more than
    # twice the L2; the small-tensor workloads (config 1, 720-15) do not
    l2_bytes = torch.cuda.get_device_properties(dev).L2_cache_size
    small = [c for c in cases if c.alg_bytes < 2 * l2_bytes]
    l2_label = ("no flush: every case moves > 2x L2 (%d MB) -- inputs larger than L2"
                % (l2_bytes // 2 ** 20)) if not small else (
        "no flush; %d of %d cases move < 2x L2 (%d MB): partly L2-resident; %s"
        % (len(small), len(cases), l2_bytes // 2 ** 20,
           "cases of one size share one A/B pair" if share else
           "every case has its own A/B pair"))
    if rank == 0:
        cpu = None
        if not args.no_cpu_baseline and world == 1:
            cpu = cpu_baseline(cases, budget_s=args.cpu_budget)
        schemas = {}
        for inf in infos:
            schemas[inf["schema"]] = schemas.get(inf["schema"], 0) + 1
        line = {
            "metric": "effective transpose GB/s (2*N*s/time)",
            "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": elapsed_ms / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f64" if cases[0].elem_bytes == 8 else "f32",
            "data": "synthetic (SplitMix64 bit patterns, generated on device)",
            "config": {"workload": name, "cases_per_step": len(cases),
                       "bytes_per_step": step_bytes, "parallelism": f"replica x{world}",
                       "mode": "repeated-use (pre-built plans)" + (
                           "; the step's launches captured once into a CUDA graph and replayed"
                           if graph is not None else "; direct launches"),
                       "timing": "value: K steps between two events (no per-launch events); "
                                 "roofline/kernels: a second pass of K steps, each kernel's "
                                 "launches grouped (as one graph in graph mode) between one "
                                 "event pair per step; cases / model error: a third pass "
                                 "with an event pair per launch"
                                 + ("; cases moving < 32 MB each as a graph of K launches "
                                    "between one event pair" if graph is not None else ""),
                       "l2": l2_label},
            "gpu_launches": launches,
            "roofline": {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak,
                         "peak_source": peak_src, "unit": "GB/s", "frac": achieved / peak,
                         "traffic": traffic, "share_of_step": dg["ms"] / sum(
                             g["ms"] for g in groups.values())},
            "frac_of_peak": value / world / peak,
            "d2d_gbs": d2d_gbs, "frac_of_d2d": value / world / d2d_gbs,
            "kernels": {k: {"gbs": g["bytes"] / (g["ms"] / 1e3) / 1e9,
                            "share": g["ms"] / sum(x["ms"] for x in groups.values()),
                            "launches": g["launches"]} for k, g in groups.items()},
            "schemas": schemas,
            "model_err_pct": 100.0 * sum(errs) / len(errs),
            "tuned": tuned,
            "direct_launch": direct,
            "clocks": clk,
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
        if os.environ.get("TTLG_BENCH_CASES"):
            line["cases"] = [{"case": c.label(), "schema": inf["schema"], "kernel": kname(inf),
                              "gbs": c.alg_bytes / (m * 1e-3) / 1e9,
                              "pred_gbs": c.alg_bytes / inf["predicted_seconds"] / 1e9}
                             for c, inf, m in zip(cases, infos, med)]
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
