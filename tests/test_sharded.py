"""Multi-process CPU tests (gloo, world_size 2 and 4) of the sharded driver's
host logic: slab decomposition, the all-to-all and the fold.  The dense local
transpositions are performed by the ORACLE here (injected as `local_fn`; test
infrastructure), so what is checked is the decomposition, not the kernels.
The gathered B slabs must equal the oracle's global transposition bit for bit.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_ipps_veduradasskhpkn18_b200.sharded import plan_shards, sharded_transpose
from synth import gen_tensor_np

CASES = [
    # (extents, perm): moved and no-move perms, incl. config 5's perms
    ([4, 6, 4, 8], [3, 2, 1, 0]),
    ([4, 6, 4, 8], [0, 3, 2, 1]),
    ([4, 4, 2, 4, 8], [4, 3, 2, 1, 0]),
    ([4, 4, 2, 4, 8], [0, 4, 2, 1, 3]),
    ([4, 4, 2, 4, 8], [2, 0, 1, 4, 3]),
    ([4, 4, 2, 4, 8], [1, 4, 0, 3, 2]),
    ([4, 4, 2, 4, 8], [3, 2, 1, 0, 4]),
    ([4, 4, 2, 4, 8], [1, 0, 3, 2, 4]),
    ([5, 3, 8], [2, 0, 1]),
]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _oracle_local(extents, perm, src, dst):
    a = src.numpy().view(np.uint64)
    dst.copy_(torch.from_numpy(oracle.transpose(a, extents, perm).view(np.float64)))


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        results = []
        for ci, (ext, perm) in enumerate(CASES):
            try:
                sp = plan_shards(ext, perm, world)
            except ValueError:
                results.append(None)
                continue
            n = int(np.prod(ext))
            full = gen_tensor_np(100 + ci, n, 8)
            slab = full[rank * sp.n_local:(rank + 1) * sp.n_local]
            A_local = torch.from_numpy(slab.view(np.float64).copy())
            B_local = sharded_transpose(A_local, ext, perm, local_fn=_oracle_local)
            gathered = [torch.empty_like(B_local) for _ in range(world)]
            dist.all_gather(gathered, B_local)
            if rank == 0:
                got = torch.cat(gathered).numpy().view(np.uint64)
                results.append(bool(np.array_equal(got, oracle.transpose(full, ext, perm))))
        if rank == 0:
            q.put(results)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_sharded_decomposition_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    checked = [r for r in res if r is not None]
    assert len(checked) >= 6
    assert all(checked), res


def test_plan_shards_rules():
    sp = plan_shards([64, 64, 64, 64, 128], [3, 2, 1, 0, 4], 8)
    assert not sp.moved and sp.local_extents[-1] == 16
    sp = plan_shards([64, 64, 64, 64, 128], [4, 3, 2, 1, 0], 8)
    assert sp.moved and sp.fold_extents == [16, 64 * 64 * 64 * 8, 8]
    with pytest.raises(ValueError):
        plan_shards([4, 4, 4, 2, 8], [2, 0, 1, 4, 3], 4)  # P=4 does not divide n_q = n_3 = 2


# ---- the same over the CUDA kernels: two processes sharing cuda:0 (gloo) -----------------
GPU_CASES = [
    ([8, 6, 4, 8], [3, 2, 1, 0]),
    ([8, 6, 4, 8], [0, 3, 2, 1]),
    ([16, 8, 8, 16, 32], [4, 3, 2, 1, 0]),
    ([16, 8, 8, 16, 32], [0, 4, 2, 1, 3]),
    ([16, 8, 8, 16, 32], [2, 0, 1, 4, 3]),
    ([16, 8, 8, 16, 32], [3, 2, 1, 0, 4]),
    ([16, 8, 8, 16, 32], [1, 0, 3, 2, 4]),
]


def _cases_for(world):
    """GPU_CASES whose sharded extents P divides (plan_shards' precondition)."""
    out = []
    for ci, (ext, perm) in enumerate(GPU_CASES):
        try:
            plan_shards(ext, perm, world)
        except ValueError:
            continue
        out.append((ci, (ext, perm)))
    return out


def _gpu_worker(rank, world, port, q, backend="gloo", own_device=False):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dev = rank if own_device else 0
    torch.cuda.set_device(dev)
    if backend == "nccl":
        dist.init_process_group("nccl", rank=rank, world_size=world,
                                device_id=torch.device("cuda", dev))
    else:
        dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_veduradasskhpkn18_b200.sharded import P2PExchange
    try:
        results = []
        for ci, (ext, perm) in _cases_for(world):
            sp = plan_shards(ext, perm, world)
            n = int(np.prod(ext))
            full = gen_tensor_np(300 + ci, n, 8)
            slab = full[rank * sp.n_local:(rank + 1) * sp.n_local]
            A_local = torch.from_numpy(slab.view(np.float64).copy()).cuda()
            expect = oracle.transpose(full, ext, perm) if rank == 0 else None
            # (1) local transpose -> all_to_all_single (gloo, CUDA tensors) -> fold
            B1 = sharded_transpose(A_local, ext, perm)
            torch.cuda.synchronize()
            # (2) fused exchange: sub-transpositions store into the peer's slab via CUDA IPC
            B2 = torch.empty_like(A_local)
            ex = P2PExchange(ext, perm, B2)
            torch.cuda.synchronize()
            dist.barrier()
            ex.run(A_local, torch.cuda.current_stream().cuda_stream)
            torch.cuda.synchronize()
            dist.barrier()
            for B in (B1, B2):
                if backend == "nccl":
                    gathered = [torch.empty_like(B) for _ in range(world)]
                    dist.all_gather(gathered, B)
                    gathered = [g.cpu() for g in gathered]
                else:
                    gathered = [torch.empty(sp.n_local, dtype=torch.float64) for _ in range(world)]
                    dist.all_gather(gathered, B.cpu())
                if rank == 0:
                    got = torch.cat(gathered).numpy().view(np.uint64)
                    results.append(bool(np.array_equal(got, expect)))
            dist.barrier()
            ex.close()
        if rank == 0:
            q.put(results)
    except Exception as e:  # surface the error in the parent
        if rank == 0:
            q.put(repr(e))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
def test_sharded_gpu_two_processes_one_device():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gpu_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
    assert isinstance(res, list), res
    assert len(res) == 2 * len(_cases_for(2)) and all(res), res


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 4, 8])
def test_sharded_nccl_one_process_per_gpu(world):
    """The multi-GPU path as bench.py runs it: one process per device, NCCL
    all_to_all_single for the all-to-all exchange and CUDA IPC peer mappings
    across devices (NVLink stores) for the fused exchange, both bit-exact
    against the global oracle.  Needs `world` visible devices (skips otherwise:
    every gpurun box of this build has one)."""
    if torch.cuda.device_count() < world:
        pytest.skip(f"needs {world} CUDA devices, {torch.cuda.device_count()} visible")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gpu_worker, args=(r, world, port, q, "nccl", True))
             for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=900)
    for p in procs:
        p.join(timeout=120)
    assert isinstance(res, list), res
    assert len(res) == 2 * len(_cases_for(world)) and all(res), res
