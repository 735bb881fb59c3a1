"""Sharded transposition across GPUs (one process per GPU, torch.distributed).

Not in the paper (single K40c, Table III); required by
BASELINE.json's north star and config 5.  A is distributed along its
outermost input dim d-1 (rank p holds i_{d-1} in [p*c, (p+1)*c), c = n_{d-1}/P,
a contiguous slab of A); B is returned distributed along its outermost output
dim o_{d-1} = input dim q = perm[d-1] (also a contiguous slab of B).

* q == d-1 ("no move"): every rank transposes its own slab with the same
  permutation -- zero communication, near-linear weak scaling.
* q != d-1 ("moved"): one exchange step, the only collective of the library:
    1. local transpose of the slab (extent c on dim d-1).  Its outermost
       output dim is o_{d-1} = q, so its P sub-ranges of i_q are contiguous
       chunks -> the local output IS the all-to-all send buffer;
    2. all_to_all_single with equal splits (NCCL over NVLink/NVSwitch);
    3. fold: the P received chunks, source rank outermost, are the FVI-first
       tensor [X, Y, P] with X = prod of the local output extents up to and
       including o_k (k = position of d-1 in perm, extent c), Y = the rest;
       the B slab is [X, P, Y], i.e. the transposition (0 2 1) of it
       (matching FVI -> FML/FMS kernels).
  Requires P | n_{d-1} and P | n_q (else ValueError: run replicas instead).

`local_fn(extents, perm, src, dst)` performs one dense transposition; the
default is the CUDA library (ttlg_transpose on the current stream).  CPU unit
tests inject the oracle there to check the decomposition over gloo.

Fused exchange (`P2PExchange`): instead of local transpose ->
all-to-all -> fold (three HBM passes plus NCCL staging), rank p runs P
sub-tensor transpositions (ttlg_plan_strided), one per destination q: the
input is the sub-box i_q in [q*cq, (q+1)*cq) of its A slab, the output is the
box o_k in [p*c, (p+1)*c) of rank q's B slab, written straight into q's
memory through a CUDA IPC mapping (NVLink/NVSwitch stores).  One HBM read of A
and one (remote) write of B per element; no send/receive buffers, no fold.
`p2p_subproblems` is the pure index arithmetic (tested on the CPU and, with
every "peer" slab on one device, against the oracle on the GPU).
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Callable, List, Optional, Sequence


@dataclass
class ShardPlan:
    world: int
    extents: List[int]        # global input extents (FVI first)
    perm: List[int]
    moved: bool               # True: needs the all-to-all
    local_extents: List[int]  # this rank's A slab
    out_local_extents: List[int]  # this rank's B slab (output order)
    fold_extents: Optional[List[int]]  # [X, Y, P] for the fold (moved only)
    n_local: int              # elements per rank


def plan_shards(extents: Sequence[int], perm: Sequence[int], world: int) -> ShardPlan:
    ext = [int(e) for e in extents]
    perm = [int(p) for p in perm]
    d = len(ext)
    if sorted(perm) != list(range(d)):
        raise ValueError("perm must be a permutation")
    if ext[d - 1] % world:
        raise ValueError(f"P={world} must divide the sharded input extent {ext[d - 1]}")
    c = ext[d - 1] // world
    local = ext[:-1] + [c]
    n_local = 1
    for e in local:
        n_local *= e
    q = perm[d - 1]
    out_global = [ext[p] for p in perm]
    if q == d - 1:
        out_local = out_global[:-1] + [c]
        return ShardPlan(world, ext, perm, False, local, out_local, None, n_local)
    if ext[q] % world:
        raise ValueError(f"P={world} must divide the output-sharded extent {ext[q]}")
    cq = ext[q] // world
    k = perm.index(d - 1)
    # local output extents (output order) of the slab transpose
    lo = [local[p] for p in perm]
    X = 1
    for i in range(k + 1):
        X *= lo[i]
    Y = 1
    for i in range(k + 1, d - 1):
        Y *= lo[i]
    Y *= cq
    out_local = out_global[:-1] + [cq]
    return ShardPlan(world, ext, perm, True, local, out_local, [X, Y, world], n_local)


def _default_local_fn(extents, perm, src, dst):
    import torch
    from .api import transpose, _dt_of_tensor
    transpose(_dt_of_tensor(src), extents, perm, src.data_ptr(), dst.data_ptr(),
              torch.cuda.current_stream(src.device).cuda_stream)


def sharded_transpose(A_local, extents: Sequence[int], perm: Sequence[int], group=None,
                      local_fn: Optional[Callable] = None, work=None, phase_events=None):
    """Transpose a tensor sharded along its outermost input dim; returns this
    rank's slab of B (flat, output-order layout of `out_local_extents`).
    `work`: optional preallocated (send, recv) flat buffers of n_local elements.
    `phase_events`: optional list that receives (name, start, end) CUDA events."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    sp = plan_shards(extents, perm, world)
    fn = local_fn or _default_local_fn
    if A_local.numel() != sp.n_local:
        raise ValueError(f"local slab has {A_local.numel()} elements, expected {sp.n_local}")

    def ev():
        if phase_events is None or not A_local.is_cuda:
            return None
        e = torch.cuda.Event(enable_timing=True)
        e.record()
        return e

    if not sp.moved:
        out = work[1] if work is not None else torch.empty_like(A_local)
        e0 = ev()
        fn(sp.local_extents, sp.perm, A_local, out)
        if phase_events is not None and e0 is not None:
            phase_events.append(("local", e0, ev()))
        return out
    send = work[0] if work is not None else torch.empty_like(A_local)
    recv = work[1] if work is not None else torch.empty_like(A_local)
    e0 = ev()
    fn(sp.local_extents, sp.perm, A_local, send)
    e1 = ev()
    dist.all_to_all_single(recv, send, group=group)
    e2 = ev()
    out = send  # the send buffer is free again: fold into it
    fn(sp.fold_extents, [0, 2, 1], recv, out)
    if phase_events is not None and e0 is not None:
        phase_events += [("local", e0, e1), ("alltoall", e1, e2), ("fold", e2, ev())]
    return out


# ---- fused transpose + exchange over peer memory ------------------
@dataclass
class SubProblem:
    dest: int                 # destination rank q
    extents: List[int]        # sub-box of the local A slab (input order)
    in_strides: List[int]     # strides of the local A slab (elements)
    out_strides: List[int]    # strides of rank q's B slab, output order (elements)
    a_offset: int             # element offset of the sub-box in the local A slab
    b_offset: int             # element offset of this rank's box in q's B slab


def _dense_strides(ext):
    s, acc = [], 1
    for e in ext:
        s.append(acc)
        acc *= e
    return s


def p2p_subproblems(sp: ShardPlan, rank: int) -> List[SubProblem]:
    """The P sub-tensor transpositions rank `rank` runs in the fused exchange.
    No-move plans: one dense local transposition into its own slab."""
    d = len(sp.extents)
    sA = _dense_strides(sp.local_extents)
    if not sp.moved:
        out_s = _dense_strides(sp.out_local_extents)
        return [SubProblem(rank, list(sp.local_extents), sA, out_s, 0, 0)]
    j = sp.perm[d - 1]                      # A dim that becomes B's sharded outermost dim
    cq = sp.extents[j] // sp.world
    k = sp.perm.index(d - 1)                # output position of A's sharded dim
    c = sp.local_extents[d - 1]
    sB = _dense_strides(sp.out_local_extents)   # every B slab has the same layout
    subs = []
    for q in range(sp.world):
        ext = list(sp.local_extents)
        ext[j] = cq
        subs.append(SubProblem(q, ext, sA, sB, q * cq * sA[j], rank * c * sB[k]))
    return subs


def map_peer_slabs(out, group=None):
    """Exchange CUDA IPC handles of every rank's `out` over the process group
    and map the peers' buffers on this device.  Returns (pointers by rank,
    [(pointer, offset)] to pass to unmap_peer_slabs)."""
    import torch.distributed as dist
    from . import api
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    h, off = api.ipc_export(out.data_ptr())
    allh = [None] * world
    dist.all_gather_object(allh, (h, off), group=group)
    ptrs, opened = [], []
    for q, (hq, oq) in enumerate(allh):
        if q == rank:
            ptrs.append(out.data_ptr())
        else:
            ptr = api.ipc_open(hq, oq)
            opened.append((ptr, oq))
            ptrs.append(ptr)
    return ptrs, opened


def unmap_peer_slabs(opened):
    from . import api
    for ptr, off in opened:
        api.ipc_close(ptr, off)


class P2PExchange:
    """Rank-local driver of the fused exchange: maps every peer's B slab
    (CUDA IPC through the process group), plans the sub-transpositions once
    (repeated use), and launches them on one stream.

    `out` is this rank's B slab (a CUDA tensor of n_local elements); it must
    stay allocated while the exchange object lives.  `run()` must be bracketed
    by a barrier (peers may still read their previous B) and followed by a
    stream synchronise + barrier before B is read (incoming remote stores)."""

    def __init__(self, extents: Sequence[int], perm: Sequence[int], out, group=None,
                 dtype=None, peer_ptrs: Optional[List[int]] = None, rank: Optional[int] = None,
                 world: Optional[int] = None):
        from . import api
        self.group = group
        if world is None or rank is None:
            import torch.distributed as dist
            world = dist.get_world_size(group)
            rank = dist.get_rank(group)
        self.rank, self.world = rank, world
        self.sp = plan_shards(extents, perm, world)
        self.esize = out.element_size()
        dt = dtype if dtype is not None else api._dt_of_tensor(out)
        self._opened = []
        self.subs = p2p_subproblems(self.sp, rank)
        # plan first (no CUDA state yet): an unsupported sub-box raises before
        # any peer mapping exists.  Every destination's sub-box has the same
        # extents and strides (only the A offset and the target slab differ),
        # so ONE plan serves all of them and run() issues ONE batched launch
        # (ttlg_execute_batch: grid.y = destinations).
        s0 = self.subs[0]
        assert all(s.extents == s0.extents and s.in_strides == s0.in_strides and
                   s.out_strides == s0.out_strides for s in self.subs)
        self.plan = api.plan_strided(dt, s0.extents, self.sp.perm, s0.in_strides,
                                     s0.out_strides)
        self.plans = [self.plan] * len(self.subs)
        if peer_ptrs is None:
            peer_ptrs = self._map_peers(out)
        self.peers = peer_ptrs

    def _map_peers(self, out):
        ptrs, self._opened = map_peer_slabs(out, self.group)
        return ptrs

    def predicted_seconds(self) -> float:
        return len(self.subs) * self.plan.describe()["predicted_seconds"]

    def run(self, A_local, stream: int):
        """All P sub-transpositions as one kernel launch (grid.y = P)."""
        a0 = A_local.data_ptr()
        self.plan.execute_batch([a0 + s.a_offset * self.esize for s in self.subs],
                                [self.peers[s.dest] + s.b_offset * self.esize
                                 for s in self.subs], stream)

    def close(self):
        unmap_peer_slabs(self._opened)
        self._opened = []


# ---- choosing the exchange (model-driven, like the paper's schema choice) -----------
NVLINK_GBS = 770.0  # measured peer copy per direction per GPU (B200_PROFILING.md)


def _dtype_bytes(dtype) -> int:
    return 8 if str(dtype) in ("f64", "float64", "torch.float64", "fp64", "1") else 4


def choose_exchange(extents: Sequence[int], perm: Sequence[int], world: int, dtype="f32",
                    nvlink_gbs: float = NVLINK_GBS) -> dict:
    """Predicted per-rank seconds of the two exchange paths and the choice.

    p2p     : max(sum of the sub-transpositions' model predictions,
                  remote bytes / NVLink)  (the stores overlap the kernels);
    alltoall: local transposition + (P-1)/P of the slab over NVLink + fold.
    Either prediction is None when the path does not apply (a sub-box whose
    FVI collapses to a non-unit stride, cq = 1 on A's FVI, has no p2p plan)."""
    from . import api
    sp = plan_shards(extents, perm, world)
    s = _dtype_bytes(dtype)
    slab = sp.n_local * s
    if not sp.moved:
        t = api.predict_time(dtype, sp.local_extents, sp.perm)
        return {"mode": "local", "p2p": t, "alltoall": t}
    remote = slab * (world - 1) / world / (nvlink_gbs * 1e9)
    try:
        t_sub = sum(api.plan_strided(dtype, q.extents, sp.perm, q.in_strides, q.out_strides)
                    .describe()["predicted_seconds"] for q in p2p_subproblems(sp, 0))
        t_p2p = max(t_sub, remote)
    except api.TtlgError:
        t_p2p = None
    t_a2a = (api.predict_time(dtype, sp.local_extents, sp.perm) + remote +
             api.predict_time(dtype, sp.fold_extents, [0, 2, 1]))
    mode = "p2p" if t_p2p is not None and t_p2p <= t_a2a else "alltoall"
    return {"mode": mode, "p2p": t_p2p, "alltoall": t_a2a}
