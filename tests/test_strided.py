"""Sub-tensor transpositions (ttlg_plan_strided) and the fused sharded
exchange built on them (sharded.P2PExchange).

CPU (-m "not gpu"):
- the strided oracle (oracle.transpose_strided) pinned to NumPy's transpose of
  as_strided views (an independent mechanism) and to the dense oracle;
- planner rules of the strided form: dense strides plan exactly like the dense
  call, fusion stops at gaps, unsupported / invalid strides are rejected;
- the fused-exchange index arithmetic (p2p_subproblems): every rank's
  sub-transpositions, run by the strided oracle into per-rank B slabs, must
  reassemble the oracle's global transposition bit for bit.
GPU (-m gpu): the CUDA path through the C ABI against the strided oracle,
whole buffers (canary bands included), and the fused exchange with every
"peer" slab on one device.
"""
import itertools

import numpy as np
import pytest

import oracle
import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
from paper_conf_ipps_veduradasskhpkn18_b200.sharded import plan_shards, p2p_subproblems
from synth import gen_tensor_np


def _dense(ext):
    s, acc = [], 1
    for e in ext:
        s.append(acc)
        acc *= e
    return s


def _span(ext, strides):
    return 1 + sum((e - 1) * s for e, s in zip(ext, strides))


def _numpy_strided(A, B, ext, perm, sa, sb, a_off, b_off):
    """Independent definition through NumPy views (row-major axes reversed)."""
    d = len(ext)
    it = A.dtype.itemsize
    Av = np.lib.stride_tricks.as_strided(A[a_off:], shape=ext[::-1],
                                         strides=[s * it for s in sa[::-1]])
    axes = [d - 1 - perm[d - 1 - a] for a in range(d)]
    m = [ext[p] for p in perm]
    Bv = np.lib.stride_tricks.as_strided(B[b_off:], shape=m[::-1],
                                         strides=[s * it for s in sb[::-1]], writeable=True)
    Bv[...] = np.transpose(Av, axes)
    return B


STRIDED_CASES = [
    # (extents, perm, in_strides or None, out_strides or None)
    ([37, 20, 9], [2, 0, 1], [1, 40, 40 * 23], None),
    ([37, 20, 9], [2, 0, 1], None, [1, 11, 11 * 40]),
    ([16, 12, 10, 6], [3, 1, 0, 2], [1, 19, 19 * 13, 19 * 13 * 11], [1, 7, 7 * 13, 7 * 13 * 20]),
    ([4, 33, 17], [0, 2, 1], [1, 8, 8 * 35], [1, 4, 4 * 18]),       # matching FVI, widenable
    ([4, 33, 17], [0, 2, 1], [1, 5, 5 * 34], [1, 6, 6 * 17]),       # matching FVI, odd strides
    ([8, 6, 5, 7, 2], [1, 4, 0, 3, 2], [1, 9, 9 * 6, 9 * 6 * 5, 9 * 6 * 5 * 8], None),
    ([64, 3, 40], [0, 1, 2], [1, 70, 70 * 4], [1, 64, 64 * 3 * 2]),  # identity with gaps
    # closed 16 x 16 leading block (k_blk) inside padded outer strides
    ([16, 16, 5, 6], [1, 0, 3, 2], [1, 16, 16 * 16 * 2, 16 * 16 * 2 * 7], [1, 16, 16 * 16 * 8,
                                                                         16 * 16 * 8 * 6]),
]


@pytest.mark.parametrize("eb", [4, 8])
@pytest.mark.parametrize("case", STRIDED_CASES, ids=lambda c: "x".join(map(str, c[0])) + "-" +
                         "".join(map(str, c[1])))
def test_oracle_strided_pins(case, eb):
    ext, perm, sa, sb = case
    sa = sa or _dense(ext)
    sb = sb or _dense([ext[p] for p in perm])
    ut = np.uint64 if eb == 8 else np.uint32
    A = gen_tensor_np(7, _span(ext, sa) + 5, eb).view(ut)
    nb = _span([ext[p] for p in perm], sb) + 9
    B0 = gen_tensor_np(8, nb, eb).view(ut)
    got = oracle.transpose_strided(A, B0.copy(), ext, perm, sa, sb, a_off=3, b_off=4)
    exp = _numpy_strided(A, B0.copy(), ext, perm, sa, sb, 3, 4)
    assert np.array_equal(got, exp)


def test_oracle_strided_dense_is_transpose():
    rng = np.random.default_rng(3)
    for _ in range(40):
        d = int(rng.integers(1, 6))
        ext = [int(x) for x in rng.integers(1, 6, size=d)]
        perm = [int(x) for x in rng.permutation(d)]
        A = gen_tensor_np(11, int(np.prod(ext)), 8)
        B = np.zeros_like(A)
        oracle.transpose_strided(A, B, ext, perm, _dense(ext), _dense([ext[p] for p in perm]))
        assert np.array_equal(B, oracle.transpose(A, ext, perm))


# ---- planner rules (no device needed: virtual B200 profile) ----------------------------------
def test_dense_strides_plan_like_dense():
    for ext, perm in [([64, 64, 64, 64], [3, 2, 1, 0]), ([320, 320, 256], [0, 2, 1]),
                      ([27, 27, 27, 27, 27], [4, 1, 2, 0, 3]), ([2, 4096, 4096], [0, 2, 1])]:
        a = ttlg.plan("f64", ext, perm).describe()
        b = ttlg.plan_strided("f64", ext, perm, _dense(ext),
                              _dense([ext[p] for p in perm])).describe()
        for k in ("schema", "kernel", "fused_extents", "fused_perm", "tile_extents", "threads",
                  "access_bytes"):
            assert a[k] == b[k], (ext, perm, k)


def test_fusion_stops_at_gaps():
    # identity: dense fuses to rank 1; a gap after dim 1 of A keeps two dims
    d = ttlg.plan_strided("f32", [16, 16, 16], [0, 1, 2], [1, 16, 300], None).describe()
    assert d["fused_rank"] == 2
    # fusable pair (1, 2) of [i0,i1,i2,i3] -> [i3,i1,i2,i0] unless B has a gap
    dense = ttlg.plan("f64", [8, 9, 10, 11], [3, 1, 2, 0]).describe()
    assert dense["fused_rank"] == 3
    gap = ttlg.plan_strided("f64", [8, 9, 10, 11], [3, 1, 2, 0], None,
                            [1, 11, 11 * 9 + 1, 11 * 9 * 11]).describe()
    assert gap["fused_rank"] == 4


def test_choose_exchange_rules():
    from paper_conf_ipps_veduradasskhpkn18_b200.sharded import choose_exchange
    ext = [64, 64, 64, 64, 128]
    assert choose_exchange(ext, [3, 2, 1, 0, 4], 8)["mode"] == "local"
    r = choose_exchange(ext, [0, 4, 2, 1, 3], 8)
    assert r["mode"] == "p2p" and r["p2p"] < r["alltoall"]
    # 32-byte sub-box runs on A's FVI at P = 8: the model prefers the all-to-all
    assert choose_exchange(ext, [4, 3, 2, 1, 0], 8)["mode"] == "alltoall"
    # cq = 1 on A's FVI: no p2p plan at all
    r = choose_exchange([4, 6, 4, 8], [3, 2, 1, 0], 4)
    assert r["p2p"] is None and r["mode"] == "alltoall"


def test_strided_rejections():
    with pytest.raises(ttlg.TtlgError) as e:   # A's FVI not unit-stride
        ttlg.plan_strided("f32", [8, 8], [1, 0], [2, 16], None)
    assert e.value.code == 7
    with pytest.raises(ttlg.TtlgError) as e:   # B's first dim not unit-stride
        ttlg.plan_strided("f32", [8, 8], [1, 0], None, [2, 16])
    assert e.value.code == 7
    with pytest.raises(ttlg.TtlgError) as e:   # B not injective
        ttlg.plan_strided("f32", [8, 8], [1, 0], None, [1, 4])
    assert e.value.code == 1
    with pytest.raises(ttlg.TtlgError) as e:   # zero stride on a non-unit dim
        ttlg.plan_strided("f32", [8, 8], [1, 0], [1, 0], None)
    assert e.value.code == 1
    # extent-1 dims ignore their strides
    ttlg.plan_strided("f32", [8, 1, 8], [2, 1, 0], [1, 0, 8], [1, 0, 8])


# ---- fused exchange: index arithmetic on the CPU (strided oracle as the local step) ---------
P2P_CASES = [
    ([4, 6, 4, 8], [3, 2, 1, 0]),
    ([4, 6, 4, 8], [0, 3, 2, 1]),
    ([4, 4, 2, 4, 8], [4, 3, 2, 1, 0]),
    ([4, 4, 2, 4, 8], [0, 4, 2, 1, 3]),
    ([4, 4, 2, 4, 8], [2, 0, 1, 4, 3]),
    ([4, 4, 2, 4, 8], [1, 4, 0, 3, 2]),
    ([4, 4, 2, 4, 8], [3, 2, 1, 0, 4]),
    ([5, 3, 8], [2, 0, 1]),
]


@pytest.mark.parametrize("world", [1, 2, 4])
@pytest.mark.parametrize("case", P2P_CASES, ids=lambda c: "".join(map(str, c[1])))
def test_p2p_subproblems_reassemble(case, world):
    ext, perm = case
    try:
        sp = plan_shards(ext, perm, world)
    except ValueError:
        pytest.skip("P does not divide the sharded extents")
    n = int(np.prod(ext))
    A = gen_tensor_np(21, n, 8)
    slabs_B = [np.zeros(sp.n_local, dtype=np.uint64) for _ in range(world)]
    written = [np.zeros(sp.n_local, dtype=np.int64) for _ in range(world)]
    for p in range(world):
        A_p = A[p * sp.n_local:(p + 1) * sp.n_local]
        for s in p2p_subproblems(sp, p):
            oracle.transpose_strided(A_p, slabs_B[s.dest], s.extents, perm, s.in_strides,
                                     s.out_strides, s.a_offset, s.b_offset)
            # every position written exactly once over all ranks
            cnt = np.zeros(sp.n_local, dtype=np.uint64)
            ones = np.ones(A_p.size, dtype=np.uint64)
            oracle.transpose_strided(ones, cnt, s.extents, perm, s.in_strides, s.out_strides,
                                     s.a_offset, s.b_offset)
            written[s.dest] += cnt.astype(np.int64)
    assert all((w == 1).all() for w in written)
    assert np.array_equal(np.concatenate(slabs_B), oracle.transpose(A, ext, perm))


# ---- GPU parity ------------------------------------------------------------------------------
def _torch_bits(t):
    import torch
    return t.view(torch.int64 if t.element_size() == 8 else torch.int32).cpu().numpy().view(
        np.uint64 if t.element_size() == 8 else np.uint32)


@pytest.mark.gpu
@pytest.mark.parametrize("variant", [None, 1, 2, 3, 9])
@pytest.mark.parametrize("eb", [4, 8])
@pytest.mark.parametrize("case", STRIDED_CASES, ids=lambda c: "x".join(map(str, c[0])) + "-" +
                         "".join(map(str, c[1])))
def test_gpu_strided_parity(case, eb, variant):
    import torch
    from synth import gen_tensor_torch
    ext, perm, sa, sb = case
    sa = sa or _dense(ext)
    sb = sb or _dense([ext[p] for p in perm])
    dt = "f64" if eb == 8 else "f32"
    kw = {} if variant is None else {"variant": variant}
    try:
        p = ttlg.plan_strided(dt, ext, perm, sa, sb, **kw)
    except ttlg.TtlgError as e:
        if variant is not None and e.code == 7:
            pytest.skip("variant does not apply")
        raise
    a_off, b_off = 4, 8          # element offsets keep 16-byte alignment for eb = 4, 8
    A = gen_tensor_torch(31, _span(ext, sa) + a_off + 7, eb, device="cuda:0")
    nb = _span([ext[q] for q in perm], sb) + b_off + 11
    B = gen_tensor_torch(32, nb, eb, device="cuda:0")   # background = canary everywhere
    A_h, B_h = _torch_bits(A), _torch_bits(B)
    p.execute(A.data_ptr() + a_off * eb, B.data_ptr() + b_off * eb,
              torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    exp = oracle.transpose_strided(A_h, B_h.copy(), ext, perm, sa, sb, a_off, b_off)
    got = _torch_bits(B)
    assert np.array_equal(got, exp), p.describe()
    assert np.array_equal(_torch_bits(A), A_h)


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 4, 8])
@pytest.mark.parametrize("case", P2P_CASES + [([16, 8, 8, 16, 32], [4, 3, 2, 1, 0]),
                                              ([16, 8, 8, 16, 32], [0, 4, 2, 1, 3]),
                                              ([16, 8, 8, 16, 32], [2, 0, 1, 4, 3])],
                         ids=lambda c: "x".join(map(str, c[0])) + "-" + "".join(map(str, c[1])))
def test_gpu_p2p_exchange_virtual_peers(case, world):
    """The fused exchange with every peer's B slab on cuda:0: the same
    sub-transposition launches as P2PExchange.run, peer pointers local."""
    import torch
    from synth import gen_tensor_torch
    from paper_conf_ipps_veduradasskhpkn18_b200.sharded import P2PExchange
    ext, perm = case
    try:
        sp = plan_shards(ext, perm, world)
    except ValueError:
        pytest.skip("P does not divide the sharded extents")
    from paper_conf_ipps_veduradasskhpkn18_b200.sharded import choose_exchange
    if choose_exchange(ext, perm, world)["p2p"] is None:
        # cq = 1 on A's FVI: no unit-stride run left; the all-to-all path serves it
        assert choose_exchange(ext, perm, world)["mode"] == "alltoall"
        pytest.skip("no p2p plan (sub-box FVI collapses)")
    n = int(np.prod(ext))
    for eb in (4, 8):
        A = gen_tensor_torch(41, n, eb, device="cuda:0")
        B = torch.empty_like(A)
        slabs = [B[q * sp.n_local:(q + 1) * sp.n_local] for q in range(world)]
        ptrs = [s.data_ptr() for s in slabs]
        stream = torch.cuda.current_stream().cuda_stream
        for p in range(world):
            ex = P2PExchange(ext, perm, slabs[p], peer_ptrs=ptrs, rank=p, world=world)
            ex.run(A[p * sp.n_local:(p + 1) * sp.n_local], stream)
        torch.cuda.synchronize()
        assert np.array_equal(_torch_bits(B), oracle.transpose(_torch_bits(A), ext, perm))


@pytest.mark.gpu
def test_gpu_transpose_tensor_strided_views():
    """transpose_tensor on strided views (slices of larger tensors) in and out,
    through ttlg_plan_strided: equals torch's permute, bit for bit."""
    import torch
    from synth import gen_tensor_torch
    base = gen_tensor_torch(51, 40 * 30 * 24, 8, device="cuda:0").view(40, 30, 24)
    x = base[3:35, 2:27, 4:20]                       # non-contiguous, innermost unit-stride
    for perm in ([2, 1, 0], [1, 0, 2], [0, 2, 1], [2, 0, 1]):
        y = ttlg.transpose_tensor(x, perm)
        ref = x.permute(*perm).contiguous()
        assert torch.equal(y.view(torch.int64), ref.view(torch.int64)), perm
        big = torch.zeros([s + 3 for s in ref.shape], dtype=x.dtype, device="cuda:0")
        view = big[1:1 + ref.shape[0], 2:2 + ref.shape[1], :ref.shape[2]]
        ttlg.transpose_tensor(x, perm, out=view)
        assert torch.equal(view.contiguous().view(torch.int64), ref.view(torch.int64)), perm
        assert int(torch.count_nonzero(big.view(torch.int64))) == \
            int(torch.count_nonzero(ref.view(torch.int64)))   # nothing written outside the view
    with pytest.raises(ttlg.TtlgError):
        ttlg.transpose_tensor(base[:, :, ::2], [2, 1, 0])   # innermost dim not unit-stride
