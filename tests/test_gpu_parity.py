"""GPU parity: the CUDA path (through the C ABI) against the oracle, bit for bit
(tolerance 0: a transposition does no arithmetic, reading R3).

- oracle-sized cases: every config, element by element, at sizes spanning
  several tiles with ragged tails, under the auto plan AND every applicable
  forced schema;
- full BASELINE sizes in the launch configuration bench.py times: sampled
  outputs checked one by one through oracle.source_index (lin_B -> lin_A),
  plus the exactly-once/index-encoding property on whole tensors;
- edge cases: rank 1, rank 15, extent-1 dims, odd extents, misaligned pointers
  (narrow-access fallback), canary bands around B, A unchanged, single-use
  path, non-default streams.
"""
import itertools
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle  # noqa: E402  (test infrastructure)
import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg  # noqa: E402
from synth import configs, gen_tensor_torch, gen_at_np, case_seed  # noqa: E402

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


def _bits(t):
    t = t.contiguous()
    if t.element_size() == 8:
        return t.view(torch.int64).cpu().numpy().view(np.uint64)
    return t.view(torch.int32).cpu().numpy().view(np.uint32)


def _dt(eb):
    return "f64" if eb == 8 else "f32"


def _run(ext, perm, eb, seed, plan_kwargs=None, single_use=False, canary=0):
    n = int(np.prod(ext))
    A = gen_tensor_torch(seed, n, eb, device=DEV)
    Bfull = torch.empty(n + 2 * canary, dtype=A.dtype, device=DEV)
    if canary:
        Bfull.view(torch.int64 if eb == 8 else torch.int32).fill_(0x5A5A5A5A)
    B = Bfull[canary:canary + n]
    stream = torch.cuda.current_stream().cuda_stream
    if single_use:
        ttlg.transpose(_dt(eb), ext, perm, A.data_ptr(), B.data_ptr(), stream)
        info = None
    else:
        p = ttlg.plan(_dt(eb), ext, perm, **(plan_kwargs or {}))
        info = p.describe()
        p.execute(A.data_ptr(), B.data_ptr(), stream)
    torch.cuda.synchronize()
    A_host = _bits(A)
    expect = oracle.transpose(A_host, ext, perm)
    got = _bits(B)
    if canary:
        band = _bits(Bfull)
        assert (band[:canary] == band[0]).all() and (band[-canary:] == band[0]).all(), \
            "write outside B"
    # A must be untouched
    assert np.array_equal(_bits(A), A_host)
    return got, expect, info


def _assert_equal(got, expect, what):
    if not np.array_equal(got, expect):
        bad = np.nonzero(got != expect)[0]
        pytest.fail(f"{what}: {bad.size} mismatches, first at {bad[:8].tolist()}")


# ---- config 1: all 24 perms of 16^4 fp64, auto + every applicable forced schema ------------
@pytest.mark.parametrize("case", configs.config1(), ids=lambda c: "".join(map(str, c.perm)))
def test_config1_all_schemas(case):
    got, exp, info = _run(case.extents, case.perm, 8, case_seed(case.case_id), canary=64)
    _assert_equal(got, exp, f"auto {info['schema']}")
    for s in ("OD", "OA", "FMS", "FML"):
        try:
            ttlg.plan("f64", case.extents, case.perm, schema=s)
        except ttlg.TtlgError:
            continue
        got, exp, info = _run(case.extents, case.perm, 8, case_seed(case.case_id),
                              plan_kwargs={"schema": s}, canary=64)
        _assert_equal(got, exp, f"forced {s}")


def _scaled_cases():
    out = []
    for grp in ("c2", "c3", "c4", "c5"):
        for c in configs.all_configs()[grp]:
            out.append(configs.scaled(c, 1 << 20))
    return out


@pytest.mark.parametrize("case", _scaled_cases(), ids=lambda c: c.label())
def test_scaled_configs_auto(case):
    got, exp, info = _run(case.extents, case.perm, case.elem_bytes, case_seed(case.case_id),
                          canary=32)
    _assert_equal(got, exp, f"auto {info['schema']} {info}")


@pytest.mark.parametrize("case", _scaled_cases()[::3], ids=lambda c: c.label())
def test_scaled_configs_forced(case):
    for s in ("OD", "OA", "FMS", "FML"):
        try:
            ttlg.plan(_dt(case.elem_bytes), case.extents, case.perm, schema=s)
        except ttlg.TtlgError:
            continue
        got, exp, info = _run(case.extents, case.perm, case.elem_bytes,
                              case_seed(case.case_id), plan_kwargs={"schema": s})
        _assert_equal(got, exp, f"forced {s} {info}")


# ---- ragged / odd extents, every rank-4 and a sample of rank-5/6 perms -----------------------
@pytest.mark.parametrize("eb", [4, 8])
@pytest.mark.parametrize("ext", [(15, 17, 13, 19), (3, 33, 65, 7), (5, 2, 129, 31),
                                 (27, 27, 27, 27), (1, 40, 1, 33)])
def test_odd_extents_rank4(ext, eb):
    for k, perm in enumerate(itertools.permutations(range(4))):
        got, exp, info = _run(list(ext), list(perm), eb, 1000 + k)
        _assert_equal(got, exp, f"{ext} {perm} {info['schema']}")


@pytest.mark.parametrize("eb", [4, 8])
def test_rank6_sample(eb):
    rng = np.random.default_rng(6)
    perms = list(itertools.permutations(range(6)))
    for k in rng.choice(len(perms), 40, replace=False):
        ext = [int(x) for x in rng.integers(2, 12, size=6)]
        got, exp, info = _run(ext, list(perms[k]), eb, 2000 + int(k))
        _assert_equal(got, exp, f"{ext} {perms[k]} {info['schema']}")


def test_block_sweep_fig5():
    """Every slice variant of the Fig. 5 sweep gives identical bytes (L1421-1436)."""
    ext, perm = [27] * 5, [4, 1, 2, 0, 3]
    for blk in (1, 2, 5, 7, 13, 27):
        got, exp, info = _run(ext, perm, 8, 7100, plan_kwargs={"schema": "OD", "in_dim": 1,
                                                                  "in_block": blk})
        _assert_equal(got, exp, f"blockA={blk}")


# ---- edge cases ---------------------------------------------------------------------------------
def test_rank1_and_identity():
    for ext, perm in [([1], [0]), ([7], [0]), ([1 << 20], [0]), ([33, 17], [0, 1])]:
        got, exp, _ = _run(ext, perm, 4, 5)
        _assert_equal(got, exp, f"{ext}")


def test_rank15():
    ext = [2] * 15
    rng = np.random.default_rng(15)
    for _ in range(6):
        perm = [int(x) for x in rng.permutation(15)]
        got, exp, info = _run(ext, perm, 8, 15)
        _assert_equal(got, exp, f"rank15 {perm}")


def test_extent_one_dims():
    got, exp, _ = _run([1, 64, 1, 1, 48, 1], [4, 2, 1, 0, 5, 3], 8, 9)
    _assert_equal(got, exp, "squeeze")


def test_single_use_path():
    for c in configs.config1()[::5]:
        got, exp, _ = _run(c.extents, c.perm, 8, case_seed(c.case_id), single_use=True)
        _assert_equal(got, exp, "ttlg_transpose")


def test_misaligned_pointers_fall_back_to_element_width():
    ext, perm = [4, 256, 96], [0, 2, 1]          # 16-byte rows -> widened plan
    n = int(np.prod(ext))
    A = gen_tensor_torch(3, n + 1, 4, device=DEV)
    B = torch.empty(n + 1, dtype=torch.float32, device=DEV)
    p = ttlg.plan("f32", ext, perm)
    assert p.describe()["access_bytes"] == 16
    p.execute(A[1:].data_ptr(), B[1:].data_ptr(), torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    _assert_equal(_bits(B[1:]), oracle.transpose(_bits(A[1:]), ext, perm), "misaligned")


def test_nondefault_stream_and_aliasing():
    s = torch.cuda.Stream()
    ext, perm = [64, 48, 40], [2, 0, 1]
    A = gen_tensor_torch(4, 64 * 48 * 40, 8, device=DEV)
    B = torch.empty_like(A)
    p = ttlg.plan("f64", ext, perm)
    with torch.cuda.stream(s):
        p.execute(A.data_ptr(), B.data_ptr(), s.cuda_stream)
    s.synchronize()
    _assert_equal(_bits(B), oracle.transpose(_bits(A), ext, perm), "stream")
    with pytest.raises(ttlg.TtlgError) as e:
        p.execute(A.data_ptr(), A.data_ptr(), 0)
    assert e.value.code == 2


def test_transpose_tensor_torch_semantics():
    x = gen_tensor_torch(8, 6 * 7 * 8 * 9, 4, device=DEV).view(6, 7, 8, 9)
    for perm_t in [(3, 2, 1, 0), (0, 2, 1, 3), (1, 3, 0, 2)]:
        y = ttlg.transpose_tensor(x, perm_t)
        torch.cuda.synchronize()
        assert torch.equal(y.view(torch.int32).cpu(),
                           x.permute(perm_t).contiguous().view(torch.int32).cpu())
    e = torch.empty(0, 5, device=DEV)
    assert ttlg.transpose_tensor(e, (1, 0)).shape == (5, 0)


# ---- full BASELINE sizes, launch config as bench.py -----------------------------------------------
def _sampled_full(case, nsamp=200_000):
    n = case.n_elems
    eb = case.elem_bytes
    seed = case_seed(case.case_id)
    A = gen_tensor_torch(seed, n, eb, device=DEV)
    B = torch.empty_like(A)
    p = ttlg.plan(_dt(eb), case.extents, case.perm)
    p.execute(A.data_ptr(), B.data_ptr(), torch.cuda.current_stream().cuda_stream)
    rng = np.random.default_rng(case.case_id)
    linB = np.unique(np.concatenate([rng.integers(0, n, nsamp), np.arange(64),
                                     np.arange(n - 64, n)]))
    Bv = B.view(torch.int64 if eb == 8 else torch.int32)
    got = Bv[torch.from_numpy(linB).to(DEV)].cpu().numpy().view(np.uint64 if eb == 8 else np.uint32)
    linA = oracle.source_index(case.extents, case.perm, linB)
    exp = gen_at_np(seed, linA, eb)
    info = p.describe()
    del A, B
    torch.cuda.empty_cache()
    return got, exp, info


@pytest.mark.parametrize("case", configs.config2(), ids=lambda c: c.label())
def test_full_ttc57_sampled(case):
    got, exp, info = _sampled_full(case)
    _assert_equal(got, exp, f"{info['schema']}")


@pytest.mark.parametrize("case", configs.config3() + configs.config4(),
                         ids=lambda c: c.label())
def test_full_ccsdt_smallfvi_sampled(case):
    got, exp, info = _sampled_full(case, nsamp=50_000)
    _assert_equal(got, exp, f"{info['schema']}")


@pytest.mark.parametrize("case", configs.config5(), ids=lambda c: c.label())
def test_full_8GiB_sampled(case):
    got, exp, info = _sampled_full(case, nsamp=50_000)
    _assert_equal(got, exp, f"{info['schema']}")


def test_full_exactly_once_index_encoding():
    """Whole-tensor check at a TTC size: with A_bits[l] = l, B must be exactly
    oracle.source_index(arange(N)) (closed form from the definition)."""
    for case in configs.config2()[::7]:
        n = case.n_elems
        A = gen_tensor_torch(0, n, 8, device=DEV, mode="index")
        B = torch.empty_like(A)
        p = ttlg.plan("f64", case.extents, case.perm)
        p.execute(A.data_ptr(), B.data_ptr(), torch.cuda.current_stream().cuda_stream)
        got = B.view(torch.int64).cpu().numpy()
        exp = oracle.source_index(case.extents, case.perm, np.arange(n, dtype=np.int64))
        assert np.array_equal(got, exp), case.label()
        del A, B


@pytest.mark.parametrize("ext,perm,eb", [([320, 320, 256], [2, 1, 0], 8),      # 25 chunks
                                         ([64, 64, 64, 130], [3, 1, 0, 2], 4),  # q != d-1
                                         ([40, 50, 60], [0, 2, 1], 8),          # small: 1 stream
                                         ([33, 17, 2048, 9], [2, 3, 0, 1], 4),
                                         ([512, 64, 8, 128], [1, 3, 2, 0], 4),  # mode A
                                         ([16, 4, 16, 20, 16, 80], [5, 4, 3, 2, 1, 0], 8),
                                         ([80, 64, 80, 64], [3, 2, 1, 0], 8),   # reversal: middle split
                                         ([40, 30, 50, 70], [1, 3, 0, 2], 4)])
def test_execute_host_pipeline(ext, perm, eb):
    """ttlg_execute_host: chunked H2D / kernel / D2H over internal streams."""
    n = int(np.prod(ext))
    A = gen_tensor_torch(77, n, eb, device="cpu").pin_memory()
    B = torch.empty_like(A).pin_memory()
    Ad = torch.empty(n, dtype=A.dtype, device=DEV)
    Bd = torch.empty_like(Ad)
    p = ttlg.plan(_dt(eb), ext, perm)
    p.execute_host(A.data_ptr(), B.data_ptr(), Ad.data_ptr(), Bd.data_ptr(),
                   torch.cuda.current_stream().cuda_stream)
    torch.cuda.current_stream().synchronize()
    iv = torch.int64 if eb == 8 else torch.int32
    uv = np.uint64 if eb == 8 else np.uint32
    _assert_equal(B.view(iv).numpy().view(uv),
                  oracle.transpose(A.view(iv).numpy().view(uv), ext, perm), "execute_host")


@pytest.mark.parametrize("eb", [4, 8])
def test_long_single_digit_output_runs(eb):
    """Output runs longer than 16 x 32 lane slots (one output digit): the store
    phase walks them in chunks; forced tile [n0, 2048] on [n0, 4096, 24] (1 0 2)."""
    blk = 2048 if eb == 4 else 1024   # tile <= 64 KB
    for n0 in (2, 3, 5):
        ext, perm = [n0, 4096, 24], [1, 0, 2]
        for variant in (1, 2):
            got, exp, info = _run(ext, perm, eb, 300 + n0, plan_kwargs={
                "in_dim": 1, "in_block": blk, "out_dim": 0, "out_block": blk,
                "variant": variant})
            assert info["out_run"] == blk
            _assert_equal(got, exp, f"long runs n0={n0} {info['kernel']}")


def test_plan_tune_measure_mode():
    """ttlg_plan_tune (N2 measure mode) keeps a correct plan and reports time."""
    for c in configs.config1()[::6] + [configs.scaled(configs.config2()[20], 1 << 20)]:
        n = c.n_elems
        A = gen_tensor_torch(case_seed(c.case_id), n, c.elem_bytes, device=DEV)
        B = torch.empty_like(A)
        p = ttlg.plan(_dt(c.elem_bytes), c.extents, c.perm)
        t = p.tune(A.data_ptr(), B.data_ptr(), torch.cuda.current_stream().cuda_stream, 6)
        assert t > 0
        B.zero_()
        p.execute(A.data_ptr(), B.data_ptr(), torch.cuda.current_stream().cuda_stream)
        torch.cuda.synchronize()
        _assert_equal(_bits(B), oracle.transpose(_bits(A), c.extents, c.perm), "tuned plan")


# ---- every staged kernel variant forced (k_tile 1, k_pipe 2, k_quad 3), ragged tiles ----------
_VARIANT_CASES = [
    ([5120 // 16, 5120 // 20], [1, 0], 8),         # 2-D OD
    ([52, 36], [1, 0], 4),                           # small 2-D, partial tiles
    ([4, 1000, 60], [1, 2, 0], 4),                   # AoS -> SoA (fuses to [4, 60000] 1 0)
    ([8, 44, 36], [2, 1, 0], 4),
    ([24, 20, 12, 8], [3, 1, 0, 2], 8),
    ([16, 6, 10, 12, 4], [2, 0, 4, 1, 3], 8),
    ([12, 14, 16, 10], [1, 0, 3, 2], 4),
    ([2, 1000, 60], [1, 2, 0], 4),                   # fp32 even FVI: 8-byte chunks (K = 2)
    ([6, 44, 36], [2, 1, 0], 4),
    ([2, 300, 40], [1, 0, 2], 4),
]


@pytest.mark.parametrize("variant", [1, 2, 3, 5, 6, 7, 8])
@pytest.mark.parametrize("ext,perm,eb", _VARIANT_CASES)
def test_kernel_variants_forced(ext, perm, eb, variant):
    try:
        ttlg.plan(_dt(eb), ext, perm, variant=variant)
    except ttlg.TtlgError:
        pytest.skip("variant not applicable")
    got, exp, info = _run(ext, perm, eb, 77, plan_kwargs={"variant": variant}, canary=64)
    _assert_equal(got, exp, f"variant {variant} {info}")


@pytest.mark.parametrize("eb", [4, 8])
def test_quad_partial_tiles_and_blocks(eb):
    """k_quad under every block factor pair that leaves partial tiles on both sides."""
    ext, perm = [20 * (16 // eb), 28, 3], [1, 0, 2]
    n_ok = 0
    for ib in (4, 8, 12):
        for ob in (4, 8, 12, 16):
            kw = {"variant": 3, "in_dim": 0, "in_block": ib, "out_dim": 0, "out_block": ob}
            try:
                ttlg.plan(_dt(eb), ext, perm, **kw)
            except ttlg.TtlgError:
                continue
            got, exp, info = _run(ext, perm, eb, 91, plan_kwargs=kw, canary=32)
            assert info["kernel"] == "quad"
            _assert_equal(got, exp, f"quad {kw}")
            n_ok += 1
    assert n_ok >= 4


def test_quad_misaligned_pointers_fall_back():
    ext, perm = [64, 96], [1, 0]
    n = int(np.prod(ext))
    A = gen_tensor_torch(5, n + 1, 4, device=DEV)
    B = torch.empty(n + 1, dtype=torch.float32, device=DEV)
    p = ttlg.plan("f32", ext, perm, variant=3)
    assert p.describe()["kernel"] == "quad"
    p.execute(A[1:].data_ptr(), B[1:].data_ptr(), torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    _assert_equal(_bits(B[1:]), oracle.transpose(_bits(A[1:]), ext, perm), "quad misaligned")


@pytest.mark.parametrize("ext,eb,ob,threads", [([8, 3000], 4, 1024, 256), ([8, 3000], 4, 512, 256),
                                               ([6, 2050], 4, 2048, 512), ([4, 1800], 8, 1024, 256)])
def test_quad_multi_column(ext, eb, ob, threads):
    """k_quad with output runs longer than the block (2 or 4 positions per thread), ragged."""
    kw = {"variant": 3, "in_dim": 0, "in_block": ext[0], "out_dim": 0, "out_block": ob,
          "threads": threads}
    got, exp, info = _run(ext, [1, 0], eb, 93, plan_kwargs=kw, canary=32)
    assert info["kernel"] == "quad" and info["out_run"] > threads
    _assert_equal(got, exp, f"quad multi-column {kw}")


@pytest.mark.parametrize("eb", [4, 8])
def test_all_720_rank6_perms(eb):
    """N3: every permutation of a rank-6 tensor (the paper's 720-perm sweep,
    L1484-1493) at an oracle-sized shape with odd and even extents."""
    ext = [3, 4, 2, 5, 2, 3]
    for k, perm in enumerate(itertools.permutations(range(6))):
        got, exp, info = _run(ext, list(perm), eb, 3000 + k)
        _assert_equal(got, exp, f"{perm} {info['schema']} {info['kernel']}")


# ---- k_deint: [n0, M(, nb)] perm (1 0 (2)), 2 <= n0 <= 8 (AoS -> SoA) ------------------------
@pytest.mark.parametrize("eb", [4, 8])
@pytest.mark.parametrize("n0", [2, 3, 4, 5, 6, 7, 8])
def test_deint_forced(n0, eb):
    K = 16 // eb
    for ext, perm in (([n0, 11 * K, 7], [1, 0, 2]), ([n0, 250 * K], [1, 0]), ([n0, K, 3], [1, 0, 2])):
        got, exp, info = _run(ext, perm, eb, 500 + n0, plan_kwargs={"variant": 4}, canary=64)
        assert info["kernel"] == "deint" and info["schema"] == "OA", info
        _assert_equal(got, exp, f"deint {ext} {perm}")


def test_deint_auto_and_rules():
    # the config-4 AoS -> SoA cases plan onto k_deint; it does not apply when M is
    # not a multiple of 16/s or n0 > 8 (forcing it is then TTLG_ERR_UNSUPPORTED)
    for n0, perm in ((2, [1, 0, 2]), (3, [1, 2, 0]), (5, [1, 0, 2])):
        got, exp, info = _run([n0, 256, 24], perm, 4, 600 + n0)
        _assert_equal(got, exp, f"auto {n0} {perm} {info['kernel']}")
    for ext in ([3, 42, 5], [9, 40, 5]):
        with pytest.raises(ttlg.TtlgError) as e:
            ttlg.plan("f32", ext, [1, 0, 2], variant=4)
        assert e.value.code == 7


def test_deint_misaligned_pointers_fall_back():
    ext, perm = [3, 400, 5], [1, 0, 2]
    n = int(np.prod(ext))
    A = gen_tensor_torch(6, n + 1, 4, device=DEV)
    B = torch.empty(n + 1, dtype=torch.float32, device=DEV)
    p = ttlg.plan("f32", ext, perm, variant=4)
    assert p.describe()["kernel"] == "deint"
    p.execute(A[1:].data_ptr(), B[1:].data_ptr(), torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    _assert_equal(_bits(B[1:]), oracle.transpose(_bits(A[1:]), ext, perm), "deint misaligned")


@pytest.mark.parametrize("eb", [4, 8])
@pytest.mark.parametrize("n1", [2, 3, 4, 5, 6, 7, 8])
def test_inter_forced(n1, eb):
    """k_inter (SoA -> AoS): [M, n1(, nb)] perm (1 0 (2)) with the small extent on dim 1."""
    K = 16 // eb
    for ext, perm in (([11 * K, n1, 7], [1, 0, 2]), ([250 * K, n1], [1, 0]), ([K, n1, 3], [1, 0, 2])):
        got, exp, info = _run(ext, perm, eb, 700 + n1, plan_kwargs={"variant": 4}, canary=64)
        # both extents small ([K, n1, 3] with n1 a multiple of K): the AoS -> SoA form wins
        both = ext[0] <= 8 and n1 % K == 0
        assert info["kernel"] == "deint" and (both or info["in_run"] == K), info
        _assert_equal(got, exp, f"inter {ext} {perm}")
    # the auto plan for an SoA -> AoS case with a tiny structure
    got, exp, info = _run([4096, n1, 8], [1, 0, 2], eb, 800 + n1)
    _assert_equal(got, exp, f"auto {info['kernel']}")


@pytest.mark.parametrize("ext", [[24, 24, 12, 4, 3, 2], [24, 24, 24, 3, 2, 2]])
def test_closed_block_deep_tiles(ext):
    """1 0 2 4 3 5 with a >= 4 KB leading block: the deep k_pipe tiles."""
    got, exp, info = _run(ext, [1, 0, 2, 4, 3, 5], 8, 901, canary=64)
    _assert_equal(got, exp, f"deep {info['kernel']} {info['tile_extents']}")


def test_cuda_graph_capture_replay():
    """ttlg_execute launches can be captured into a CUDA graph (parameter
    blocks are baked into the kernel nodes) and replayed: bit-exact, and the
    plan may be destroyed after capture."""
    cases = [([64, 48, 40], [2, 0, 1], 8), ([3, 256, 24], [1, 0, 2], 4), ([40, 30, 20], [0, 2, 1], 4)]
    s = torch.cuda.Stream()
    bufs = []
    for k, (ext, perm, eb) in enumerate(cases):
        n = int(np.prod(ext))
        A = gen_tensor_torch(950 + k, n, eb, device=DEV)
        bufs.append((A, torch.empty_like(A), ttlg.plan(_dt(eb), ext, perm)))
    torch.cuda.synchronize()
    for A, B, p in bufs:  # warm-up outside capture (one-time function attributes)
        p.execute(A.data_ptr(), B.data_ptr(), s.cuda_stream)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for A, B, p in bufs:
            p.execute(A.data_ptr(), B.data_ptr(), s.cuda_stream)
    plans = [p for _, _, p in bufs]
    for p in plans:
        p.destroy()
    for _, B, _ in bufs:
        B.zero_()
    g.replay()
    torch.cuda.synchronize()
    for (ext, perm, eb), (A, B, _) in zip(cases, bufs):
        _assert_equal(_bits(B), oracle.transpose(_bits(A), ext, perm), f"graph {ext} {perm}")


def test_tuned_plan_on_misaligned_views():
    """A plan tuned on aligned buffers (its winner carries slice / kernel
    hints of the widened problem) still runs on element-aligned views: the
    element-width twin keeps only schema / no_fusion.  Tuning on
    misaligned buffers works too, and the twin is built once per plan."""
    stream = torch.cuda.current_stream().cuda_stream
    for ext, perm, eb in (([64, 64, 64], [0, 2, 1], 8), ([4, 256, 96], [0, 2, 1], 4),
                          ([64, 96], [1, 0], 4), ([3, 400, 8], [1, 0, 2], 4)):
        n = int(np.prod(ext))
        A = gen_tensor_torch(31, n + 1, eb, device=DEV)
        B = torch.empty_like(A)
        exp = oracle.transpose(_bits(A[1:]), ext, perm)
        p = ttlg.plan(_dt(eb), ext, perm)
        p.tune(A[:n].data_ptr(), B[:n].data_ptr(), stream, 6)
        for _ in range(2):
            B.zero_()
            p.execute(A[1:].data_ptr(), B[1:].data_ptr(), stream)
            torch.cuda.synchronize()
            _assert_equal(_bits(B[1:]), exp, f"tuned, misaligned {ext} {perm}")
        q = ttlg.plan(_dt(eb), ext, perm)
        q.tune(A[1:].data_ptr(), B[1:].data_ptr(), stream, 6)
        B.zero_()
        q.execute(A[1:].data_ptr(), B[1:].data_ptr(), stream)
        torch.cuda.synchronize()
        _assert_equal(_bits(B[1:]), exp, f"tuned on misaligned {ext} {perm}")


def test_transpose_tensor_rejects_mismatched_plan():
    x = gen_tensor_torch(8, 6 * 7 * 8, 4, device=DEV).view(6, 7, 8)
    ext, perm = ttlg.torch_to_c(list(x.shape), (2, 1, 0))
    good = ttlg.plan("f32", ext, perm)
    y = ttlg.transpose_tensor(x, (2, 1, 0), plan_=good)
    torch.cuda.synchronize()
    assert torch.equal(y.view(torch.int32).cpu(),
                       x.permute(2, 1, 0).contiguous().view(torch.int32).cpu())
    for bad in (ttlg.plan("f32", [8, 7, 7], perm), ttlg.plan("f64", ext, perm),
                ttlg.plan("f32", ext, [1, 0, 2])):
        with pytest.raises(ValueError):
            ttlg.transpose_tensor(x, (2, 1, 0), plan_=bad)


@pytest.mark.parametrize("count", [1, 3, 16, 21])
def test_execute_batch(count):
    """ttlg_execute_batch: one plan on `count` independent (A, B) pairs, one
    launch per 16 pairs (grid.y = pairs), each bit-exact; every kernel family."""
    stream = torch.cuda.current_stream().cuda_stream
    for ext, perm, eb, hints in (([64, 48, 40], [2, 0, 1], 8, {}),
                                 ([64, 96], [1, 0], 4, {"variant": 3}),
                                 ([40, 30, 20], [0, 2, 1], 4, {}),
                                 ([3, 256, 24], [1, 0, 2], 4, {"variant": 4}),
                                 ([24, 20, 12, 8], [3, 1, 0, 2], 8, {"variant": 2})):
        n = int(np.prod(ext))
        As = [gen_tensor_torch(1200 + i, n, eb, device=DEV) for i in range(count)]
        Bs = [torch.empty_like(a) for a in As]
        p = ttlg.plan(_dt(eb), ext, perm, **hints)
        p.execute_batch([a.data_ptr() for a in As], [b.data_ptr() for b in Bs], stream)
        torch.cuda.synchronize()
        for i in range(count):
            _assert_equal(_bits(Bs[i]), oracle.transpose(_bits(As[i]), ext, perm),
                          f"batch {i}/{count} {ext} {perm} {p.describe()['kernel']}")
    X, Y, Z = (torch.empty_like(As[0]) for _ in range(3))
    with pytest.raises(ttlg.TtlgError) as e:   # the A of pair 0 is the B of pair 1
        p.execute_batch([X.data_ptr(), Y.data_ptr()], [Z.data_ptr(), X.data_ptr()], stream)
    assert e.value.code == 2


def _bulk_cases():
    out = []
    for grp in ("c2", "c3", "c4", "c5"):
        out += [configs.scaled(c, 1 << 21) for c in configs.all_configs()[grp]]
    return out + [configs.scaled(c, 1 << 18) for c in configs.sweep720(16)[::37]]


@pytest.mark.parametrize("variant", [5, 6, 7])
@pytest.mark.parametrize("case", _bulk_cases(), ids=lambda c: c.label())
def test_bulk_forced(case, variant):
    """k_bulk (TMA bulk row loads into an mbarrier ring; 5 = quad consumers,
    6 = gather consumers) and k_vec (7: 16-byte cp.async loads, gathered
    16-byte stores) forced on every config shape they apply to."""
    try:
        ttlg.plan(_dt(case.elem_bytes), case.extents, case.perm, variant=variant)
    except ttlg.TtlgError:
        pytest.skip("k_bulk / k_vec not applicable (rows not 16-byte aligned)")
    got, exp, info = _run(case.extents, case.perm, case.elem_bytes, case_seed(case.case_id),
                          plan_kwargs={"variant": variant}, canary=64)
    assert info["kernel"] == {5: "bulkq", 6: "bulkg", 7: "vec"}[variant]
    _assert_equal(got, exp, f"bulk {variant} {info}")


@pytest.mark.parametrize("eb", [4, 8])
def test_bulk_partial_tiles(eb):
    """k_bulk with ragged tiles on both blocked dims (partial rows / row counts)."""
    K = 16 // eb
    n_ok = 0
    for ext, perm in (([6 * K, 40, 7], [1, 0, 2]), ([4 * K, 30, 3 * K], [2, 1, 0]),
                      ([2 * K, 50, 60], [0, 2, 1]), ([3, 4 * K * 11, 4 * K * 9], [2, 1, 0])):
        for variant in (5, 6, 7):
            for ib, ob in ((None, None), (3, 5), (K, 2 * K), (2 * K, 3 * K)):
                kw = {"variant": variant}
                if ib:
                    kw.update(in_dim=1, in_block=ib, out_dim=0, out_block=ob)
                try:
                    ttlg.plan(_dt(eb), ext, perm, **kw)
                except ttlg.TtlgError:
                    continue
                got, exp, info = _run(ext, perm, eb, 95, plan_kwargs=kw, canary=32)
                _assert_equal(got, exp, f"bulk partial {ext} {perm} {kw} {info}")
                n_ok += 1
    assert n_ok >= 6


@pytest.mark.parametrize("eb", [4, 8])
def test_rows_fml_unaligned_rows(eb):
    """k_rows (FML rows that are not 16-byte multiples): same-phase rows in
    16-byte chunks between an element-wise head and tail, different-phase rows
    element-wise; all-odd extents, mixed parities, row lengths of 1-300
    elements, partial tiles and misaligned base pointers.  k_rows is opt-in
    (TTLG_ROWS=1, read once per process): run in a child process."""
    import subprocess
    import sys
    if os.environ.get("TTLG_ROWS") != "1":
        r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", __file__ + "::"
                            f"test_rows_fml_unaligned_rows[{eb}]"],
                           env={**os.environ, "TTLG_ROWS": "1"}, capture_output=True, text=True)
        assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
        return
    for ext, perm in (([127, 7, 9], [0, 2, 1]), ([15, 15, 15, 15], [0, 2, 1, 3]),
                      ([17, 6, 9, 5], [0, 3, 2, 1]), ([127, 128, 5], [0, 2, 1]),
                      ([3, 50, 7], [0, 2, 1]), ([301, 3, 4, 5], [0, 3, 1, 2]),
                      ([1, 5, 13, 11], [0, 3, 2, 1]), ([129, 33], [0, 1])):
        got, exp, info = _run(ext, perm, eb, 1300, canary=32)
        _assert_equal(got, exp, f"rows {ext} {perm} {info['kernel']}")
        n = int(np.prod(ext))
        A = gen_tensor_torch(1301, n + 3, eb, device=DEV)
        B = torch.empty_like(A)
        p = ttlg.plan(_dt(eb), ext, perm)
        p.execute(A[1:].data_ptr(), B[3:].data_ptr(), torch.cuda.current_stream().cuda_stream)
        torch.cuda.synchronize()
        _assert_equal(_bits(B[3:]), oracle.transpose(_bits(A[1:n + 1]), ext, perm),
                      f"rows misaligned {ext} {perm}")


@pytest.mark.parametrize("eb", [4, 8])
def test_phase_forced_odd_extents(eb):
    """k_phase (16-byte loads at any row alignment, per-row phase in shared
    memory): every rank-4 perm of odd and mixed extents, ragged tiles, the
    end-of-tensor chunk, misaligned-by-one-element views (element-width twin)."""
    n_ok = 0
    for ext in ([15, 17, 13, 19], [3, 33, 65, 7], [17, 6, 9, 5], [5, 2, 129, 31]):
        for k, perm in enumerate(itertools.permutations(range(4))):
            try:
                ttlg.plan(_dt(eb), ext, list(perm), variant=8)
            except ttlg.TtlgError:
                continue
            got, exp, info = _run(ext, list(perm), eb, 1400 + k,
                                  plan_kwargs={"variant": 8}, canary=32)
            assert info["kernel"] == "phase"
            _assert_equal(got, exp, f"phase {ext} {perm} {info['tile_extents']}")
            n_ok += 1
    assert n_ok >= 40
    for ext, perm in (([17, 17, 17, 17], [3, 1, 2, 0]), ([15, 15, 15], [2, 0, 1])):
        for tiles in ({}, {"in_dim": 0, "in_block": 7, "out_dim": 0, "out_block": 5}):
            try:
                ttlg.plan(_dt(eb), ext, perm, variant=8, **tiles)
            except ttlg.TtlgError:
                continue
            got, exp, _ = _run(ext, perm, eb, 1500, plan_kwargs={"variant": 8, **tiles}, canary=32)
            _assert_equal(got, exp, f"phase {ext} {perm} {tiles}")


def _blk_cases():
    """Closed leading blocks: 2-D and 3-D inner perms, 16 / 8 / 4-byte chunks,
    1-16 chunks per lane, outer perms of every shape, a single block, blocks
    whose outer strides are odd element counts."""
    return [
        ([16, 16, 6, 5, 7], [1, 0, 2, 4, 3]),
        ([16, 16, 16, 16, 16, 16], [1, 0, 3, 5, 2, 4]),
        ([24, 24, 5, 7, 3], [1, 0, 4, 3, 2]),
        ([15, 15, 9, 11], [1, 0, 3, 2]),
        ([17, 17, 4, 9], [1, 0, 2, 3]),
        ([8, 8, 8, 33], [2, 1, 0, 3]),
        ([8, 4, 8, 20, 3], [2, 0, 1, 4, 3]),
        ([4, 8, 16, 2, 9], [1, 2, 0, 4, 3]),
        ([32, 32, 7, 3], [1, 0, 3, 2]),
        ([6, 12, 11, 13], [1, 0, 3, 2]),
        ([45, 45, 8], [1, 0, 2]),
        ([16, 16], [1, 0]),
        ([20, 12, 3, 7, 2], [1, 0, 4, 2, 3]),
    ]


@pytest.mark.parametrize("eb", [4, 8])
@pytest.mark.parametrize("ext,perm", _blk_cases(), ids=lambda v: "x".join(map(str, v)))
def test_blk_forced(ext, perm, eb):
    """k_blk (one warp per closed leading block, chunk loads, gathered chunk
    stores, padded per-warp staging) forced, against the oracle; also on a
    misaligned-by-one-element view (its element-width twin)."""
    try:
        ttlg.plan(_dt(eb), ext, perm, variant=9)
    except ttlg.TtlgError:
        pytest.skip("k_blk not applicable (block > 8 KB or < 32 chunks)")
    got, exp, info = _run(ext, perm, eb, 1700 + len(ext), plan_kwargs={"variant": 9}, canary=64)
    assert info["kernel"] == "blk"
    _assert_equal(got, exp, f"blk {ext} {perm} {info}")
    n = int(np.prod(ext))
    A = gen_tensor_torch(1799, n + 1, eb, device=DEV)
    B = torch.zeros(n + 3, dtype=A.dtype, device=DEV)
    p = ttlg.plan(_dt(eb), ext, perm, variant=9)
    p.execute(A[1:].data_ptr(), B[3:].data_ptr(), torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    _assert_equal(_bits(B[3:]), oracle.transpose(_bits(A[1:n + 1]), ext, perm),
                  f"blk misaligned {ext} {perm}")


def test_blk_batch():
    """k_blk through ttlg_execute_batch (grid.y); strided sub-boxes:
    tests/test_strided.py variant 9."""
    ext, perm = [16, 16, 5, 9], [1, 0, 3, 2]
    n = int(np.prod(ext))
    p = ttlg.plan("f64", ext, perm, variant=9)
    As = [gen_tensor_torch(1800 + i, n, 8, device=DEV) for i in range(3)]
    Bs = [torch.empty_like(a) for a in As]
    p.execute_batch([a.data_ptr() for a in As], [b.data_ptr() for b in Bs],
                    torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    for a, b in zip(As, Bs):
        _assert_equal(_bits(b), oracle.transpose(_bits(a), ext, perm), "blk batch")


@pytest.mark.parametrize("case", _bulk_cases(), ids=lambda c: c.label())
def test_tmap_forced(case):
    """k_tmap (variant 10: TMA tensor-map box loads, swizzled box rows, k_bulk's
    quad consumers) forced on every config shape it applies to (fused rank
    <= 5, 16-byte aligned strides)."""
    try:
        ttlg.plan(_dt(case.elem_bytes), case.extents, case.perm, variant=10)
    except ttlg.TtlgError:
        pytest.skip("k_tmap not applicable")
    got, exp, info = _run(case.extents, case.perm, case.elem_bytes, case_seed(case.case_id),
                          plan_kwargs={"variant": 10}, canary=64)
    assert info["kernel"] == "tmap"
    _assert_equal(got, exp, f"tmap {info}")


@pytest.mark.parametrize("eb", [4, 8])
def test_tmap_partial_tiles_panels_and_candidates(eb):
    """k_tmap on ragged tiles (the box's zero fill past the edge), input runs
    split into 128-byte panels, every candidate slice of a few shapes, and a
    batch of pairs (one tensor map per pair)."""
    K = 16 // eb
    n_ok = 0
    for ext, perm in (([6 * K, 40, 7], [1, 0, 2]), ([4 * K, 30, 3 * K], [2, 1, 0]),
                      ([64, 72, 5], [1, 0, 2]), ([80, 4, 16, 20, 16], [3, 2, 0, 4, 1]),
                      ([2 * K, 50, 3, 4 * K], [3, 1, 0, 2]), ([200, 136], [1, 0])):
        try:
            cands = ttlg.plan_candidates(_dt(eb), ext, perm, variant=10)
        except ttlg.TtlgError:
            continue
        for cd in cands[:: max(1, len(cands) // 12)]:
            kw = dict(cd["hints"])
            got, exp, info = _run(ext, perm, eb, 96, plan_kwargs=kw, canary=32)
            assert info["kernel"] == "tmap"
            _assert_equal(got, exp, f"tmap {ext} {perm} {kw} {info}")
            n_ok += 1
    assert n_ok >= 20
    ext, perm = [64, 72, 5], [1, 0, 2]
    n = int(np.prod(ext))
    p = ttlg.plan(_dt(eb), ext, perm, variant=10)
    As = [gen_tensor_torch(1900 + i, n, eb, device=DEV) for i in range(3)]
    Bs = [torch.empty_like(a) for a in As]
    p.execute_batch([a.data_ptr() for a in As], [b.data_ptr() for b in Bs],
                    torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    for a, b in zip(As, Bs):
        _assert_equal(_bits(b), oracle.transpose(_bits(a), ext, perm), "tmap batch")
