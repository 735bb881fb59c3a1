"""Host-side logic through the C ABI, on a CPU-only box (virtual B200 profile):
ABI exports, argument validation, squeeze + index fusion,
schema applicability (Alg. 1), forced schemas, kernel-parameter
legality, model sanity, and the torch <-> FVI-first convention conversion."""
import ctypes
import itertools
import os
import re
import subprocess

import numpy as np
import pytest

import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg
from paper_conf_ipps_veduradasskhpkn18_b200 import _ffi
from synth import configs

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


# ---- ABI ----------------------------------------------------------------------------
def test_header_symbols_exported():
    hdr = open(os.path.join(ROOT, "include", "ttlg.h")).read()
    declared = set(re.findall(r"\b(ttlg_[a-z_]+)\s*\(", hdr))
    out = subprocess.run(["nm", "-D", "--defined-only", _ffi.LIB_PATH], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r"\bT (ttlg_[a-z_]+)\b", out))
    assert declared, "no declarations parsed"
    assert declared <= exported, declared - exported
    assert set(_ffi.EXPORTS) == declared


def test_status_strings_and_version():
    assert _ffi.lib.ttlg_version() == 100
    assert _ffi.lib.ttlg_status_string(0) == b"TTLG_OK"
    assert _ffi.lib.ttlg_status_string(2) == b"TTLG_ERR_ALIASING"
    assert _ffi.lib.ttlg_schema_name(3) == b"OD"


def test_library_has_sm100a_code():
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", _ffi.LIB_PATH],
                         capture_output=True, text=True, check=True).stdout
    assert "sm_100a" in out


# ---- validation ------------------------------------------------------------------------
@pytest.mark.parametrize("ext,perm", [
    ([], []), ([2] * 16, list(range(16))), ([0, 3], [1, 0]), ([2, 3], [0, 0]),
    ([2, 3], [0, 2]), ([-1, 3], [1, 0]), ([1 << 40, 1 << 30], [1, 0])])
def test_invalid_arguments(ext, perm):
    with pytest.raises(ttlg.TtlgError) as e:
        ttlg.plan("f64", ext, perm)
    assert e.value.code == 1


def test_bad_dtype_code():
    with pytest.raises(ttlg.TtlgError):
        ttlg.plan(7, [4, 4], [1, 0])


def test_execute_without_gpu_is_device_error():
    p = ttlg.plan("f32", [64, 64], [1, 0])
    with pytest.raises(ttlg.TtlgError) as e:
        p.execute(1 << 20, 1 << 30)
    assert e.value.code == 3  # TTLG_ERR_DEVICE (no device here), never a CPU fallback


def test_aliasing_detected_before_device_check():
    p = ttlg.plan("f64", [64, 64], [1, 0])
    with pytest.raises(ttlg.TtlgError) as e:
        p.execute(1 << 20, (1 << 20) + 8)
    assert e.value.code == 2
    with pytest.raises(ttlg.TtlgError) as e:
        p.execute((1 << 20) + 4, 1 << 30)   # not element aligned
    assert e.value.code == 1


# ---- fusion -----------------------------------------------------------------------------
def test_paper_fusion_example():
    # [i0,i1,i2,i3] => [i3,i1,i2,i0] fuses i1,i2 into rank 3
    d = ttlg.plan("f32", [5, 6, 7, 8], [3, 1, 2, 0]).describe()
    assert d["fused_rank"] == 3
    assert d["fused_extents"] == [5, 42, 8]
    assert d["fused_perm"] == [2, 1, 0]


def test_fused_rank_histogram_720():
    # the "staircase" of Figs 6-11 (L1586-1588): scaled ranks of all 720 6-D perms
    hist = {}
    for p in itertools.permutations(range(6)):
        d = ttlg.plan("f32", [3] * 6, p).describe()["fused_rank"]
        hist[d] = hist.get(d, 0) + 1
    assert hist == {1: 1, 2: 5, 3: 30, 4: 110, 5: 265, 6: 309}


def test_squeeze_and_identity():
    d = ttlg.plan("f64", [1, 7, 1, 9], [3, 2, 0, 1]).describe()
    assert d["fused_rank"] == 2 and d["fused_extents"] == [7, 9] and d["fused_perm"] == [1, 0]
    d = ttlg.plan("f32", [4, 5, 6], [0, 1, 2]).describe()
    assert d["schema"] == "COPY" and d["fused_rank"] == 1
    d = ttlg.plan("f64", [1, 1], [1, 0]).describe()
    assert d["schema"] == "COPY"


def test_widening_small_fvi():
    # [2,4096,4096] fp32 perm 0 2 1: 8-byte rows -> one access element -> 2-D transpose
    d = ttlg.plan("f32", [2, 4096, 4096], [0, 2, 1]).describe()
    assert d["access_bytes"] == 8 and d["fused_rank"] == 2 and d["fused_perm"] == [1, 0]
    d = ttlg.plan("f32", [4, 4096, 4096], [0, 2, 1]).describe()
    assert d["access_bytes"] == 16 and d["fused_rank"] == 2
    d = ttlg.plan("f32", [3, 4096, 4096], [0, 2, 1]).describe()
    assert d["access_bytes"] == 4 and d["fused_rank"] == 3


# ---- schema applicability -------------------------------------------------------------------
def _groups(d):
    a, b = d["in_dim"], d["out_dim"]
    IS = set(range(a + 1))
    OS = set(d["fused_perm"][: b + 1])
    return IS, OS


def _check_plan_legal(d):
    IS, OS = _groups(d)
    fp, te, fe = d["fused_perm"], d["tile_extents"], d["fused_extents"]
    for k in range(d["fused_rank"]):
        assert 1 <= te[k] <= fe[k]
        if k not in IS and k not in OS:
            assert te[k] == 1
    for k in range(d["in_dim"]):
        assert te[k] == fe[k]                      # only the slowest input-group dim is blocked
    for i in range(d["out_dim"]):
        assert te[fp[i]] == fe[fp[i]]              # only the slowest output-group dim is blocked
    if d["schema"] == "OD":
        assert not (IS & OS)
    if d["schema"] == "OA":
        assert IS & OS and fp[0] != 0
    if d["schema"] in ("FML", "FMS", "COPY"):
        assert fp[0] == 0
    assert d["param_bytes"] <= 32764
    assert d["smem_bytes"] <= 227 * 1024
    assert d["predicted_seconds"] >= d["bytes"] / 6555.5e9 * 0.999


@pytest.mark.parametrize("group", ["c1", "c2", "c3", "c4", "c5"])
def test_auto_plans_legal(group):
    for c in configs.all_configs()[group]:
        d = ttlg.plan("f64" if c.elem_bytes == 8 else "f32", c.extents, c.perm).describe()
        _check_plan_legal(d)


def test_forced_schemas():
    ok = {"OD": 0, "OA": 0, "FMS": 0, "FML": 0}
    for c in configs.config1():
        fp0 = c.perm[0]
        for s in ("OD", "OA", "FMS", "FML"):
            try:
                d = ttlg.plan("f64", c.extents, c.perm, schema=s).describe()
            except ttlg.TtlgError as e:
                assert e.code == 7
                continue
            assert d["schema"] == s or (s == "FML" and d["schema"] == "COPY")
            _check_plan_legal(d)
            ok[s] += 1
        # applicability: OD whenever the fused FVI differs; FML whenever it matches
        d0 = ttlg.plan("f64", c.extents, c.perm).describe()
        if d0["fused_perm"][0] != 0:
            ttlg.plan("f64", c.extents, c.perm, schema="OD")
        else:
            ttlg.plan("f64", c.extents, c.perm, schema="FML")
    assert all(v > 0 for v in ok.values()), ok


def test_forced_blocks_respected():
    d = ttlg.plan("f64", [27] * 5, [4, 1, 2, 0, 3], schema="OD", in_dim=1, in_block=7,
                  out_dim=0, out_block=27).describe()
    # Fig. 5's choice (L1435-1436): input slice 27x7 = 189, output slice 27
    assert d["in_run"] == 189 and d["out_run"] == 27


def test_predict_time_monotone_in_volume():
    t1 = ttlg.predict_time("f64", [256, 256, 64], [2, 1, 0])
    t2 = ttlg.predict_time("f64", [256, 256, 512], [2, 1, 0])
    assert t2 > 2.5 * t1   # 8x the volume
    assert t2 >= 2 * 256 * 256 * 512 * 8 / 6555.5e9


# ---- torch convention -------------------------------------------------------------------------
def test_torch_to_c_matches_numpy_transpose():
    import oracle
    rng = np.random.default_rng(0)
    for _ in range(50):
        d = int(rng.integers(1, 6))
        shape = [int(x) for x in rng.integers(1, 5, size=d)]
        perm_t = [int(x) for x in rng.permutation(d)]
        X = np.arange(int(np.prod(shape)), dtype=np.uint64).reshape(shape)
        ext, perm = ttlg.torch_to_c(shape, perm_t)
        got = oracle.transpose(X.ravel(), ext, perm)
        assert np.array_equal(got, np.ascontiguousarray(X.transpose(perm_t)).ravel())
    # 2-D: (1, 0) <-> (1, 0)
    assert ttlg.torch_to_c([3, 5], [1, 0]) == ([5, 3], [1, 0])


def test_plan_candidates_every_config_case():
    """Listing mode (calibration) builds the exact parameter block of every
    candidate of every kernel family: must never fault on any config case."""
    from synth import configs
    groups = configs.all_configs()
    for g in ("c1", "c2", "c3", "c4"):
        for c in groups[g]:
            dt = "f64" if c.elem_bytes == 8 else "f32"
            cands = ttlg.plan_candidates(dt, c.extents, c.perm)
            assert cands, c.label()
            kinds = {d["kernel"] for d in cands}
            # k_bulk only when forced or TTLG_BULK=1
            assert kinds <= {"direct", "tile", "pipe", "quad", "deint", "vec", "blk"}
            for d in cands:
                if d["kernel"] == "vec":   # every listed k_vec slice plans as itself
                    assert d["access_bytes"] in (4, 8)
    # forced k_bulk / k_vec listings hold only their kernel and every entry re-plans
    for c in groups["c2"][::6]:
        for v, name in ((5, "bulkq"), (6, "bulkg"), (7, "vec")):
            try:
                cands = ttlg.plan_candidates("f64", c.extents, c.perm, variant=v)
            except ttlg.TtlgError:
                continue
            assert {d["kernel"] for d in cands} <= {name}
            for d in cands[:5]:
                info = ttlg.plan("f64", c.extents, c.perm, **d["hints"]).describe()
                assert info["kernel"] == name and info["tile_extents"] == d["tile_extents"]


def test_bench_reference_arm_contract():
    """bench.py --impl reference (the oracle on the host cores) prints ONE JSON
    line with the driver's keys; runs on a CPU-only host."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--impl", "reference",
                          "--workload", "c1", "--steps", "2", "--warmup", "3",
                          "--ref-cases-per-step", "4"], capture_output=True, text=True,
                         timeout=300, cwd=root)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "scaling", "vs_baseline", "dtype", "data", "config",
              "cpu_baseline", "e2e", "impl"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["steps"] == 2
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0


def test_deep_tiles_only_for_closed_leading_blocks():
    """Input runs one dim past 4 KB (k_pipe only) are enumerated only when the
    leading input block is also the leading output block (1 0 2 4 3 5 family)."""
    cands = ttlg.plan_candidates("f64", [24] * 6, [1, 0, 2, 4, 3, 5])
    assert any(c["kernel"] == "pipe" and c["in_dim"] == 2 and c["tile_extents"][2] > 1
               for c in cands)
    # not closed (perm[0..1] = 2 0): no deep candidate may appear
    for c in ttlg.plan_candidates("f64", [16, 4, 16, 20, 16, 80], [2, 0, 4, 1, 5, 3]):
        fe, te = c["fused_extents"], c["tile_extents"]
        pre = 1
        for k in range(c["in_dim"]):
            pre *= fe[k]
        assert pre * 8 < 4096 or c["in_dim"] == 0, c


def test_vec_and_bulk_applicability():
    """k_vec / k_bulk move whole 16-byte chunks: every A-row (and B-row) of every
    tile must start 16-byte aligned; odd fp64
    extents never qualify, 12-byte pencils do with 4-pencil blocks."""
    p = ttlg.plan("f32", [3, 4096, 4096], [0, 2, 1], variant=7).describe()
    assert p["kernel"] == "vec"
    t = p["tile_extents"]
    assert (t[0] * t[1] * 4) % 16 == 0 and (t[0] * t[2] * 4) % 16 == 0
    for v in (5, 6, 7):
        with pytest.raises(ttlg.TtlgError) as e:
            ttlg.plan("f64", [17, 17, 17], [2, 1, 0], variant=v)
        assert e.value.code == 7
    # quad consumers need an Orthogonal-Distinct tile
    with pytest.raises(ttlg.TtlgError):
        ttlg.plan("f32", [4, 64, 64], [0, 2, 1], variant=5, schema="FMS")
    b = ttlg.plan("f64", [64, 96], [1, 0], variant=5).describe()
    assert b["kernel"] == "bulkq" and b["stages"] >= 2 and b["threads"] in (288, 544)


def test_generalised_quad_chunks():
    """k_quad needs chunk-aligned rows, not FVI multiples of K: [3, 4096, 4096]
    fp32 `2 1 0` runs in 16-byte chunks with t1 a multiple of 4."""
    d = ttlg.plan("f32", [3, 4096, 4096], [2, 1, 0], variant=3).describe()
    assert d["kernel"] == "quad"
    assert (d["tile_extents"][0] * d["tile_extents"][1]) % 4 == 0
    with pytest.raises(ttlg.TtlgError):
        ttlg.plan("f32", [3, 4096, 4096], [2, 1, 0], variant=3, in_dim=1, in_block=21)


def test_execute_batch_validation_without_gpu():
    p = ttlg.plan("f64", [64, 64], [1, 0])
    with pytest.raises(ttlg.TtlgError) as e:   # pair 1's B is pair 0's A
        p.execute_batch([1 << 20, 1 << 28], [1 << 30, 1 << 20])
    assert e.value.code == 2
    with pytest.raises(ttlg.TtlgError) as e:
        p.execute_batch([1 << 20, (1 << 28) + 4], [1 << 30, 1 << 32])
    assert e.value.code == 1                    # not element aligned
    with pytest.raises(ttlg.TtlgError) as e:
        p.execute_batch([1 << 20] * 3, [1 << 30, 1 << 31, 1 << 32])
    assert e.value.code == 3                    # valid arguments, no device here
    with pytest.raises(ValueError):
        p.execute_batch([1 << 20], [])


def test_blk_applicability():
    """k_blk needs a closed leading block ({perm[0..c-1]} = {0..c-1}, c >= 2)
    of 32 chunks .. 8 KB, contiguous in both tensors; the chunk width divides
    the dim-0 row, the block and every outer stride."""
    cases = [  # (dtype, extents, perm, applies, chunk bytes)
        ("f64", [16] * 6, [1, 0, 2, 4, 3, 5], True, 16),
        ("f64", [24] * 6, [1, 0, 5, 4, 3, 2], True, 16),
        ("f64", [15] * 6, [1, 0, 2, 4, 3, 5], True, 8),   # odd rows: 8-byte chunks
        ("f32", [15, 15, 40], [1, 0, 2], True, 4),
        ("f64", [8, 8, 8, 64], [2, 1, 0, 3], True, 16),   # 3-D inner permutation
        ("f64", [80, 16, 80, 256], [1, 0, 3, 2], False, 0),  # 10 KB block
        ("f64", [16] * 6, [2, 0, 4, 1, 5, 3], False, 0),    # not closed before dim 5
        ("f64", [16] * 6, [0, 2, 1, 3, 4, 5], False, 0),    # matching FVI (FML)
        ("f64", [4, 4, 64], [1, 0, 2], False, 0),           # 16 chunks: lanes idle
    ]
    for dt, ext, perm, ok, wc in cases:
        if ok:
            d = ttlg.plan(dt, ext, perm, variant=9).describe()
            assert d["kernel"] == "blk" and d["access_bytes"] == wc, (ext, perm, d)
            assert d["schema"] == "OA" and d["threads"] == 256
        else:
            with pytest.raises(ttlg.TtlgError) as e:
                ttlg.plan(dt, ext, perm, variant=9)
            assert e.value.code == 7
    # slice hints rule it out; the element-width twin keeps it at element width
    with pytest.raises(ttlg.TtlgError):
        ttlg.plan("f64", [16] * 6, [1, 0, 2, 4, 3, 5], variant=9, in_dim=2, in_block=4)
    d = ttlg.plan("f64", [16] * 6, [1, 0, 2, 4, 3, 5], variant=9,
                  access_bytes=8).describe()
    assert d["kernel"] == "blk" and d["access_bytes"] == 8


def test_tmap_applicability():
    """k_tmap (variant 10) describes the OD tile as a TMA box: fused rank <= 5,
    16-byte multiples for every A stride past the FVI, box rows <= 128 bytes
    (longer input runs split into 128-byte panels), k_quad's chunk alignment.
    Not in the automatic choice unless TTLG_TMA=1."""
    d = ttlg.plan("f64", [5120, 5120], [1, 0], variant=10).describe()
    assert d["kernel"] == "tmap" and d["schema"] == "OD" and d["stages"] >= 2
    assert d["threads"] in (288, 544)
    # a fused rank-5 problem qualifies; rank 6 (16^6 reversal) does not
    assert ttlg.plan("f64", [80, 4, 16, 20, 16], [3, 2, 0, 4, 1],
                     variant=10).describe()["kernel"] == "tmap"
    for ext, perm in (([16] * 6, [5, 4, 3, 2, 1, 0]), ([17, 17, 17], [2, 1, 0]),
                      ([3, 4096, 4096], [2, 1, 0])):
        with pytest.raises(ttlg.TtlgError) as e:
            ttlg.plan("f64" if ext[0] != 3 else "f32", ext, perm, variant=10)
        assert e.value.code == 7
    # every candidate keeps the box rule: the input run is one box row of a
    # swizzle span (16 / 32 / 64 / 128 bytes) or whole 128-byte panels of dim a
    for c in ttlg.plan_candidates("f64", [200, 136], [1, 0], variant=10):
        la = c["in_run"] * 8
        assert la in (16, 32, 64, 128) or la % 128 == 0
    auto = ttlg.plan("f64", [5120, 5120], [1, 0]).describe()
    assert auto["kernel"] != "tmap"


def test_direct_cap_for_odd_short_rows():
    """k_direct tiles of >= 32 output rows that are not 32-byte multiples and
    shorter than 2 KB stay <= 34 KB (r2e45-47: 127^4 `0 2 1 3`
    [127, 127] ran 4.6 TB/s, [127, 33] 6.5); 2312-byte rows (17^6) are not
    capped; TTLG_FML_CAP=0 lifts the cap (checked in a child process: the
    flag is read once)."""
    for ext in ([127] * 4, [63] * 4, [31] * 4):
        for c in ttlg.plan_candidates("f64", ext, [0, 2, 1, 3]):
            if c["kernel"] == "direct" and c["tile_volume"] // c["tile_extents"][0] >= 32:
                assert c["tile_volume"] * 8 <= 34 * 1024, c
    big = [c for c in ttlg.plan_candidates("f64", [17] * 6, [0, 1, 4, 3, 2, 5])
           if c["kernel"] == "direct" and c["tile_volume"] * 8 > 34 * 1024]
    assert big
    import subprocess
    import sys
    code = ("import paper_conf_ipps_veduradasskhpkn18_b200 as t\n"
            "c = t.plan_candidates('f64', [127] * 4, [0, 2, 1, 3])\n"
            "print(max(x['tile_volume'] for x in c if x['kernel'] == 'direct') * 8)\n")
    env = dict(os.environ, TTLG_FML_CAP="0")
    out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True,
                         cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    assert int(out.stdout.strip()) > 34 * 1024, out.stderr
