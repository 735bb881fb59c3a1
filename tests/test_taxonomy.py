"""The strict Alg. 1 classifier (oracle/taxonomy.py, test infrastructure) pinned
to what the paper and SURVEY.md App. A fix, and the product planner checked
against it (SURVEY §8(c) "Schema (a2)" pin; reading R6).

Pins:
- PAPER.md L263-277: [a,b,c,d] => [d,c,b,a] with extents 16,2,32,32 is
  Orthogonal-Distinct, with I = {a,b} (16*2 = 32 elements) and O = {d};
- PAPER.md L435-452: [a,b,c,d] => [c,b,d,a] with extents 8,2,8,8 is
  Orthogonal-Arbitrary: I = {a,b,c}, O = {c,b,d} overlap;
- Fig. 2 (L402-418): (0 1 2) -> (2 1 0) is Orthogonal-Distinct; its 9x7x64
  slice in 4 phases of 32x32 fixes n0 = 9, n1 = 7 (I = {i0,i1}, 63 >= 32) and
  n2 >= 32 (O = {i2}) -- the figure's extents are garbled, this is the reading;
- L596-601 and the flowchart text L674-681: matching FVI >= 32 -> FML,
  < 32 with the two-index products >= 32 -> FMS, else OA;
- L668-685: the fusion example [i0,i1,i2,i3] => [i3,i1,i2,i0] -> rank 3;
- SURVEY.md App. A label counts (derived independently from the same
  reading): TTC-57 37 OD / 8 OA / 10 FML / 2 FMS, 16^4 4 OD / 14 OA / 4 FMS /
  2 FML, 720-perm sweeps 288 / 312 / 96 / 24 at every size, the CCSD(T),
  small-FVI and 8 GiB tables, and the fused-rank staircase
  {1: 1, 2: 5, 3: 30, 4: 110, 5: 265, 6: 309} (Figs. 6-11).
"""
import itertools
from collections import Counter

import pytest

from oracle.taxonomy import FML, FMS, OA, OD, classify, fuse, _prefix_group
from synth import configs
import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg


# ---- the paper's worked examples ----------------------------------------------------------
def test_l263_orthogonal_distinct_example():
    ext, perm = [16, 2, 32, 32], [3, 2, 1, 0]      # [a,b,c,d] => [d,c,b,a]
    assert fuse(ext, perm) == (ext, perm)           # nothing fuses
    assert _prefix_group(range(4), ext, 32) == {0, 1}   # "a and b ... combined", 32 elements
    assert _prefix_group(perm, ext, 32) == {3}          # 'd' alone (32)
    assert classify(ext, perm) == OD


def test_l435_orthogonal_arbitrary_example():
    ext, perm = [8, 2, 8, 8], [2, 1, 3, 0]          # [a,b,c,d] => [c,b,d,a]
    assert _prefix_group(range(4), ext, 32) == {0, 1, 2}   # {a,b,c}: 128
    assert _prefix_group(perm, ext, 32) == {2, 1, 3}       # {c,b,d}: 128
    assert classify(ext, perm) == OA


def test_fig2_orthogonal_distinct():
    # (0 1 2) -> (2 1 0), 9 x 7 x 64 slice (reading of the garbled figure)
    assert classify([9, 7, 64], [2, 1, 0]) == OD
    assert classify([9, 7, 640], [2, 1, 0]) == OD


@pytest.mark.parametrize("n0,n1,n3,want", [(64, 8, 8, FML), (32, 2, 2, FML),
                                           (16, 4, 4, FMS), (8, 4, 4, FMS),
                                           (4, 4, 16, OA), (8, 2, 64, OA),
                                           (8, 8, 2, OA)])
def test_fvi_match_branches(n0, n1, n3, want):
    # [a,b,c,d] => [a,d,c,b] (L596-601): perm (0 3 2 1), n2 = 5 keeps c unfused
    assert classify([n0, n1, 5, n3], [0, 3, 2, 1]) == want


def test_fusion_example_l668():
    ext, perm = [3, 5, 7, 11], [3, 1, 2, 0]
    assert fuse(ext, perm) == ([3, 35, 11], [2, 1, 0])
    assert fuse([2, 3, 4], [0, 1, 2]) == ([24], [0])
    assert fuse([1, 5, 1, 7], [3, 2, 1, 0]) == ([5, 7], [1, 0])   # squeeze, then fuse
    assert classify([4, 4, 4], [0, 1, 2]) == FML                   # copy


def test_fused_rank_staircase_720():
    hist = Counter(len(fuse([16] * 6, p)[0]) for p in itertools.permutations(range(6)))
    assert dict(hist) == {1: 1, 2: 5, 3: 30, 4: 110, 5: 265, 6: 309}


# ---- SURVEY.md App. A label tables -------------------------------------------------------------
def _counts(cases):
    return dict(Counter(classify(c.extents, c.perm) for c in cases))


def test_appA_counts_configs_1_2_and_sweeps():
    assert _counts(configs.config1()) == {OD: 4, OA: 14, FMS: 4, FML: 2}
    assert _counts(configs.config2()) == {OD: 37, OA: 8, FML: 10, FMS: 2}
    for e in (15, 16, 17):
        assert _counts(configs.sweep720(e)) == {FML: 24, FMS: 96, OA: 312, OD: 288}


def test_appA_ttc_rows():
    # App. A: perm -> schema per extent profile (P1, P2, P3)
    rows = {"0 2 1": "FML FML FML", "1 0 2": "OD OD OD", "2 1 0": "OD OD OD",
            "0 3 2 1": "FML FML FML", "2 1 3 0": "OD OD OD", "2 0 3 1": "OD OD OD",
            "1 0 3 2": "OD OA OA", "3 2 1 0": "OD OD OD",
            "0 4 2 1 3": "FML FML FML", "3 2 1 4 0": "OD OD OD", "2 0 4 1 3": "OA OA OA",
            "1 3 0 4 2": "OD OD OD", "4 3 2 1 0": "OD OD OD",
            "0 3 2 5 4 1": "FMS FML FMS", "3 2 0 5 1 4": "OD OD OD", "2 0 4 1 5 3": "OA OA OA",
            "3 2 5 1 0 4": "OD OD OD", "5 4 3 2 1 0": "OD OD OD", "1 0": "OD OD OD"}
    got = {}
    for c in configs.config2():
        got.setdefault(" ".join(map(str, c.perm)), []).append(classify(c.extents, c.perm))
    assert {k: " ".join(v) for k, v in got.items()} == rows


def test_appA_ccsdt_table():
    want = {(16,) * 6: "FMS FMS FML OA OD OD OA OA",
            (24,) * 6: "FMS FMS FML OA OD OD OA OA",
            (32, 32, 32, 16, 16, 16): "FML FML FML OD OD OD OD OD",
            (48, 48, 48, 16, 16, 16): "FML FML FML OD OD OD OD OD",
            (72, 72, 16, 16, 16, 16): "FML FML FML OD OD OD OD OD"}
    got = {}
    for c in configs.config3():
        got.setdefault(c.extents, []).append(classify(c.extents, c.perm))
    assert {k: " ".join(v) for k, v in got.items()} == want


def test_appA_smallfvi_and_8gib():
    for c in configs.config4():
        want = {(0, 2, 1): FMS, (2, 1, 0): OD, (1, 0, 2): OA, (1, 2, 0): OA,
                (2, 0, 1): OD}[c.perm]
        assert classify(c.extents, c.perm) == want, c.label()
    assert [classify(c.extents, c.perm) for c in configs.config5()] == [OD, OD, OD, FML, OD]


# ---- the product planner against the strict reading ----------------------------------------
def _product_cases():
    out = []
    for grp in ("c1", "c2", "c3", "c4", "c5"):
        out += configs.all_configs()[grp]
    return out + configs.sweep720(15)[::7] + configs.sweep720(17)[::7]


def test_product_accepts_the_strict_schema():
    """Every strict Alg. 1 label is a schema the product can run (forced): the
    production choice differs only by model arbitration (readings R9-R11),
    never by applicability.  The one exception is DESIGN.md's FVI widening:
    an FMS pencil of exactly one 8/16-byte access element ([2|4, 4096, 4096]
    fp32 `0 2 1`) is squeezed into the element, so the problem becomes a 2-D
    Orthogonal-Distinct transpose of wide elements."""
    for c in _product_cases():
        s = classify(c.extents, c.perm)
        dt = "f64" if c.elem_bytes == 8 else "f32"
        try:
            ttlg.plan(dt, c.extents, c.perm, schema=s)
        except ttlg.TtlgError:
            info = ttlg.plan(dt, c.extents, c.perm).describe()
            assert s == FMS and c.perm[0] == 0 and info["schema"] == OD
            assert c.extents[0] * c.elem_bytes == info["access_bytes"], c.label()
