"""TTGT tensor contraction driven by the transposition performance model.

The paper's motivating client: a
Transpose-Transpose-GEMM-Transpose contraction system asks the transposition
library how long each candidate layout change would take and picks the
cheapest set (the model "can be queried ... to choose the best layout").
SURVEY.md §8(f) N4.

    C[idx_c] = sum_k A[idx_a] * B[idx_b]          (einsum-style, torch row-major)

Indices of A and C are "m" (free left), of B and C "n" (free right), of A and
B only "k" (contracted).  A GEMM computes C' = A' @ B' with A' an M x K (or
K x M, passed transposed) matrix view, B' K x N (or N x K), C' M x N (or the
transposed product N x M).  Each matrix view is a permutation of the operand;
the order of the indices inside each group is free.  `plan_contraction`
enumerates the group orders (as they appear in A, in B or in C) and the three
transposed/non-transposed GEMM forms, prices every needed transposition with
`ttlg_predict_time` (identity permutations cost nothing: the view is free) and
keeps the cheapest.  The contraction itself is the library's transposition
kernels around a cuBLAS GEMM (torch.matmul).  Batch indices (present in A, B
and C) and repeated indices are not supported.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Dict, List, Sequence, Tuple

from .api import predict_time, torch_to_c, transpose_tensor


def _parse(spec: str) -> Tuple[str, str, str]:
    lhs, out = spec.replace(" ", "").split("->")
    a, b = lhs.split(",")
    for s in (a, b, out):
        if len(set(s)) != len(s):
            raise ValueError(f"repeated index in {s!r}")
    if set(out) - set(a) - set(b):
        raise ValueError("output index missing from the inputs")
    if set(a) & set(b) & set(out):
        raise ValueError("batch indices (in A, B and C) are not supported")
    if (set(a) ^ set(b)) - set(out):
        raise ValueError("an index of only one input must appear in the output")
    return a, b, out


def _perm_to(src: str, dst: str) -> List[int]:
    """torch permute order taking a tensor indexed `src` to the index order `dst`."""
    return [src.index(ch) for ch in dst]


def _is_identity(p: Sequence[int]) -> bool:
    return all(i == v for i, v in enumerate(p))


def transpose_cost(dtype, shape: Sequence[int], perm_t: Sequence[int]) -> float:
    """Predicted seconds of x.permute(perm_t).contiguous() (0 for a no-op)."""
    if _is_identity(perm_t):
        return 0.0
    ext, perm = torch_to_c(list(shape), list(perm_t))
    return predict_time(dtype, ext, perm)


@dataclass
class ContractionPlan:
    spec: str
    a_order: str        # index order of A's matrix view (row-major)
    b_order: str
    c_order: str        # index order of the GEMM result before the final transpose
    a_perm: List[int]   # torch permute orders (identity = no transposition)
    b_perm: List[int]
    c_perm: List[int]
    m: int
    n: int
    k: int
    swap: bool          # True: the GEMM computes C'^T = B'^T A'^T (result rows = n-group)
    a_mk: bool          # A's view is [m-group, k-group] (else [k, m], read transposed)
    b_kn: bool          # B's view is [k-group, n-group] (else [n, k], read transposed)
    predicted_transpose_s: float
    candidates: int
    costs: Dict[str, float] = field(default_factory=dict)


def plan_contraction(spec: str, shape_a: Sequence[int], shape_b: Sequence[int],
                     dtype="f64") -> ContractionPlan:
    a, b, out = _parse(spec)
    dims = {}
    for s, shp in ((a, shape_a), (b, shape_b)):
        if len(s) != len(shp):
            raise ValueError("spec / shape rank mismatch")
        for ch, e in zip(s, shp):
            if dims.setdefault(ch, int(e)) != int(e):
                raise ValueError(f"extent mismatch for index {ch!r}")
    mg = [ch for ch in a if ch in out]
    ng = [ch for ch in b if ch in out]
    kg = [ch for ch in a if ch in b]

    def prod(g):
        p = 1
        for ch in g:
            p *= dims[ch]
        return p

    def orders(group, *sources):
        seen, res = set(), []
        for src in sources:
            o = "".join(ch for ch in src if ch in group)
            if o not in seen:
                seen.add(o)
                res.append(o)
        return res

    best, n_cand = None, 0
    for mo in orders(mg, a, out):
        for no in orders(ng, b, out):
            for ko in orders(kg, a, b):
                # A view: [m, k] (A' = M x K) or [k, m] (A'^T, consumed transposed)
                for a_mk in (True, False):
                    for b_kn in (True, False):
                        for swap in (False, True):
                            a_ord = mo + ko if a_mk else ko + mo
                            b_ord = ko + no if b_kn else no + ko
                            c_ord = no + mo if swap else mo + no
                            ap = _perm_to(a, a_ord)
                            bp = _perm_to(b, b_ord)
                            cp = _perm_to(c_ord, out)
                            costs = {
                                "A": transpose_cost(dtype, [dims[c] for c in a], ap),
                                "B": transpose_cost(dtype, [dims[c] for c in b], bp),
                                "C": transpose_cost(dtype, [dims[c] for c in c_ord], cp),
                            }
                            t = sum(costs.values())
                            n_cand += 1
                            if best is None or t < best.predicted_transpose_s - 1e-15:
                                best = ContractionPlan(spec, a_ord, b_ord, c_ord, ap, bp, cp,
                                                       prod(mg), prod(ng), prod(kg), swap,
                                                       a_mk, b_kn, t, 0, costs)
    best.candidates = n_cand
    return best


def contract(spec: str, A, B, plan: ContractionPlan = None, transpose_fn=None):
    """C = einsum(spec, A, B) by TTGT: library transpositions + cuBLAS GEMM.

    `transpose_fn(x, perm_t)` defaults to the library (CUDA tensors only); the
    CPU tests pass torch's permute to check the index bookkeeping alone."""
    tr = transpose_fn or transpose_tensor
    if plan is None:
        dt = "f64" if A.element_size() == 8 else "f32"
        plan = plan_contraction(spec, A.shape, B.shape, dt)
    a, b, out = _parse(spec)
    dims = {ch: e for s, x in ((a, A), (b, B)) for ch, e in zip(s, x.shape)}

    def view(x, perm):
        if _is_identity(perm):
            return x.contiguous()
        return tr(x.contiguous(), perm)

    Am = view(A, plan.a_perm)
    Bm = view(B, plan.b_perm)
    M, N, K = plan.m, plan.n, plan.k
    # A' as M x K (or the K x M storage read transposed); same for B'
    Amat = Am.reshape(M, K) if plan.a_mk else Am.reshape(K, M).t()
    Bmat = Bm.reshape(K, N) if plan.b_kn else Bm.reshape(N, K).t()
    Cm = (Bmat.t() @ Amat.t()) if plan.swap else (Amat @ Bmat)
    Cm = Cm.contiguous()
    C = Cm.reshape([dims[ch] for ch in plan.c_order])
    if _is_identity(plan.c_perm):
        return C
    return tr(C, plan.c_perm)

