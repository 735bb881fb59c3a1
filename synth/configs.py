"""Workload catalogue (shapes, permutations, case ids) for BASELINE.json's configs.

Conventions (readings R1/R2): extents[0] is the fastest-varying index
(PAPER.md L284-286 footnote, MATLAB/Fortran notation); perm[i] = j means output
dimension i is input dimension j (§VI).

Shapes follow SURVEY.md Appendix A (a synthetic re-creation: the upstream TTC
57-case list [PAPER.md L1495-1499, ref 12] is not available offline, so it is
never labelled as the upstream list).  Holds no transposition arithmetic.
"""
from __future__ import annotations

import itertools
from dataclasses import dataclass
from typing import List, Tuple


@dataclass(frozen=True)
class Case:
    case_id: int
    extents: Tuple[int, ...]
    perm: Tuple[int, ...]
    elem_bytes: int
    group: str

    @property
    def n_elems(self) -> int:
        n = 1
        for e in self.extents:
            n *= e
        return n

    @property
    def alg_bytes(self) -> int:
        """Algorithmic traffic 2*N*s."""
        return 2 * self.n_elems * self.elem_bytes

    def label(self) -> str:
        ext = "x".join(str(e) for e in self.extents)
        return f"{self.case_id}:{ext}:{''.join(str(p) for p in self.perm)}"


def _p(s: str) -> Tuple[int, ...]:
    return tuple(int(c) for c in s.split())


# ---- config 1: rank-4 fp64 16^4, all 24 perms (lexicographic) -------------------
def config1() -> List[Case]:
    return [Case(1001 + k, (16, 16, 16, 16), tuple(p), 8, "c1-16^4")
            for k, p in enumerate(itertools.permutations(range(4)))]


# ---- config 2: TTC-like 57-case suite, fp64, 26,214,400 elements each ------------
TTC_SUITE = [
    # rank, profiles (P1, P2, P3), perms
    (2, [(5120, 5120), (20480, 1280), (1280, 20480)], ["1 0"]),
    (3, [(320, 320, 256), (1280, 80, 256), (320, 80, 1024)],
     ["0 2 1", "1 0 2", "2 1 0"]),
    (4, [(80, 64, 80, 64), (320, 16, 80, 64), (80, 16, 80, 256)],
     ["0 3 2 1", "2 1 3 0", "2 0 3 1", "1 0 3 2", "3 2 1 0"]),
    (5, [(32, 32, 25, 32, 32), (128, 8, 25, 32, 32), (32, 8, 25, 32, 128)],
     ["0 4 2 1 3", "3 2 1 4 0", "2 0 4 1 3", "1 3 0 4 2", "4 3 2 1 0"]),
    (6, [(16, 20, 16, 20, 16, 16), (80, 4, 16, 20, 16, 16), (16, 4, 16, 20, 16, 80)],
     ["0 3 2 5 4 1", "3 2 0 5 1 4", "2 0 4 1 5 3", "3 2 5 1 0 4", "5 4 3 2 1 0"]),
]


def config2() -> List[Case]:
    out, cid = [], 2001
    for _rank, profiles, perms in TTC_SUITE:
        for ps in perms:
            for prof in profiles:
                out.append(Case(cid, tuple(prof), _p(ps), 8, "c2-ttc57"))
                cid += 1
    return out


# ---- config 3: CCSD(T)-style rank-6 fp64 ----------------------------------------
CCSD_SHAPES = [(16,) * 6, (24,) * 6, (32, 32, 32, 16, 16, 16), (48, 48, 48, 16, 16, 16),
               (72, 72, 16, 16, 16, 16)]
CCSD_PERMS = ["0 2 5 1 4 3", "0 2 1 3 5 4", "0 1 2 5 4 3",      # matching FVI
              "4 1 2 5 3 0", "3 4 5 0 1 2", "5 4 3 2 1 0", "2 1 0 5 4 3", "1 0 2 4 3 5"]


def config3() -> List[Case]:
    out, cid = [], 3001
    for sh in CCSD_SHAPES:
        for ps in CCSD_PERMS:
            out.append(Case(cid, sh, _p(ps), 8, "c3-ccsdt"))
            cid += 1
    return out


# ---- config 4: rank-3 fp32, small FVI ---------------------------------------------
SMALL_FVI_N0 = [2, 3, 4, 5, 8]
SMALL_FVI_PERMS = ["0 2 1", "2 1 0", "1 0 2", "1 2 0", "2 0 1"]


def config4(big: int = 4096) -> List[Case]:
    out, cid = [], 4001
    for n0 in SMALL_FVI_N0:
        for ps in SMALL_FVI_PERMS:
            out.append(Case(cid, (n0, big, big), _p(ps), 4, "c4-smallfvi"))
            cid += 1
    return out


# ---- config 5: 8 GiB rank-5 fp32, sharded on an outer index ------------------------
SHARD_EXTENTS = (64, 64, 64, 64, 128)
SHARD_PERMS = ["3 2 1 0 4", "1 0 3 2 4", "4 3 2 1 0", "0 4 2 1 3", "2 0 1 4 3"]


def config5() -> List[Case]:
    return [Case(5001 + k, SHARD_EXTENTS, _p(ps), 4, "c5-8GiB")
            for k, ps in enumerate(SHARD_PERMS)]


# ---- paper workloads (Fig 5) -----
def sweep720(extent: int, elem_bytes: int = 8, base_id: int = 6000) -> List[Case]:
    return [Case(base_id + k, (extent,) * 6, tuple(p), elem_bytes, f"720-{extent}^6")
            for k, p in enumerate(itertools.permutations(range(6)))]


def fig13(elem_bytes: int = 8) -> List[Case]:
    return [Case(7000 + k, (e,) * 4, (0, 2, 1, 3), elem_bytes, "fig13")
            for k, e in enumerate([15, 16, 31, 32, 63, 64, 127, 128])]


def fig5_case() -> Case:
    return Case(7100, (27,) * 5, (4, 1, 2, 0, 3), 8, "fig5")


def scaled(case: Case, max_elems: int) -> Case:
    """Shrink a case's extents (keeping rank, perm and odd/even structure roughly)
    until it has <= max_elems elements; used for oracle-sized parity runs that
    still span several tiles and a ragged tail."""
    ext = list(case.extents)
    while True:
        n = 1
        for e in ext:
            n *= e
        if n <= max_elems:
            break
        k = max(range(len(ext)), key=lambda i: ext[i])
        ext[k] = max(1, (ext[k] * 2) // 3)
    return Case(case.case_id, tuple(ext), case.perm, case.elem_bytes, case.group + "-scaled")


def all_configs() -> dict:
    return {"c1": config1(), "c2": config2(), "c3": config3(), "c4": config4(),
            "c5": config5()}
