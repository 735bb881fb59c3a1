"""Whole-tensor parity at the FULL BASELINE sizes (VERDICT r1 "Next round" 1).

Every output element of every case is compared with the oracle, in the launch
configuration bench.py times (the auto plan of `ttlg.plan`, one
`ttlg_execute`).  Inputs are index-encoded (A_bits[l] = l, synth mode
"index"): every value is unique, so equality of the whole output with the
oracle's transposition of the same input proves that every element landed
exactly where the definition puts it -- a misplaced tile,
a dropped ragged tail or a double write cannot hide.

- configs 2, 3, 4 (57 + 40 + 25 cases, 128 MiB - 3.4 GiB): B against
  oracle.transpose(arange(N)) (the C d-nested loop, threaded over the
  outermost index);
- the paper's 720-permutation sweeps of 15^6 / 16^6 / 17^6 fp64 (every plan
  bench.py --workload 720-N times);
- config 5 (8 GiB fp32, 2^31 elements): the memory-light form of SURVEY
  §8(c): B is read back per slab of 2^28 outputs and compared with
  oracle.source_index (lin_B -> lin_A) of that slab.
"""
import os
import time

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle  # noqa: E402  (test infrastructure)
import paper_conf_ipps_veduradasskhpkn18_b200 as ttlg  # noqa: E402
from oracle.taxonomy import classify  # noqa: E402
from synth import configs, gen_tensor_torch  # noqa: E402

pytestmark = pytest.mark.gpu
DEV = "cuda:0"
CORES = max(1, len(os.sched_getaffinity(0)))
_host_idx = {}


def _uint(eb):
    return np.uint64 if eb == 8 else np.uint32


def _host_index(n, eb):
    key = (n, eb)
    if key not in _host_idx:
        _host_idx.clear()
        _host_idx[key] = np.arange(n, dtype=_uint(eb))
    return _host_idx[key]


class _Dev:
    """Device A (index-encoded) and B of one size, reused across perms."""

    def __init__(self):
        self.key = None

    def get(self, n, eb):
        if self.key != (n, eb):
            self.A = self.B = None
            torch.cuda.empty_cache()
            self.A = gen_tensor_torch(0, n, eb, device=DEV, mode="index")
            self.B = torch.empty_like(self.A)
            self.key = (n, eb)
        return self.A, self.B


_dev = _Dev()


def _check_whole(case):
    n, eb = case.n_elems, case.elem_bytes
    A, B = _dev.get(n, eb)
    p = ttlg.plan("f64" if eb == 8 else "f32", case.extents, case.perm)
    info = p.describe()
    B.view(torch.int64 if eb == 8 else torch.int32).fill_(-1)
    p.execute(A.data_ptr(), B.data_ptr(), torch.cuda.current_stream().cuda_stream)
    got = B.view(torch.int64 if eb == 8 else torch.int32).cpu().numpy().view(_uint(eb))
    exp = oracle.transpose(_host_index(n, eb), case.extents, case.perm, threads=CORES)
    if not np.array_equal(got, exp):
        bad = np.nonzero(got != exp)[0]
        pytest.fail(f"{case.label()} {info['schema']} {info['kernel']}: {bad.size} "
                    f"mismatches, first at {bad[:8].tolist()}")
    return info


@pytest.mark.parametrize("case", configs.config2(), ids=lambda c: c.label())
def test_whole_ttc57(case):
    _check_whole(case)


@pytest.mark.parametrize("case", configs.config3(), ids=lambda c: c.label())
def test_whole_ccsdt(case):
    _check_whole(case)


@pytest.mark.parametrize("case", configs.config4(), ids=lambda c: c.label())
def test_whole_smallfvi(case):
    _check_whole(case)


@pytest.mark.parametrize("e", [15, 16, 17])
def test_whole_720_sweep(e):
    """Every one of the 720 plans of the e^6 fp64 sweep."""
    t0 = time.time()
    kernels = {}
    for c in configs.sweep720(e):
        info = _check_whole(c)
        kernels[info["kernel"]] = kernels.get(info["kernel"], 0) + 1
    print(f"720-{e}: {kernels} in {time.time() - t0:.1f} s")


@pytest.mark.parametrize("case", configs.config5(), ids=lambda c: c.label())
def test_whole_8GiB_slabs(case):
    """Config 5 at full size (2^31 fp32 elements), compared slab by slab."""
    n = case.n_elems
    A, B = _dev.get(n, 4)
    p = ttlg.plan("f32", case.extents, case.perm)
    B.view(torch.int32).fill_(-1)
    p.execute(A.data_ptr(), B.data_ptr(), torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    Bi = B.view(torch.int32)
    slab = 1 << 28
    for lo in range(0, n, slab):
        hi = min(n, lo + slab)
        got = Bi[lo:hi].cpu().numpy().view(np.uint32)
        exp = oracle.source_index(case.extents, case.perm, np.arange(lo, hi, dtype=np.int64),
                                  threads=CORES)
        if not np.array_equal(got.astype(np.int64), exp):
            bad = np.nonzero(got.astype(np.int64) != exp)[0]
            pytest.fail(f"{case.label()} slab {lo}: {bad.size} mismatches, first at "
                        f"{(bad[:8] + lo).tolist()}")


def _scaled_all():
    out = []
    for grp in ("c2", "c3", "c4", "c5"):
        out += [configs.scaled(c, 1 << 20) for c in configs.all_configs()[grp]]
    return out


@pytest.mark.parametrize("case", _scaled_all(), ids=lambda c: c.label())
def test_strict_schema_forced_bytes(case):
    """The strict Alg. 1 schema (oracle/taxonomy.py), forced on the product,
    gives the oracle's bytes (every forced schema must)."""
    s = classify(case.extents, case.perm)
    dt = "f64" if case.elem_bytes == 8 else "f32"
    try:
        p = ttlg.plan(dt, case.extents, case.perm, schema=s)
    except ttlg.TtlgError:
        pytest.skip("strict FMS pencil widened into one access element (OD)")
    n, eb = case.n_elems, case.elem_bytes
    A = gen_tensor_torch(0, n, eb, device=DEV, mode="index")
    B = torch.empty_like(A)
    p.execute(A.data_ptr(), B.data_ptr(), torch.cuda.current_stream().cuda_stream)
    got = B.view(torch.int64 if eb == 8 else torch.int32).cpu().numpy().view(_uint(eb))
    exp = oracle.transpose(np.arange(n, dtype=_uint(eb)), case.extents, case.perm)
    assert np.array_equal(got, exp), f"{case.label()} forced {s}"
