"""The shared input generator: published SplitMix64 values, and the NumPy and
torch implementations agree bit for bit (fp32 keeps the low 32 bits)."""
import numpy as np
import pytest

from synth import splitmix64_np, gen_tensor_np, gen_tensor_torch, configs


def test_splitmix64_published_values():
    # SplitMix64 finaliser self-check values (SURVEY.md §8(c) "Input generator")
    out = splitmix64_np(np.array([0, 1], dtype=np.uint64))
    assert int(out[0]) == 0xE220A8397B1DCDAF
    assert int(out[1]) == 0x910A2DEC89025CC1


@pytest.mark.parametrize("eb", [4, 8])
@pytest.mark.parametrize("mode", ["splitmix", "index"])
def test_numpy_torch_agree(eb, mode):
    import torch
    n, start, seed = 10007, 123456789, 0x77150000 + 42
    a = gen_tensor_np(seed, n, eb, start=start, mode=mode)
    t = gen_tensor_torch(seed, n, eb, device="cpu", start=start, mode=mode, chunk=4096)
    tb = t.view(torch.int64 if eb == 8 else torch.int32).numpy()
    assert np.array_equal(tb.view(np.uint64 if eb == 8 else np.uint32), a)


def test_catalogue_shapes():
    c = configs.all_configs()
    assert len(c["c1"]) == 24 and len(c["c2"]) == 57 and len(c["c3"]) == 40
    assert len(c["c4"]) == 25 and len(c["c5"]) == 5
    for case in c["c2"]:
        assert case.n_elems == 26214400          # 200 MiB fp64 each
    for case in c["c5"]:
        assert case.n_elems == 1 << 31
    ids = [x.case_id for v in c.values() for x in v]
    assert len(ids) == len(set(ids))
    for v in c.values():
        for case in v:
            assert sorted(case.perm) == list(range(len(case.extents)))
