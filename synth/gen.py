"""Counter-based input generator: A_bits[l] = splitmix64(seed ^ l).

Used by both the oracle tests and the CUDA path (benchmarks, parity tests).
It is NOT part of the method: the transposition is content-agnostic
(§I: a pure permutation of element positions), so the inputs
only need to be reproducible and to cover every bit pattern class (NaN
payloads, -0.0, subnormals, inf) -- uniform 64-bit patterns do.

SplitMix64 finaliser (Steele et al.), uint64 wrap-around arithmetic:
    z = x + 0x9E3779B97F4A7C15
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9
    z = (z ^ (z >> 27)) * 0x94D049BB133111EB
    return z ^ (z >> 31)
fp64 inputs take all 64 bits; fp32 inputs keep the low 32 bits.
Seeds: seed = SEED_BASE + case_id.

Two implementations of the SAME generator are provided: NumPy (host) and
torch integer ops (any device, used to fill device memory without a host
round trip). `tests/test_synth.py` checks that they agree bit for bit and
checks the published SplitMix64 self-test values.
"""
from __future__ import annotations

import numpy as np

SEED_BASE = 0x77150000

_G = 0x9E3779B97F4A7C15
_M1 = 0xBF58476D1CE4E5B9
_M2 = 0x94D049BB133111EB


def case_seed(case_id: int) -> int:
    return SEED_BASE + int(case_id)


def splitmix64_np(x: np.ndarray) -> np.ndarray:
    """SplitMix64 finaliser on a uint64 array (wrap-around arithmetic)."""
    z = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z + np.uint64(_G)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(_M1)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(_M2)
        z = z ^ (z >> np.uint64(31))
    return z


def gen_bits_np(seed: int, start: int, count: int) -> np.ndarray:
    """uint64 bits for linear indices [start, start+count)."""
    l = np.arange(start, start + count, dtype=np.uint64)
    return splitmix64_np(np.uint64(seed) ^ l)


def gen_tensor_np(seed: int, n_elems: int, elem_bytes: int, start: int = 0,
                  mode: str = "splitmix") -> np.ndarray:
    """Flat host tensor of `n_elems` elements as uint32 (fp32) / uint64 (fp64) bits.

    mode="splitmix": A_bits[l] = splitmix64(seed ^ l)
    mode="index":    A_bits[l] = l (index encoding, for debugging / closed forms)
    """
    if mode == "index":
        bits = np.arange(start, start + n_elems, dtype=np.uint64)
    else:
        bits = gen_bits_np(seed, start, n_elems)
    if elem_bytes == 8:
        return bits
    if elem_bytes == 4:
        return (bits & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    raise ValueError("elem_bytes must be 4 or 8")


def _i64(v: int) -> int:
    """uint64 constant -> the int64 with the same bit pattern."""
    v &= (1 << 64) - 1
    return v - (1 << 64) if v >= (1 << 63) else v


def _lsr(t, k: int):
    """Logical shift right on int64 tensors (torch's >> is arithmetic)."""
    return (t >> k) & ((1 << (64 - k)) - 1)


def gen_tensor_torch(seed: int, n_elems: int, elem_bytes: int, device="cpu",
                     start: int = 0, mode: str = "splitmix", chunk: int = 1 << 26):
    """Same generator as gen_tensor_np, computed with torch int64 ops on `device`.

    Returns a flat float32/float64 tensor holding the generated bit patterns
    (viewed, never converted).  Generated in chunks to bound temporaries.
    """
    import torch

    out_dtype = torch.float64 if elem_bytes == 8 else torch.float32
    out = torch.empty(n_elems, dtype=out_dtype, device=device)
    ob = out.view(torch.int64) if elem_bytes == 8 else out.view(torch.int32)
    g, m1, m2 = _i64(_G), _i64(_M1), _i64(_M2)
    s = _i64(seed)
    for c0 in range(0, n_elems, chunk):
        c1 = min(n_elems, c0 + chunk)
        l = torch.arange(start + c0, start + c1, dtype=torch.int64, device=device)
        if mode == "index":
            z = l
        else:
            z = torch.bitwise_xor(l, s)
            z = z + g
            z = torch.bitwise_xor(z, _lsr(z, 30)) * m1
            z = torch.bitwise_xor(z, _lsr(z, 27)) * m2
            z = torch.bitwise_xor(z, _lsr(z, 31))
        if elem_bytes == 8:
            ob[c0:c1] = z
        else:
            lo = z & 0xFFFFFFFF
            lo = torch.where(lo >= (1 << 31), lo - (1 << 32), lo)
            ob[c0:c1] = lo.to(torch.int32)
        del z, l
    return out


def gen_at_np(seed: int, idx, elem_bytes: int, mode: str = "splitmix") -> np.ndarray:
    """Generator values at arbitrary linear indices (for sampled checks)."""
    l = np.asarray(idx, dtype=np.uint64)
    bits = l.copy() if mode == "index" else splitmix64_np(np.uint64(seed) ^ l)
    if elem_bytes == 8:
        return bits
    return (bits & np.uint64(0xFFFFFFFF)).astype(np.uint32)
