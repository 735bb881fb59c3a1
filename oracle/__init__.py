"""TTLG oracle -- TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously correct CPU implementation of the transposition
B[rho(i0..id-1)] <- A[i0..id-1] (§I).  Only `tests/`,
`__graft_entry__.smoke()` and `bench.py`'s cpu_baseline / `--impl reference`
legs may import this package.  The product package
(`paper_conf_ipps_veduradasskhpkn18_b200`) never imports it and shares no
code with it.

- `transpose(...)`      : the C d-nested loop (oracle.c), optionally threaded
                          over the outermost input index.
- `transpose_py(...)`   : the same definition as a pure-Python loop (tiny cases).
- `source_index(...)`   : lin_B -> lin_A, the definition read backwards, for
                          sampled checks at full sizes.

Conventions: extents[0] is the fastest-varying index; perm[i] = j means output
dim i is input dim j (readings R1, R2).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None


def build_oracle(force: bool = False) -> str:
    """Compile oracle.c with gcc -O2 (no blocking, no intrinsics)."""
    src = os.path.join(_HERE, "oracle.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-pthread",
                               "-o", _SO, src])
    return _SO


def _load():
    global _lib
    if _lib is None:
        build_oracle()
        lib = ctypes.CDLL(_SO)
        lib.oracle_transpose.argtypes = [ctypes.c_int, ctypes.c_int,
                                         ctypes.POINTER(ctypes.c_int64),
                                         ctypes.POINTER(ctypes.c_int32),
                                         ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int]
        lib.oracle_transpose.restype = ctypes.c_int
        lib.oracle_source_index.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_int64),
                                            ctypes.POINTER(ctypes.c_int32),
                                            ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64]
        lib.oracle_source_index.restype = ctypes.c_int
        lib.oracle_transpose_strided.argtypes = [
            ctypes.c_int, ctypes.c_int, ctypes.POINTER(ctypes.c_int64),
            ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_int64),
            ctypes.POINTER(ctypes.c_int64), ctypes.c_void_p, ctypes.c_int64,
            ctypes.c_void_p, ctypes.c_int64]
        lib.oracle_transpose_strided.restype = ctypes.c_int
        _lib = lib
    return _lib


def out_extents(extents: Sequence[int], perm: Sequence[int]):
    """B's extents: m[i] = n[perm[i]]."""
    return tuple(int(extents[p]) for p in perm)


def _arrs(extents, perm):
    d = len(extents)
    ext = (ctypes.c_int64 * d)(*[int(e) for e in extents])
    pr = (ctypes.c_int32 * d)(*[int(p) for p in perm])
    return ext, pr


def transpose(A: np.ndarray, extents: Sequence[int], perm: Sequence[int],
              threads: int = 1) -> np.ndarray:
    """B = T(A) by the C loop. A: flat uint32/uint64 (or float32/float64) array."""
    A = np.ascontiguousarray(A).reshape(-1)
    if A.dtype.itemsize not in (4, 8):
        raise ValueError("element size must be 4 or 8 bytes")
    n = 1
    for e in extents:
        n *= int(e)
    if A.size != n:
        raise ValueError("A size does not match extents")
    B = np.empty_like(A)
    ext, pr = _arrs(extents, perm)
    rc = _load().oracle_transpose(A.dtype.itemsize, len(extents), ext, pr,
                                  A.ctypes.data, B.ctypes.data, int(threads))
    if rc != 0:
        raise ValueError("oracle: invalid rank/extents/perm")
    return B


def transpose_strided(A: np.ndarray, B: np.ndarray, extents: Sequence[int],
                      perm: Sequence[int], in_strides: Sequence[int],
                      out_strides: Sequence[int], a_off: int = 0, b_off: int = 0) -> np.ndarray:
    """Sub-tensor transposition into B in place (only the addressed positions
    change): B[b_off + sum_i o_i out_strides[i]] = A[a_off + sum_k i_k in_strides[k]],
    o_i = i_{perm[i]}.  A, B: flat contiguous arrays of the same item size."""
    if not (A.flags.c_contiguous and B.flags.c_contiguous) or A.dtype.itemsize != B.dtype.itemsize:
        raise ValueError("A and B must be contiguous with the same element size")
    d = len(extents)
    span_a = a_off + sum((int(e) - 1) * int(s) for e, s in zip(extents, in_strides))
    span_b = b_off + sum((int(extents[p]) - 1) * int(s) for p, s in zip(perm, out_strides))
    if span_a >= A.size or span_b >= B.size or a_off < 0 or b_off < 0:
        raise ValueError("strided box exceeds the buffers")
    ext, pr = _arrs(extents, perm)
    sa = (ctypes.c_int64 * d)(*[int(x) for x in in_strides])
    sb = (ctypes.c_int64 * d)(*[int(x) for x in out_strides])
    rc = _load().oracle_transpose_strided(A.dtype.itemsize, d, ext, pr, sa, sb, A.ctypes.data,
                                          int(a_off), B.ctypes.data, int(b_off))
    if rc != 0:
        raise ValueError("oracle: invalid rank/extents/perm")
    return B


def source_index(extents: Sequence[int], perm: Sequence[int], linB,
                 threads: int = 1) -> np.ndarray:
    """For each output linear index, the input linear index it is copied from.
    threads > 1 splits the index list into contiguous pieces evaluated
    concurrently (each piece is the same C loop; ctypes releases the GIL)."""
    linB = np.ascontiguousarray(np.asarray(linB, dtype=np.int64))
    linA = np.empty_like(linB)
    ext, pr = _arrs(extents, perm)
    lib = _load()

    def piece(lo, hi):
        return lib.oracle_source_index(len(extents), ext, pr,
                                       linB.ctypes.data + 8 * lo, linA.ctypes.data + 8 * lo,
                                       hi - lo)
    n = linB.size
    threads = max(1, min(int(threads), n // 65536 or 1))
    if threads == 1:
        rcs = [piece(0, n)]
    else:
        from concurrent.futures import ThreadPoolExecutor
        cuts = [n * t // threads for t in range(threads + 1)]
        with ThreadPoolExecutor(threads) as ex:
            rcs = list(ex.map(lambda t: piece(cuts[t], cuts[t + 1]), range(threads)))
    if any(rc != 0 for rc in rcs):
        raise ValueError("oracle: invalid rank/extents/perm")
    return linA


def transpose_py(A, extents: Sequence[int], perm: Sequence[int]):
    """The d-nested loop of PAPER.md L38-42 in pure Python (tiny inputs only)."""
    d = len(extents)
    n = [int(e) for e in extents]
    sA = [1] * d
    for k in range(1, d):
        sA[k] = sA[k - 1] * n[k - 1]
    m = [n[p] for p in perm]
    sB = [1] * d
    for i in range(1, d):
        sB[i] = sB[i - 1] * m[i - 1]
    total = 1
    for e in n:
        total *= e
    B = [None] * total
    idx = [0] * d
    for _ in range(total):
        linA = sum(idx[k] * sA[k] for k in range(d))
        linB = sum(idx[perm[i]] * sB[i] for i in range(d))
        B[linB] = A[linA]
        k = 0
        while k < d:
            idx[k] += 1
            if idx[k] < n[k]:
                break
            idx[k] = 0
            k += 1
    return B
