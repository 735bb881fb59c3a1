"""Pins for the oracle (CPU only).  Each test ties oracle/ to something other
than itself: closed forms, invariants, textbook special cases, library
routines, brute force, hand-derived vectors and independently computed digests.
A plausible oracle bug (swapped stride roles, perm read in the wrong direction,
an off-by-one in the odometer, a truncated element width) fails at least one.
"""
import hashlib
import itertools
import os
import random

import numpy as np
import pytest

import oracle
from synth import gen_tensor_np, case_seed

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _inv(p):
    q = [0] * len(p)
    for i, j in enumerate(p):
        q[j] = i
    return q


def _rand_case(rng, max_rank=6, max_ext=7):
    d = rng.randint(1, max_rank)
    ext = [rng.randint(1, max_ext) for _ in range(d)]
    perm = list(range(d))
    rng.shuffle(perm)
    return ext, perm


def _numpy_transpose(A, ext, perm):
    """Library-routine pin: NumPy works in C order (last axis fastest), so the
    FVI-first tensor with extents n is the NumPy array of shape n[::-1], and
    output dim i (= input dim perm[i]) becomes NumPy axis d-1-i."""
    d = len(ext)
    axes = [d - 1 - perm[d - 1 - a] for a in range(d)]
    return np.ascontiguousarray(np.transpose(A.reshape(ext[::-1]), axes)).ravel()


# --- closed form: identity ---------------------------------------------------------
@pytest.mark.parametrize("eb", [4, 8])
def test_identity_returns_A(eb):
    rng = random.Random(1)
    for _ in range(20):
        ext, _ = _rand_case(rng)
        A = gen_tensor_np(7, int(np.prod(ext)), eb)
        B = oracle.transpose(A, ext, list(range(len(ext))))
        assert np.array_equal(A, B)


# --- invariant: inverse --------------------------------------------------------------
def test_inverse_roundtrip():
    rng = random.Random(2)
    for _ in range(100):
        ext, perm = _rand_case(rng)
        A = gen_tensor_np(11, int(np.prod(ext)), 8)
        B = oracle.transpose(A, ext, perm)
        C = oracle.transpose(B, oracle.out_extents(ext, perm), _inv(perm))
        assert np.array_equal(A, C), (ext, perm)


# --- invariant: composition ----------------------------------------------------------
def test_composition():
    rng = random.Random(3)
    for _ in range(100):
        ext, p = _rand_case(rng)
        q = list(range(len(ext)))
        rng.shuffle(q)
        A = gen_tensor_np(13, int(np.prod(ext)), 4)
        B = oracle.transpose(A, ext, p)
        C = oracle.transpose(B, oracle.out_extents(ext, p), q)
        pq = [p[q[i]] for i in range(len(ext))]
        D = oracle.transpose(A, ext, pq)
        assert np.array_equal(C, D), (ext, p, q)


# --- special case: 2-D is the textbook matrix transpose -----------
@pytest.mark.parametrize("n0,n1", [(1, 1), (2, 3), (5, 7), (32, 33), (64, 17)])
def test_2d_is_matrix_transpose(n0, n1):
    A = gen_tensor_np(17, n0 * n1, 8)
    B = oracle.transpose(A, [n0, n1], [1, 0])
    for i0 in range(n0):
        for i1 in range(n1):
            assert B[i1 + n1 * i0] == A[i0 + n0 * i1]


# --- library routine: NumPy transpose --------------------------------------------------
@pytest.mark.parametrize("eb", [4, 8])
def test_matches_numpy(eb):
    rng = random.Random(4)
    for _ in range(300):
        ext, perm = _rand_case(rng, max_rank=7, max_ext=6)
        A = gen_tensor_np(19, int(np.prod(ext)), eb)
        assert np.array_equal(oracle.transpose(A, ext, perm), _numpy_transpose(A, ext, perm))


# --- brute force: dict over every multi-index -------------------------------------------
def _brute(A, ext, perm):
    d = len(ext)
    sA = [1] * d
    for k in range(1, d):
        sA[k] = sA[k - 1] * ext[k - 1]
    m = [ext[p] for p in perm]
    table = {}
    for idx in itertools.product(*[range(e) for e in ext]):
        out_idx = tuple(idx[perm[i]] for i in range(d))
        table[out_idx] = A[sum(idx[k] * sA[k] for k in range(d))]
    # read B back in output order, o0 fastest
    B = []
    for o in itertools.product(*[range(e) for e in reversed(m)]):
        B.append(table[tuple(reversed(o))])
    return np.array(B, dtype=A.dtype)


def test_brute_force_rank_le4():
    ext_all = [2, 3, 4, 5]
    for d in range(1, 5):
        ext = ext_all[:d]
        A = gen_tensor_np(23, int(np.prod(ext)), 8)
        for perm in itertools.permutations(range(d)):
            assert np.array_equal(oracle.transpose(A, ext, perm), _brute(A, ext, list(perm)))


def test_brute_force_all_720_rank6():
    ext = [2, 2, 2, 2, 3, 2]
    A = gen_tensor_np(29, int(np.prod(ext)), 4)
    for perm in itertools.permutations(range(6)):
        assert np.array_equal(oracle.transpose(A, ext, perm), _brute(A, ext, list(perm)))


def test_pure_python_loop_agrees():
    rng = random.Random(5)
    for _ in range(50):
        ext, perm = _rand_case(rng, max_rank=5, max_ext=5)
        A = gen_tensor_np(31, int(np.prod(ext)), 8)
        assert np.array_equal(oracle.transpose(A, ext, perm),
                              np.array(oracle.transpose_py(list(A), ext, perm), dtype=A.dtype))


# --- exactly once + index-encoding closed form ------------------------------------------
def test_exactly_once_and_source_index():
    rng = random.Random(6)
    for _ in range(60):
        ext, perm = _rand_case(rng)
        n = int(np.prod(ext))
        A = np.arange(n, dtype=np.uint64)
        B = oracle.transpose(A, ext, perm)
        assert np.array_equal(np.sort(B), A)          # every element written exactly once
        linA = oracle.source_index(ext, perm, np.arange(n))
        assert np.array_equal(B.astype(np.int64), linA)  # B_bits[lin_B] = lin_A(lin_B)


def test_counter_array_all_ones():
    ext, perm = [3, 4, 2, 5], [2, 0, 3, 1]
    n = int(np.prod(ext))
    B = oracle.transpose(np.arange(n, dtype=np.uint64), ext, perm)
    counts = np.bincount(B.astype(np.int64), minlength=n)
    assert (counts == 1).all()


# --- bit patterns survive (NaN payloads, -0.0, subnormals, inf) ---------------------------
def test_bit_patterns_preserved():
    special = np.array([0x7FF8000000000001, 0xFFF0000000000000, 0x8000000000000000,
                        0x0000000000000001, 0x7FF0000000000000, 0x7FF4DEADBEEF0001],
                       dtype=np.uint64)
    A = np.tile(special, 4)                                  # 24 elements
    B = oracle.transpose(A.view(np.float64), [4, 6], [1, 0])
    assert np.array_equal(np.sort(B.view(np.uint64)), np.sort(A))
    A32 = np.array([0x7FC00001, 0xFF800000, 0x80000000, 0x00000001, 0x7F800000, 0x7FA0BEEF],
                   dtype=np.uint32)
    B32 = oracle.transpose(np.tile(A32, 4).view(np.float32), [6, 4], [1, 0])
    assert np.array_equal(np.sort(B32.view(np.uint32)), np.sort(np.tile(A32, 4)))


# --- threading only splits the outermost index ---------------------------------------------
def test_threads_agree():
    ext, perm = [17, 5, 9, 13], [3, 1, 0, 2]
    A = gen_tensor_np(37, int(np.prod(ext)), 8)
    ref = oracle.transpose(A, ext, perm, threads=1)
    for t in (2, 3, 8, 64):
        assert np.array_equal(oracle.transpose(A, ext, perm, threads=t), ref)


def test_bad_args_rejected():
    A = np.zeros(6, dtype=np.uint64)
    with pytest.raises(ValueError):
        oracle.transpose(A, [2, 3], [0, 0])
    with pytest.raises(ValueError):
        oracle.transpose(A, [2, 3], [0, 2])


# --- golden fixtures ------------------------------------------------------------------------
def _read_golden(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line)
    return rows


def test_tiny_index_encoding_vectors():
    rows = _read_golden("tiny_index_encoding.txt")
    assert len(rows) == 4
    for row in rows:
        e, p, b = [s.split() for s in row.split("|")]
        ext, perm, expect = [int(x) for x in e], [int(x) for x in p], [int(x) for x in b]
        A = np.arange(int(np.prod(ext)), dtype=np.uint64)
        assert oracle.transpose(A, ext, perm).tolist() == expect


def test_survey_config1_digests():
    rows = _read_golden("survey_c1_digests.txt")
    assert len(rows) == 24
    ext = [16, 16, 16, 16]
    for row in rows:
        f = row.split()
        case, perm, digest = int(f[0]), [int(x) for x in f[1:5]], f[5]
        A = gen_tensor_np(case_seed(case), 16 ** 4, 8)
        B = oracle.transpose(A, ext, perm)
        got = hashlib.sha256(B.astype("<u8").tobytes()).hexdigest()[:16]
        assert got == digest, (case, perm)
