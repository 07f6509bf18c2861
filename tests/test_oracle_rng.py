"""Pins for oracle C1 (Philox4x32-10) and C2 (draw word, range map).  CPU only.

C1 is pinned to the Random123 known-answer vectors (tests/golden/philox_kat.txt) and to
an independent implementation: the CUDA toolkit's curand_Philox4x32_10, compiled for the
host (tests/pins/curand_philox_ref.cu).  C2's range map is pinned by its inverse
(interval boundaries) and closed forms, not by retyping the product formula.
"""
import os
import shutil
import subprocess

import numpy as np
import pytest

from oracle import oracle as O

HERE = os.path.dirname(os.path.abspath(__file__))


def _kat():
    rows = []
    for line in open(os.path.join(HERE, "golden", "philox_kat.txt")):
        if line.startswith("#") or not line.strip():
            continue
        w = [int(x, 16) for x in line.split()]
        rows.append((w[:4], w[4:6], w[6:10]))
    return rows


def test_philox_known_answers():
    for ctr, key, out in _kat():
        assert O.philox4x32_10(ctr, key) == out


@pytest.fixture(scope="module")
def curand_ref(tmp_path_factory):
    nvcc = shutil.which("nvcc") or "/usr/local/cuda/bin/nvcc"
    if not os.path.exists(nvcc):
        pytest.skip("nvcc not available to build the curand reference")
    exe = str(tmp_path_factory.mktemp("curand") / "curand_ref")
    subprocess.check_call([nvcc, "-O2", "-Wno-deprecated-gpu-targets", "-o", exe,
                           os.path.join(HERE, "pins", "curand_philox_ref.cu")])

    def run(ctr_key: np.ndarray) -> np.ndarray:
        r = subprocess.run([exe], input=np.ascontiguousarray(ctr_key, dtype=np.uint32).tobytes(),
                           capture_output=True, check=True).stdout
        return np.frombuffer(r, dtype=np.uint32).reshape(-1, 4)
    return run


def test_philox_matches_curand(curand_ref):
    rng = np.random.default_rng(12345)
    ck = rng.integers(0, 2**32, size=(200_000, 6), dtype=np.uint64).astype(np.uint32)
    ck[:1000, :4] = np.arange(4000, dtype=np.uint32).reshape(1000, 4)   # structured counters
    assert np.array_equal(O.philox4x32_10_many(ck), curand_ref(ck))


def test_draw_word_packs_philox_x_y(curand_ref):
    """u = y << 32 | x of Philox(ctr=(t, v, h, b), key=(lo32 seed, hi32 seed))."""
    seed = 0x0123456789ABCDEF
    cases = [(0, 0, 0, 0), (3, 77, 2, 9), (31, 2**31 - 1, 1, 2**32 - 1), (24, 123456789, 0, 5)]
    ck = np.array([[t, v, h, b, seed & 0xFFFFFFFF, seed >> 32] for t, v, h, b in cases], dtype=np.uint32)
    ref = curand_ref(ck)
    for (t, v, h, b), r in zip(cases, ref):
        assert O.draw_word(t, v, h, b, seed) == (int(r[1]) << 32) | int(r[0])


def test_randint_closed_forms():
    M = 2**64 - 1
    for j in [0, 1, 2, 6, 14, 1000, 2**31 - 1, 2**32, 2**40 + 17, 2**62]:
        assert O.randint(0, j) == 0
        assert O.randint(M, j) == j                       # top of the range maps to j
    for k in range(0, 63):                                # j + 1 = 2^k: the top k bits of u
        for u in [0, 1, 0xDEADBEEFCAFEBABE, M, 1 << 63, (1 << 63) - 1]:
            assert O.randint(u, (1 << k) - 1) == (u >> (64 - k) if k else 0)
    assert O.randint(1 << 63, 2**31 - 1) == 2**30         # midpoint of [0, 2^31)


def test_randint_interval_boundaries():
    """randint(u, j) = r exactly on u in [ceil(r 2^64/(j+1)), ceil((r+1) 2^64/(j+1)))."""
    rng = np.random.default_rng(7)
    for _ in range(2000):
        j = int(rng.integers(1, 2**40))
        r = int(rng.integers(1, j + 1))
        lo = -((-r * 2**64) // (j + 1))                  # ceil
        assert O.randint(lo, j) == r
        assert O.randint(lo - 1, j) == r - 1
