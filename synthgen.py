"""Seeded synthetic input generators shared by the oracle tests and the bench.

This module holds NO arithmetic of the method (no partitioning, no kernel
formula).  It only turns (seed, array_id, index) into reproducible numbers with
a counter-based hash, so that the CPU oracle (``oracle/``) and the CUDA path
(``paper_conf_icpp_shenvms15_b200``) can be fed identical inputs.  The CUDA
library implements the same generator on the device (``mm_fill_uniform``);
``tests/test_gpu_parity.py`` checks the two bit for bit.

Generator:
    h = splitmix64(seed ^ (array_id << 48) ^ index)
    u = (h >> 40) * 2**-24                       # 24-bit, exact in float32
    x = float32(lo) + float32(hi - lo) * u        # two float32 roundings, this order
    k = lo_int + ((h >> 40) % span)              # integer variant

Workload shapes follow the paper (PAPER.md P311, P319, P473) and BASELINE.json
configs; DESIGN.md states the recipe per app.
"""
from __future__ import annotations

import numpy as np

SEED = 20150901  # BASELINE.md §2 (the paper's conference month)

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_C0 = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on a uint64 array (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = x + _C0
        z = (z ^ (z >> np.uint64(30))) * _C1
        z = (z ^ (z >> np.uint64(27))) * _C2
        return z ^ (z >> np.uint64(31))


def _hash24(seed: int, array_id: int, start: int, count: int) -> np.ndarray:
    idx = np.arange(start, start + count, dtype=np.uint64)
    key = np.uint64((seed ^ (array_id << 48)) & 0xFFFFFFFFFFFFFFFF)
    return splitmix64(idx ^ key) >> np.uint64(40)


def uniform(n: int, array_id: int, lo: float, hi: float, seed: int = SEED,
            start: int = 0, chunk: int = 1 << 24) -> np.ndarray:
    """float32 array x[i] = lo + (hi-lo)*u(i), i in [start, start+n)."""
    out = np.empty(n, dtype=np.float32)
    lo32 = np.float32(lo)
    span32 = np.float32(np.float32(hi) - np.float32(lo))
    scale = np.float32(2.0 ** -24)
    for s in range(0, n, chunk):
        m = min(chunk, n - s)
        u = _hash24(seed, array_id, start + s, m).astype(np.float32) * scale
        out[s:s + m] = lo32 + span32 * u
    return out


def integers(n: int, array_id: int, lo: int, hi: int, seed: int = SEED,
             start: int = 0) -> np.ndarray:
    """int64 array in [lo, hi] inclusive: lo + (h24 % (hi-lo+1))."""
    span = np.uint64(hi - lo + 1)
    h = _hash24(seed, array_id, start, n)
    return (h % span).astype(np.int64) + lo


def constant(n: int, value: float) -> np.ndarray:
    return np.full(n, value, dtype=np.float32)


# ---------------------------------------------------------------------------
# Per-app recipes. array ids are fixed per role so
# the device generator can reproduce any sub-range in place.
# ---------------------------------------------------------------------------
AID_STREAM_A, AID_STREAM_B, AID_STREAM_C = 1, 2, 3
AID_HOT_T, AID_HOT_P = 11, 12
AID_BS_S, AID_BS_X, AID_BS_T = 21, 22, 23
AID_MM_A, AID_MM_B = 31, 32
AID_CHOL_L, AID_CHOL_S = 41, 42


def stream_random(n: int, seed: int = SEED):
    """STREAM random-init variant: a, b, c ~ U[-1, 1)."""
    return (uniform(n, AID_STREAM_A, -1.0, 1.0, seed),
            uniform(n, AID_STREAM_B, -1.0, 1.0, seed),
            uniform(n, AID_STREAM_C, -1.0, 1.0, seed))


def stream_canonical(n: int):
    """STREAM canonical init after its pre-loop doubling: a=2, b=2, c=0."""
    return constant(n, 2.0), constant(n, 2.0), constant(n, 0.0)


def hotspot(rows: int, cols: int, seed: int = SEED):
    """T0 = 323.15 + 20u K, P = 1e-3 u (SURVEY §8(c) c9 input recipe)."""
    n = rows * cols
    t = uniform(n, AID_HOT_T, 323.15, 343.15, seed).reshape(rows, cols)
    p = uniform(n, AID_HOT_P, 0.0, 1e-3, seed).reshape(rows, cols)
    return t, p


def blackscholes(n: int, seed: int = SEED):
    """NVIDIA-SDK ranges: S in [5,30), X in [1,100), T in [0.25,10)."""
    return (uniform(n, AID_BS_S, 5.0, 30.0, seed),
            uniform(n, AID_BS_X, 1.0, 100.0, seed),
            uniform(n, AID_BS_T, 0.25, 10.0, seed))


def matmul_uniform(m: int, k: int, n: int, seed: int = SEED):
    a = uniform(m * k, AID_MM_A, 0.0, 1.0, seed).reshape(m, k)
    b = uniform(k * n, AID_MM_B, 0.0, 1.0, seed).reshape(k, n)
    return a, b


def matmul_integer(m: int, k: int, n: int, seed: int = SEED):
    """Integer-valued inputs in {-4..4}: every partial sum exact in fp32."""
    a = integers(m * k, AID_MM_A, -4, 4, seed).astype(np.float32).reshape(m, k)
    b = integers(k * n, AID_MM_B, -4, 4, seed).astype(np.float32).reshape(k, n)
    return a, b


def cholesky_exact_factor(n: int, band: int = 4, seed: int = SEED):
    """L0 lower-triangular integer, diag in [32,64], off-diagonals in {-1,0,1}
    within ``band`` of the diagonal; A = L0 L0^T (exact integer arithmetic,
    entries far below 2**24).  Returns (A float32, L0 float32)."""
    i = np.arange(n)
    L = np.zeros((n, n), dtype=np.int64)
    L[i, i] = integers(n, AID_CHOL_L, 32, 64, seed)
    for d in range(1, band + 1):
        off = integers(n - d, AID_CHOL_L + 100 + d, -1, 1, seed)
        L[i[d:], i[:-d]] = off
    Lf = L.astype(np.float64)
    A = (Lf @ Lf.T).astype(np.int64)  # integer input construction (not the method); every
    # product and partial sum is an integer far below 2**53, so FP64 BLAS is exact
    assert np.abs(A).max() < 2 ** 24
    return A.astype(np.float32), L.astype(np.float32)


def spd_random(n: int, seed: int = SEED):
    """A = (S + S^T)/2 + n I with S ~ U[0,1) (diagonally dominant SPD)."""
    s = uniform(n * n, AID_CHOL_S, 0.0, 1.0, seed).reshape(n, n).astype(np.float64)
    a = (s + s.T) * 0.5 + n * np.eye(n)
    return a.astype(np.float32)


AID_NB_P, AID_NB_V = 51, 52


def nbody(n: int, seed: int = SEED):
    """Positions U[-1,1)^3 with masses U[0.5,1) (w), velocities U[-0.01,0.01)^3
    with w = 0; (n, 4) float32 each."""
    p = uniform(4 * n, AID_NB_P, -1.0, 1.0, seed).reshape(n, 4)
    m = uniform(n, AID_NB_P + 100, 0.5, 1.0, seed)
    p[:, 3] = m
    v = uniform(4 * n, AID_NB_V, -0.01, 0.01, seed).reshape(n, 4)
    v[:, 3] = 0.0
    return p, v
