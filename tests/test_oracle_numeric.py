"""Pins of the numeric oracle (oracle/numeric.c) against what the paper and the
mathematics fix — closed forms, special cases, textbook values, identities and
library routines on special inputs.  CPU only."""
import math

import numpy as np
import pytest

import synthgen
from oracle import numeric as on


# ---------------------------------------------------------------- STREAM ---
@pytest.mark.parametrize("passes", [1, 2, 3, 6])
def test_stream_canonical_closed_form(passes):
    # McCalpin init a=1,b=2,c=0 then a=2a; one pass maps (a,b,c) to
    # (15a_prev, 3a_prev', ...): closed form a=2*15^k, b=6*15^(k-1), c=8*15^(k-1),
    # exact in FP32 while 15^k < 2^24 (k <= 6).  SURVEY §8(c) c7.
    n = 1000
    a, b, c = synthgen.stream_canonical(n)
    a, b, c = on.stream_run(a, b, c, passes)
    k = passes
    assert np.all(a == np.float32(2 * 15 ** k))
    assert np.all(b == np.float32(6 * 15 ** (k - 1)))
    assert np.all(c == np.float32(8 * 15 ** (k - 1)))


def test_stream_index_pin_dyadic():
    # Index-dependent dyadic a0 with few significant bits: every op is exact, so
    # one pass must give b=3a0, c=4a0, a=15a0 AT THE SAME INDEX whatever b0, c0
    # were (scale reads c not b; add writes c; triad reads the new b and c).
    n = 4099
    i = np.arange(n)
    a0 = ((i % 251) - 125).astype(np.float32) / np.float32(8.0)
    b0 = synthgen.uniform(n, 2, -1, 1)
    c0 = synthgen.uniform(n, 3, -1, 1)
    a, b, c = on.stream_run(a0, b0, c0, 1)
    assert np.array_equal(b, 3 * a0)
    assert np.array_equal(c, 4 * a0)
    assert np.array_equal(a, 15 * a0)


def test_stream_triad_single_rounding():
    # triad is one fused multiply-add (R14): for b = -s*c exactly representable
    # cancellation the result is the rounding error of s*c, not zero.
    c = np.array([1.0 + 2.0 ** -23], np.float32)
    b = np.array([-3.0 - 3.0 * 2.0 ** -23], np.float64).astype(np.float32)
    a = np.zeros(1, np.float32)
    on.stream_triad(a, b, c, 3.0)
    exact = 3.0 * float(c[0]) + float(b[0])
    assert a[0] == np.float32(exact)


def test_stream_fp32_overflow_bound():
    # 2*15^k exceeds FP32 max at k = 33: loops are capped at 32.
    a, b, c = synthgen.stream_canonical(4)
    a32, _, _ = on.stream_run(a, b, c, 32)
    assert np.all(np.isfinite(a32))
    a33, _, _ = on.stream_run(a, b, c, 33)
    assert np.all(np.isinf(a33))


# --------------------------------------------------------------- HotSpot ---
def test_hotspot_fixed_point_exact():
    # T == T_amb with P == 0 is an exact fixed point of the scheme (c9).
    t = np.full((17, 33), on.HOT_AMB, np.float32)
    p = np.zeros_like(t)
    out = np.empty_like(t)
    on.hotspot_rows(t, p, out)
    assert np.array_equal(out, t)


def test_hotspot_uniform_scalar_recurrence():
    # Uniform T and P: the lateral terms vanish (clamped edges included) and
    # every cell follows T <- T + sdc (P + rz1 (amb - T)); fp64 reference.
    rows, cols, iters = 9, 13, 50
    t0 = np.full((rows, cols), 330.0, np.float32)
    p = np.full((rows, cols), 7e-4, np.float32)
    out = on.hotspot_run(t0, p, iters)
    ref = 330.0
    for _ in range(iters):
        ref = ref + on.HOT_SDC * (7e-4 + on.HOT_RZ1 * (on.HOT_AMB - ref))
    assert np.all(out == out[0, 0])
    assert abs(out[0, 0] - ref) / ref < 1e-6


def test_hotspot_dense_operator_anisotropic():
    # One step equals T' = M T + b with M assembled from the physical model:
    # M = I + sdc (ry1 (S + N - 2I) + rx1 (E + W - 2I) - rz1 I), clamped
    # neighbours -> diagonal; b = sdc (P + rz1 amb).  rx1 != ry1 so a transposed
    # stencil fails.
    rows, cols = 6, 8
    coef = on.HotCoef(1.25, 0.05, 0.11, 1e-3, 80.0)
    rng = np.random.default_rng(1)
    t = (300 + 40 * rng.random((rows, cols))).astype(np.float32)
    p = (1e-3 * rng.random((rows, cols))).astype(np.float32)
    n = rows * cols
    M = np.eye(n)
    sdc, rx1, ry1, rz1, amb = (float(np.float32(v)) for v in (1.25, 0.05, 0.11, 1e-3, 80.0))
    for y in range(rows):
        for x in range(cols):
            i = y * cols + x
            for (yy, xx, cf) in ((y - 1, x, ry1), (y + 1, x, ry1), (y, x - 1, rx1), (y, x + 1, rx1)):
                j = yy * cols + xx if (0 <= yy < rows and 0 <= xx < cols) else i
                M[i, j] += sdc * cf
                M[i, i] -= sdc * cf
            M[i, i] -= sdc * rz1
    b = sdc * (p.reshape(-1).astype(np.float64) + rz1 * amb)
    ref = M @ t.reshape(-1).astype(np.float64) + b
    out = np.empty_like(t)
    on.hotspot_rows(t, p, out, coef=coef)
    assert np.max(np.abs(out.reshape(-1) - ref) / np.abs(ref)) < 2e-6


def test_hotspot_row_range_partition_invariance():
    # Computing rows [0,r) and [r,rows) separately equals the full step exactly.
    t, p = synthgen.hotspot(37, 29)
    full = np.empty_like(t)
    on.hotspot_rows(t, p, full)
    part = np.empty_like(t)
    on.hotspot_rows(t, p, part, 0, 11)
    on.hotspot_rows(t, p, part, 11, 37)
    assert np.array_equal(full, part)


@pytest.mark.parametrize("h", [1, 2, 3, 5])
def test_hotspot_block_rows_is_h_full_steps_and_reads_only_the_halo(h):
    """Temporal block: rows [r0, r1) after one block of h
    iterations equal h full-grid iterations (P319), and rows of T_in outside
    [r0-h, r1+h) are never read (poisoned with NaN)."""
    rows, cols = 29, 13
    t, p = synthgen.hotspot(rows, cols)
    full = on.hotspot_run(t, p, h)
    for r0, r1 in [(0, rows), (0, 7), (9, 17), (20, rows), (14, 15)]:
        tp = t.copy()
        tp[: max(0, r0 - h)] = np.nan
        tp[min(rows, r1 + h):] = np.nan
        out = np.full_like(t, -1.0)
        on.hotspot_block_rows(tp, p, out, r0, r1, h)
        assert np.array_equal(out[r0:r1], full[r0:r1]), (r0, r1)
        assert np.all(out[:r0] == -1.0) and np.all(out[r1:] == -1.0)


def test_hotspot_stable_over_many_iterations():
    # R15 coefficients keep the explicit scheme stable (sum of coefficients
    # < 1): after 1000 iterations the grid stays within the initial range
    # widened by the heat injected (sdc*Pmax*iters).
    t, p = synthgen.hotspot(32, 32)
    out = on.hotspot_run(t, p, 1000)
    assert np.all(np.isfinite(out))
    assert out.min() >= on.HOT_AMB - 1e-3
    assert out.max() <= t.max() + on.HOT_SDC * 1e-3 * 1000


def test_row_residual_matches_fsum():
    t0, _ = synthgen.hotspot(5, 1000)
    t1 = t0 + synthgen.uniform(5000, 99, -1e-2, 1e-2).reshape(5, 1000)
    rs = on.row_residual(t0, t1)
    for y in range(5):
        d = t1[y].astype(np.float64) - t0[y].astype(np.float64)
        ref = math.fsum(d * d)   # exact squares (float differences), correctly rounded sum
        assert abs(rs[y] - ref) <= 1e-12 * ref
    assert np.all(on.row_residual(t0, t0) == 0.0)


# ---------------------------------------------------------- BlackScholes ---
def test_cnd_within_abramowitz_stegun_bound():
    for d in np.linspace(-6, 6, 241):
        exact = 0.5 * math.erfc(-d / math.sqrt(2.0))
        assert abs(on.cnd(float(d)) - exact) < 7.5e-8


def test_blackscholes_put_call_parity():
    S, X, T = synthgen.blackscholes(20000)
    call, put = on.blackscholes(S, X, T)
    lhs = call - put
    rhs = S.astype(np.float64) - X.astype(np.float64) * np.exp(-on.BS_R * T.astype(np.float64))
    scale = np.maximum(S, X).astype(np.float64)
    assert np.max(np.abs(lhs - rhs) / scale) < 1e-13
    assert np.all(call >= -1e-12) and np.all(put >= -1e-12)


def test_blackscholes_textbook_value():
    # Hull, Options Futures & Other Derivatives, Example 15.6 [ext]:
    # S=42, X=40, r=10%, sigma=20%, T=0.5 -> c = 4.76, p = 0.81.
    S = np.array([42.0], np.float32)
    X = np.array([40.0], np.float32)
    T = np.array([0.5], np.float32)
    call, put = on.blackscholes(S, X, T, R=0.10, V=0.20)
    assert abs(call[0] - 4.76) < 5e-3
    assert abs(put[0] - 0.81) < 5e-3


# -------------------------------------------------------------- MatrixMul ---
def test_sgemm_integer_exact():
    A, B = synthgen.matmul_integer(67, 45, 38)
    ref = A.astype(np.int64) @ B.astype(np.int64)
    out = on.sgemm(A, B)
    assert np.array_equal(out.astype(np.int64), ref)


def test_sgemm_uniform_vs_library():
    A, B = synthgen.matmul_uniform(50, 70, 30)
    ref = A.astype(np.float64) @ B.astype(np.float64)
    out = on.sgemm(A, B)
    assert np.max(np.abs(out - ref) / np.abs(ref)) < 1e-7   # one fp32 rounding


def test_sgemm_row_range():
    A, B = synthgen.matmul_uniform(40, 16, 24)
    full = on.sgemm(A, B)
    part = on.sgemm(A, B, 8, 19)
    assert np.array_equal(part[8:19], full[8:19])
    assert np.all(part[:8] == 0) and np.all(part[19:] == 0)


# --------------------------------------------------------------- Cholesky ---
@pytest.mark.parametrize("n", [1, 7, 64, 129])
def test_cholesky_exact_factor(n):
    A, L0 = synthgen.cholesky_exact_factor(n)
    L = on.cholesky(A)
    assert np.array_equal(L, L0.astype(np.float64))


def test_cholesky_random_spd():
    A = synthgen.spd_random(90).astype(np.float64)
    L = on.cholesky(A)
    assert np.allclose(np.triu(L, 1), 0)
    assert np.max(np.abs(L @ L.T - A)) / np.max(np.abs(A)) < 1e-14
    assert np.max(np.abs(L - np.linalg.cholesky(A))) / np.max(np.abs(L)) < 1e-13


def test_cholesky_rejects_indefinite():
    with pytest.raises(ValueError):
        on.cholesky(np.array([[1.0, 2.0], [2.0, 1.0]]))


# ----------------------------------------------------------------- Nbody ---
def test_nbody_two_body_closed_form():
    # two bodies on the x axis: a_1 = m_2 r / (r^2 + eps2)^{3/2}, equal and
    # opposite momentum change; one step of the semi-implicit Euler integrator
    pos = np.array([[0.0, 0, 0, 2.0], [0.5, 0, 0, 3.0]], np.float32)
    vel = np.zeros((2, 4), np.float32)
    dt, eps2 = 1e-3, 1e-2
    p1, v1 = on.nbody_run(pos, vel, 1, dt, eps2)
    r = 0.5
    a0 = 3.0 * r / (r * r + eps2) ** 1.5
    a1 = -2.0 * r / (r * r + eps2) ** 1.5
    assert abs(v1[0, 0] - a0 * dt) < 1e-6 * abs(a0 * dt)
    assert abs(v1[1, 0] - a1 * dt) < 1e-6 * abs(a1 * dt)
    assert abs(p1[0, 0] - a0 * dt * dt) < 1e-9 and v1[0, 1] == 0 and v1[0, 2] == 0
    assert abs(2.0 * v1[0, 0] + 3.0 * v1[1, 0]) < 1e-9        # momentum conserved
    assert p1[0, 3] == 2.0 and p1[1, 3] == 3.0                 # masses carried


def test_nbody_single_body_at_rest_and_drift():
    p, v = on.nbody_run(np.array([[0.3, -0.2, 0.1, 1.0]], np.float32),
                        np.array([[1.0, 2.0, -1.0, 0.0]], np.float32), 5)
    # self-interaction contributes 0 (softened): uniform motion
    assert np.allclose(p[0, :3], [0.3 + 5e-3, -0.2 + 1e-2, 0.1 - 5e-3], atol=1e-7)
    assert np.array_equal(v, np.array([[1.0, 2.0, -1.0, 0.0]], np.float32))


def test_nbody_momentum_conservation_many():
    pos, vel = synthgen.nbody(300)
    p1, v1 = on.nbody_run(pos, vel, 1)
    m = pos[:, 3].astype(np.float64)
    dp = (m[:, None] * (v1[:, :3].astype(np.float64) - vel[:, :3].astype(np.float64))).sum(0)
    # sum_i m_i a_i = 0 analytically; FP32 storage of v' rounds each term
    assert np.max(np.abs(dp)) < 300 * 2.0 * 6e-8 * np.max(np.abs(v1[:, :3]))
