"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (one logical device, the Table I first choice, profiled plan): sampled
outputs against the oracle computed one by one, or properties that hold at
any size.  Seams of the kernels' tilings are part of every sample."""
import numpy as np
import pytest

import synthgen
from oracle import numeric as on

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def R(gpu):
    from paper_conf_icpp_shenvms15_b200 import mm, runner
    return mm, runner


def _bench_plan(s, mm):
    """bench.py: profile -> Table I rank -> plan of the first choice."""
    prof = s.profile(reps=2)
    best = mm.mm_rank(s.classify(), mm.mm_needs_sync(s.app))[0]
    s.fill()
    return s.plan(best, prof)


def test_blackscholes_p311_size_sampled(R):
    """SK-One BlackScholes, 80,530,632 options (P311): sampled options
    (first/last 64, float4-group and CTA seams, random) vs the FP64 oracle."""
    mm, runner = R
    n = 80530632
    rng = np.random.default_rng(1)
    idx = np.unique(np.concatenate([np.arange(64), np.arange(n - 64, n), rng.integers(0, n, 4096),
                                    np.arange(1023, 1030), np.arange(n // 2 - 3, n // 2 + 3)]))
    import torch
    with runner.session(mm.MM_APP_BLACKSCHOLES, [n], G=1) as s:
        plan = _bench_plan(s, mm)
        s.run(plan)
        ti = torch.from_numpy(idx).cuda()
        call = s.bufs[(3, 0)][ti].cpu().numpy().astype(np.float64)
        put = s.bufs[(4, 0)][ti].cpu().numpy().astype(np.float64)
    S = np.concatenate([synthgen.uniform(1, synthgen.AID_BS_S, 5.0, 30.0, start=int(i)) for i in idx])
    X = np.concatenate([synthgen.uniform(1, synthgen.AID_BS_X, 1.0, 100.0, start=int(i)) for i in idx])
    T = np.concatenate([synthgen.uniform(1, synthgen.AID_BS_T, 0.25, 10.0, start=int(i)) for i in idx])
    rc, rp = on.blackscholes(S, X, T)
    assert np.max(np.abs(call - rc) / np.maximum(np.abs(rc), 1.0)) <= 1e-5     # R19
    assert np.max(np.abs(put - rp) / np.maximum(np.abs(rp), 1.0)) <= 1e-5


@pytest.mark.parametrize("integer", [True, False])
def test_sgemm_p311_size_sampled_rows(R, integer):
    """SK-One MatrixMul 6144^2 (P311) on tcgen05 3xTF32: sampled rows (tile
    seams at 128, first/last) vs the FP64 oracle on those rows; integer inputs
    are exact in FP32, so bit-exact."""
    mm, runner = R
    n = 6144
    rows = np.array([0, 1, 127, 128, 129, 3071, 3072, 6015, 6016, n - 1])
    import torch
    with runner.session(mm.MM_APP_SGEMM, [n, n, n, 2], G=1) as s:
        prof = s.profile(reps=2)
        s.fill(integer=integer)
        plan = s.plan(mm.MM_SP_SINGLE, prof)
        s.run(plan)
        got = s.bufs[(2, 0)].view(n, n)[torch.from_numpy(rows).cuda()].cpu().numpy()
    if integer:
        A, B = synthgen.matmul_integer(n, n, n)
    else:
        A, B = synthgen.matmul_uniform(n, n, n)
    ref = on.sgemm(np.ascontiguousarray(A[rows]), B)
    if integer:
        assert np.array_equal(got, ref)
    else:
        assert np.max(np.abs(got - ref) / np.abs(ref)) <= 1e-4


def test_cholesky_configs4_sampled_entries(R):
    """MK-DAG Cholesky 32768^2, tile 1024 (BASELINE configs[4]) from the
    device SPD generator: for sampled (i, j), i >= j (tile seams included),
    sum_k L_ik L_jk reproduces A_ij (the definition A = L L^T), relative to
    sqrt(A_ii A_jj); the diagonal of L is positive and tiles above the
    diagonal are untouched."""
    mm, runner = R
    n, b = 32768, 1024
    T = n // b
    import torch
    with runner.session(mm.MM_APP_CHOLESKY, [n, b], G=1) as s:
        plan = _bench_plan(s, mm)
        s.run(plan)
        tiles = s.bufs[(0, 0)].view(T, T, b, b)
        want = sorted({0, 1, 1023, 1024, 1025, 16383, 16384, 31743, 31744, n - 1})
        rows = {}
        for i in want:
            ti, ri = divmod(i, b)
            rows[i] = tiles[ti, : ti + 1, ri, :].reshape(-1).cpu().numpy().astype(np.float64)
        upper = tiles[0, 1].abs().max().item(), tiles[T - 2, T - 1].abs().max().item()
    def a_ij(i, j):
        sij = synthgen.uniform(1, synthgen.AID_CHOL_S, 0.0, 1.0, start=i * n + j)[0]
        sji = synthgen.uniform(1, synthgen.AID_CHOL_S, 0.0, 1.0, start=j * n + i)[0]
        return float(np.float32((np.float64(sij) + np.float64(sji)) * 0.5 + (n if i == j else 0.0)))
    diag = {i: a_ij(i, i) for i in want}
    for i in want:
        assert rows[i][i] > 0
        for j in want:
            if j > i:
                continue
            lij = np.dot(rows[i][: j + 1], rows[j][: j + 1])
            err = abs(lij - a_ij(i, j)) / np.sqrt(diag[i] * diag[j])
            assert err <= 2e-5, (i, j, err)
    # upper tiles keep the generator's values (untouched, R23)
    assert upper[0] > 0 and upper[1] > 0


def test_nbody_p319_size_sampled_bodies(R):
    """Nbody 1,048,576 bodies (P319), one step: sampled bodies (CTA and pair
    seams) vs the FP64 oracle summing over all bodies."""
    mm, runner = R
    n = 1 << 20
    bodies = np.array([0, 1, 255, 256, 511, 512, 513, 524287, 524288, n - 2, n - 1]
                      + list(np.random.default_rng(3).integers(0, n, 21)))
    import torch
    with runner.session(mm.MM_APP_NBODY, [n, 1], G=1) as s:
        plan = _bench_plan(s, mm)
        s.run(plan)
        ti = torch.from_numpy(bodies).cuda()
        gp = s.bufs[(1, 0)].view(n, 4)[ti].cpu().numpy().astype(np.float64)
        gv = s.bufs[(3, 0)].view(n, 4)[ti].cpu().numpy().astype(np.float64)
    pos, vel = synthgen.nbody(n)
    rp, rv = on.nbody_step_bodies(pos, vel, bodies)
    # FP32 sum of 2^20 terms in a fixed order: relative error ~ sqrt(n) u
    # (u = 2^-24) times the terms' cancellation ratio; 2e-4 leaves 3x margin
    dv_abs = np.linalg.norm(gv[:, :3] - rv[:, :3], axis=1)
    dv = dv_abs / np.linalg.norm(rv[:, :3], axis=1)
    assert np.max(dv) <= 2e-4, np.max(dv)
    # x' = x + v' dt in FP32: |dx'| <= dt |dv'| + a few roundings of |x'|
    dp_abs = np.linalg.norm(gp[:, :3] - rp[:, :3], axis=1)
    bound = on.NBODY_DT * dv_abs * 1.01 + 4 * 2.0 ** -24 * np.maximum(np.linalg.norm(rp[:, :3], axis=1), 1.0)
    assert np.all(dp_abs <= bound), np.max(dp_abs / bound)
    assert np.array_equal(gp[:, 3], pos[bodies, 3])


def test_stencil_reduction_configs3_sampled_rows(R):
    """MK-Loop stencil + FP64 residual, 16384^2 (BASELINE configs[3]), 3
    steps with w-sync: sampled rows bit-exact vs the oracle on a row window,
    and their residual row sums of the last step."""
    mm, runner = R
    rows = cols = 16384
    steps = 3
    import torch
    with runner.session(mm.MM_APP_STENCIL_REDUCTION, [rows, cols, steps, 1], G=1) as s:
        plan = _bench_plan(s, mm)
        s.run(plan)
        out = s.bufs[(steps % 2, 0)].view(rows, cols)
        sample = [0, 1, 8191, 8192, rows - 1]
        got = {y: out[y].cpu().numpy() for y in sample}
        rs = s.bufs[(3, 0)][torch.tensor(sample).cuda()].cpu().numpy()
    t_full, p_full = synthgen.hotspot(rows, cols)
    for k, y in enumerate(sample):
        lo, hi = max(0, y - steps - 1), min(rows, y + steps + 2)
        prev = on.hotspot_run(t_full[lo:hi], p_full[lo:hi], steps - 1)
        last = on.hotspot_run(t_full[lo:hi], p_full[lo:hi], steps)
        assert np.array_equal(got[y], last[y - lo]), y
        ref = on.row_residual(prev, last)[y - lo]
        assert abs(rs[k] - ref) <= 1e-12 * max(ref, 1e-300), (y, rs[k], ref)
