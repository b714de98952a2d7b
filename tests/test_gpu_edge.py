"""Degenerate and edge-case inputs of the CUDA path vs the oracle: empty and
tiny index spaces (fewer items than devices, than the granule, than one
warp), single-row / single-column grids, 1x1 matrices and a one-tile
Cholesky.  Integer / bit-exact work must match exactly; FP32 apps within the
tolerances of the other parity tests."""
import numpy as np
import pytest

import synthgen
from oracle import numeric as on

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def R():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_icpp_shenvms15_b200 import mm, runner
    return mm, runner


def prof(mm, G, K):
    return mm.make_profile(G, [[1000 + 500 * d] * K for d in range(G)], [[10 ** 5] * K] * G, [10 ** 11] * G)


@pytest.mark.parametrize("n", [1, 5, 31, 33])
@pytest.mark.parametrize("strategy", [2, 3, 4, 5])
@pytest.mark.parametrize("G", [1, 3])
def test_stream_tiny(R, n, strategy, G):
    mm, runner = R
    a0, b0, c0 = synthgen.stream_random(n)
    ref = on.stream_run(a0, b0, c0, 1)
    with runner.session(mm.MM_APP_STREAM, [n, 1, 0, 32, 1], G=G) as s:
        s.fill()
        plan = s.plan(strategy, prof(mm, G, 4), chunks_per_dev=2)
        s.run(plan)
        for slot in range(3):
            assert np.array_equal(s.collect(plan, slot), ref[slot]), (n, strategy, G, slot)


@pytest.mark.parametrize("app, params", [("MM_APP_STREAM", [0, 1, 0, 32, 1]), ("MM_APP_BLACKSCHOLES", [0, 32, 1])])
def test_empty_index_space_runs_nothing(R, app, params):
    """n = 0: the plan has no items and the run launches no kernel."""
    mm, runner = R
    with runner.session(getattr(mm, app), params, G=2) as s:
        plan = s.plan(1 if app == "MM_APP_BLACKSCHOLES" else 2, prof(mm, 2, s.K))
        l0 = mm.mm_kernel_launch_count()
        st = s.run(plan)
        assert st.n_launches == 0 and mm.mm_kernel_launch_count() == l0


@pytest.mark.parametrize("n", [1, 7, 40])
@pytest.mark.parametrize("G", [1, 3])
def test_blackscholes_tiny(R, n, G):
    mm, runner = R
    S, X, T = synthgen.blackscholes(n)
    rc, rp = on.blackscholes(S, X, T)
    with runner.session(mm.MM_APP_BLACKSCHOLES, [n, 32, 1], G=G) as s:
        s.fill()
        plan = s.plan(4, prof(mm, G, 1), chunks_per_dev=2)
        s.run(plan)
        c = s.collect(plan, 3).astype(np.float64)
        p = s.collect(plan, 4).astype(np.float64)
    assert np.max(np.abs(c - rc) / np.maximum(np.abs(rc), 1.0)) <= 1e-5
    assert np.max(np.abs(p - rp) / np.maximum(np.abs(rp), 1.0)) <= 1e-5


@pytest.mark.parametrize("shape", [(1, 1), (1, 7), (5, 1), (2, 3), (3, 130)])
@pytest.mark.parametrize("strategy", [1, 4])
@pytest.mark.parametrize("G", [1, 3])
def test_hotspot_degenerate_grids(R, shape, strategy, G):
    """Single-row / single-column grids (every neighbour is a mirrored edge)
    and grids with fewer rows than devices."""
    mm, runner = R
    rows, cols = shape
    iters = 5
    t0, p = synthgen.hotspot(rows, cols)
    ref = on.hotspot_run(t0, p, iters)
    with runner.session(mm.MM_APP_HOTSPOT, [rows, cols, iters, 1, 1], G=G) as s:
        s.fill()
        plan = s.plan(strategy, prof(mm, G, 1), chunks_per_dev=2)
        s.run(plan)
        got = s.collect(plan, 1).reshape(rows, cols)
    assert np.array_equal(got, ref), (shape, strategy, G)


@pytest.mark.parametrize("shape", [(1, 1, 1), (1, 5, 3), (7, 1, 2), (3, 2, 1), (2, 300, 33)])
@pytest.mark.parametrize("variant", [1, 2])
@pytest.mark.parametrize("G", [1, 2])
def test_sgemm_degenerate(R, shape, variant, G):
    """1 x 1 products, single rows / columns, K = 1 (K padded to 32 in the
    3xTF32 operand split), fewer rows than devices.  Integer inputs: exact."""
    mm, runner = R
    M, N, K = shape
    A, B = synthgen.matmul_integer(M, K, N)
    ref = on.sgemm(A, B)
    with runner.session(mm.MM_APP_SGEMM, [M, N, K, variant, 1, 1], G=G) as s:
        s.fill(integer=True)
        plan = s.plan(1, prof(mm, G, 1))
        s.run(plan)
        got = s.collect(plan, 2).reshape(M, N)
    assert np.array_equal(got, ref), (shape, variant, G)


@pytest.mark.parametrize("b", [128, 256])
@pytest.mark.parametrize("strategy", [4, 5, 6])
def test_cholesky_single_tile(R, b, strategy):
    """T = 1: the DAG is one POTRF task (no TRSM / update)."""
    mm, runner = R
    A, L0 = synthgen.cholesky_exact_factor(b)
    with runner.session(mm.MM_APP_CHOLESKY, [b, b], G=2) as s:
        s.load(0, A.reshape(-1))
        plan = s.plan(strategy, prof(mm, 2, 4))
        s.run(plan)
        L = s.collect(plan, 0).reshape(b, b)
    assert np.array_equal(np.tril(L), L0)
    assert np.all(np.triu(L, 1) == 0)


@pytest.mark.parametrize("shape", [(1, 4), (2, 8), (5, 12), (9, 1028), (17, 116)])
@pytest.mark.parametrize("tb", [3, 8])
@pytest.mark.parametrize("G", [1, 2])
def test_hotspot_temporal_block_small_grids(R, shape, tb, G):
    """Temporal blocks on grids shorter than the block's halo (rows < 2 tb),
    one or two float4 columns, and widths just past one warp tile (116 = 112
    output columns + 4): the strip head, the chip-edge warps and the grid's
    first/last rows in one launch; bit-identical to the oracle."""
    mm, runner = R
    rows, cols = shape
    iters = 2 * tb
    t0, p = synthgen.hotspot(rows, cols)
    ref = on.hotspot_run(t0, p, iters)
    with runner.session(mm.MM_APP_HOTSPOT, [rows, cols, iters, 1, 1, tb], G=G) as s:
        s.fill()
        plan = s.plan(1, prof(mm, G, 1), chunks_per_dev=2)
        s.run(plan)
        got = s.collect(plan, 0).reshape(rows, cols)
    assert np.array_equal(got, ref), (shape, tb, G)
