"""GPU parity: the CUDA path (libmm.so through its C ABI) against the oracle,
element by element, on the same seeded inputs.  Several logical devices are
mapped onto GPU 0 (separate streams and full-size buffer copies), so every
partitioning strategy, re-sync, halo and sync path runs on one B200.

Tolerances (BASELINE north_star): bit-exact for STREAM, HotSpot and
integer-input MatrixMul (FP32 with a fixed operation order, R13/R16); <= 1e-5
for BlackScholes (FP32 vs the FP64 oracle, R19); <= 1e-4 relative for
MatrixMul on U[0,1) data; rowsum within 1e-12 relative (FP64)."""
import numpy as np
import pytest

import synthgen
from oracle import numeric as on

pytestmark = pytest.mark.gpu

SP = {1: "SP-Single", 2: "SP-Unified", 3: "SP-Varied", 4: "DP-Perf", 5: "DP-Dep"}


@pytest.fixture(scope="module")
def R(gpu):
    from paper_conf_icpp_shenvms15_b200 import mm, runner
    return mm, runner


def rand_profile(mm, G, K, seed):
    rnd = np.random.default_rng(seed)
    ps = rnd.integers(500, 3000, size=(G, K)).tolist()
    est = rnd.integers(10 ** 4, 10 ** 6, size=(G, K)).tolist()
    link = rnd.integers(10 ** 9, 10 ** 12, size=G).tolist()
    return mm.make_profile(G, ps, est, link)


def test_device_generator_matches_synthgen(R):
    mm, runner = R
    with runner.session(mm.MM_APP_STREAM, [100003, 1, 0, 32, 1], G=1) as s:
        s.fill()
        for slot, aid in ((0, synthgen.AID_STREAM_A), (1, synthgen.AID_STREAM_B)):
            got = s.bufs[(slot, 0)].cpu().numpy()
            assert np.array_equal(got, synthgen.uniform(100003, aid, -1.0, 1.0))
        t = s.bufs[(2, 0)]
        mm.mm_fill_integers(s.ctx, 0, t.data_ptr(), 5000, synthgen.SEED, 31, 17, -4, 4)
        assert np.array_equal(t[:5000].cpu().numpy(),
                              synthgen.integers(5000, 31, -4, 4, start=17).astype(np.float32))


@pytest.mark.parametrize("strategy", [2, 3, 4, 5])
@pytest.mark.parametrize("sync", [0, 1, 2])
@pytest.mark.parametrize("G", [1, 3])
def test_stream_bit_exact(R, strategy, sync, G):
    mm, runner = R
    n, passes = 100003, 3
    a0, b0, c0 = synthgen.stream_random(n)
    ra, rb, rc = on.stream_run(a0, b0, c0, passes)
    with runner.session(mm.MM_APP_STREAM, [n, passes, sync, 32, 1], G=G) as s:
        s.fill()
        prof = rand_profile(mm, G, 4, strategy * 10 + sync)
        plan = s.plan(strategy, prof, chunks_per_dev=3)
        s.run(plan)
        for slot, ref in ((0, ra), (1, rb), (2, rc)):
            got = s.collect(plan, slot)
            assert np.array_equal(got, ref), (SP[strategy], sync, G, slot)


def test_stream_graph_replay_and_staged(R):
    mm, runner = R
    n = 65536 + 77
    a0, b0, c0 = synthgen.stream_random(n)
    ra, rb, rc = on.stream_run(a0, b0, c0, 2)
    import torch
    with runner.session(mm.MM_APP_STREAM, [n, 1, 0, 32, 1], G=2) as s:
        s.fill()
        plan = s.plan(4, rand_profile(mm, 2, 4, 5), chunks_per_dev=4)
        s.run(plan, use_graph=True)
        s.run(plan, use_graph=True)       # replay: second pass
        assert np.array_equal(s.collect(plan, 0), ra)
        # staged mode: host inputs, H2D/D2H inside the run
        host = [torch.from_numpy(x.copy()).pin_memory() for x in (a0, b0, c0)]
        splan = s.plan(2, rand_profile(mm, 2, 4, 6), staged=True)
        st = s.run(splan, host=[h.data_ptr() for h in host])
        r1 = on.stream_run(a0, b0, c0, 1)
        assert st.h2d_bytes > 0 and st.d2h_bytes > 0
        for h, ref in zip(host, r1):
            assert np.array_equal(h.numpy(), ref)


@pytest.mark.parametrize("shape", [(257, 256), (100, 37), (64, 1032)])
@pytest.mark.parametrize("strategy", [1, 4, 5])
@pytest.mark.parametrize("G", [1, 3])
def test_hotspot_bit_exact(R, shape, strategy, G):
    mm, runner = R
    rows, cols = shape
    iters = 7
    t0, p = synthgen.hotspot(rows, cols)
    ref = on.hotspot_run(t0, p, iters)
    with runner.session(mm.MM_APP_HOTSPOT, [rows, cols, iters, 1, 1], G=G) as s:
        s.fill()
        plan = s.plan(strategy, rand_profile(mm, G, 1, rows + strategy), chunks_per_dev=2)
        s.run(plan)
        out_slot = 0 if iters % 2 == 0 else 1
        got = s.collect(plan, out_slot).reshape(rows, cols)
        assert np.array_equal(got, ref), (SP[strategy], G, shape)


@pytest.mark.parametrize("tb", [2, 3, 4, 6, 8])
@pytest.mark.parametrize("shape", [(257, 256), (100, 36), (64, 1032), (37, 4)])
@pytest.mark.parametrize("strategy", [1, 4, 5])
@pytest.mark.parametrize("G", [1, 3])
def test_hotspot_temporal_block_bit_exact(R, tb, shape, strategy, G):
    """One launch = tb iterations (warp tiles of 128 columns streaming down
    row strips with a tb-level register pipeline): bit-identical to 24 plain
    iterations of the oracle, across partitions and halo exchanges."""
    mm, runner = R
    rows, cols = shape
    iters = 24
    t0, p = synthgen.hotspot(rows, cols)
    ref = on.hotspot_run(t0, p, iters)
    with runner.session(mm.MM_APP_HOTSPOT, [rows, cols, iters, 1, 1, tb], G=G) as s:
        s.fill()
        plan = s.plan(strategy, rand_profile(mm, G, 1, rows + strategy + tb), chunks_per_dev=2)
        s.run(plan)
        out_slot = 0 if (iters // tb) % 2 == 0 else 1
        got = s.collect(plan, out_slot).reshape(rows, cols)
        assert np.array_equal(got, ref), (SP[strategy], G, shape, tb)


@pytest.mark.parametrize("case", ["stream", "hotspot", "hotspot_tb4", "blackscholes"])
def test_dp_static_bit_exact(R, case):
    """§V conversion (P565): DP chunks assigned by the static ratio run
    through the same engine; results identical to the oracle."""
    mm, runner = R
    G = 3
    if case == "stream":
        n = 100003
        with runner.session(mm.MM_APP_STREAM, [n, 2, 0, 32, 1], G=G) as s:
            s.fill()
            plan = s.plan(mm.MM_DP_STATIC, rand_profile(mm, G, 4, 7), chunks_per_dev=3)
            s.run(plan)
            got = [s.collect(plan, k) for k in range(3)]
        ref = on.stream_run(*synthgen.stream_random(n), 2)
        for g_, r_ in zip(got, ref):
            assert np.array_equal(g_, r_)
    elif case.startswith("hotspot"):
        rows, cols, tb = 203, 132, (4 if case.endswith("tb4") else 1)
        iters = 8
        t0, p = synthgen.hotspot(rows, cols)
        ref = on.hotspot_run(t0, p, iters)
        with runner.session(mm.MM_APP_HOTSPOT, [rows, cols, iters, 1, 1, tb], G=G) as s:
            s.fill()
            plan = s.plan(mm.MM_DP_STATIC, rand_profile(mm, G, 1, 11), chunks_per_dev=4)
            s.run(plan)
            got = s.collect(plan, 0 if (iters // tb) % 2 == 0 else 1).reshape(rows, cols)
        assert np.array_equal(got, ref)
    else:
        n = 50021
        S, X, T = synthgen.blackscholes(n)
        with runner.session(mm.MM_APP_BLACKSCHOLES, [n, 32, 1], G=G) as s:
            s.fill()
            plan = s.plan(mm.MM_DP_STATIC, rand_profile(mm, G, 1, 5), chunks_per_dev=2)
            s.run(plan)
            call, put = s.collect(plan, 3), s.collect(plan, 4)
        rc, rp = on.blackscholes(S, X, T)
        assert np.max(np.abs(call - rc) / np.maximum(np.abs(rc), 1.0)) < 1e-5
        assert np.max(np.abs(put - rp) / np.maximum(np.abs(rp), 1.0)) < 1e-5


@pytest.mark.parametrize("strategy", [4, 5, 7])
def test_tune_chunks(R, strategy):
    """Task-size auto-tuning (P565): the returned count is a candidate with the
    smallest median time; a non-DP strategy is rejected."""
    mm, runner = R
    with runner.session(mm.MM_APP_STREAM, [1 << 20, 1, 0, 32, 1], G=2) as s:
        s.fill()
        prof = s.profile(reps=2)
        cand = [1, 2, 8, 32]
        best, ms = s.tune_chunks(strategy, prof, cand, reps=2)
        assert best in cand and all(t > 0 for t in ms)
        assert ms[cand.index(best)] == min(ms)
        with pytest.raises(mm.MMError):
            s.tune_chunks(mm.MM_SP_UNIFIED, prof, cand)


@pytest.mark.parametrize("strategy", [2, 3, 4, 5])
def test_stencil_reduction(R, strategy):
    mm, runner = R
    rows, cols, steps = 131, 64, 4
    t0, p = synthgen.hotspot(rows, cols)
    tf, rs = on.stencil_reduction_run(t0, p, steps)
    prev = on.hotspot_run(t0, p, steps - 1)
    last_rows = on.row_residual(prev, tf)
    with runner.session(mm.MM_APP_STENCIL_REDUCTION, [rows, cols, steps, 2, 1, 1], G=3) as s:
        s.fill()
        plan = s.plan(strategy, rand_profile(mm, 3, 2, strategy), chunks_per_dev=2)
        s.run(plan)
        got = s.collect(plan, 0 if steps % 2 == 0 else 1).reshape(rows, cols)
        assert np.array_equal(got, tf)
        rowsum = s.collect(plan, 3)
        assert np.max(np.abs(rowsum - last_rows) / np.maximum(last_rows, 1e-300)) < 1e-12
        import math
        assert abs(math.fsum(rowsum) - rs[-1]) <= 1e-12 * rs[-1]


@pytest.mark.parametrize("G", [1, 2])
@pytest.mark.parametrize("strategy", [1, 4, 5])
def test_blackscholes(R, G, strategy):
    mm, runner = R
    n = 100003
    S, X, T = synthgen.blackscholes(n)
    rc, rp = on.blackscholes(S, X, T)
    with runner.session(mm.MM_APP_BLACKSCHOLES, [n, 32, 1], G=G) as s:
        s.fill()
        plan = s.plan(strategy, rand_profile(mm, G, 1, 3), chunks_per_dev=2)
        s.run(plan)
        c = s.collect(plan, 3).astype(np.float64)
        p = s.collect(plan, 4).astype(np.float64)
    err_c = np.max(np.abs(c - rc) / np.maximum(np.abs(rc), 1.0))
    err_p = np.max(np.abs(p - rp) / np.maximum(np.abs(rp), 1.0))
    assert err_c <= 1e-5 and err_p <= 1e-5, (err_c, err_p)
    # put-call parity on the GPU's own outputs (FP32 rounding of ~max(S,X))
    par = (c - p) - (S - X * np.exp(-on.BS_R * T.astype(np.float64)))
    assert np.max(np.abs(par) / np.maximum(S, X)) < 4e-6


@pytest.mark.parametrize("shape", [(300, 200, 96), (257, 520, 77), (1024, 1024, 1024), (512, 301, 1000)])
@pytest.mark.parametrize("variant", [1, 2])
@pytest.mark.parametrize("G", [1, 2])
def test_sgemm(R, variant, G, shape):
    """variant 1 = FFMA, 2 = tcgen05 3xTF32 (TMA + TMEM); ragged M, N, K.
    1024^3 and 512 x 301 x 1000 take the split-K path (4 K splits of 2-SM
    tile pairs + ordered reduction; the latter with a ragged N and K)."""
    mm, runner = R
    M, N, K = shape
    Ai, Bi = synthgen.matmul_integer(M, K, N)
    ref_i = on.sgemm(Ai, Bi)
    Au, Bu = synthgen.matmul_uniform(M, K, N)
    ref_u = on.sgemm(Au, Bu)
    for integer, ref in ((True, ref_i), (False, ref_u)):
        with runner.session(mm.MM_APP_SGEMM, [M, N, K, variant, 16, 1], G=G) as s:
            s.fill(integer=integer)
            plan = s.plan(1, rand_profile(mm, G, 1, 9))
            s.run(plan)
            got = s.collect(plan, 2).reshape(M, N)
        if integer:
            assert np.array_equal(got, ref)
        else:
            assert np.max(np.abs(got - ref) / np.abs(ref)) <= 1e-4


@pytest.mark.parametrize("strategy", [4, 5, 7])
@pytest.mark.parametrize("shape", [(520, 300, 77), (1024, 512, 256)])
def test_sgemm_dp_chunks(R, strategy, shape):
    """DP-Perf / DP-Dep / DP-Static chunk the rows of one SGEMM over 2 logical
    devices: every chunk after a device's first reuses that device's cached
    B split (the split launch then covers A only); ragged K exercises the
    scalar split path.  Integer inputs: bit-exact; uniform: 1e-4."""
    mm, runner = R
    M, N, K = shape
    for integer in (True, False):
        A, B = (synthgen.matmul_integer if integer else synthgen.matmul_uniform)(M, K, N)
        ref = on.sgemm(A, B)
        with runner.session(mm.MM_APP_SGEMM, [M, N, K, 2, 16, 1], G=2) as s:
            s.fill(integer=integer)
            plan = s.plan(strategy, rand_profile(mm, 2, 1, 5), chunks_per_dev=4)
            s.run(plan)
            s.run(plan)
            got = s.collect(plan, 2).reshape(M, N)
        if integer:
            assert np.array_equal(got, ref)
        else:
            assert np.max(np.abs(got - ref) / np.abs(ref)) <= 1e-4


def test_sgemm_splitk_repeat_and_graph(R):
    """Split-K SGEMM (1024^3: the last arrival per tile sums the K partials in
    split order inside the GEMM) gives the same bits on every eager run and
    every CUDA-graph replay of the same session (the arrival counters are
    cleared by the last arrival; graph replays reuse the captured launch tag)."""
    mm, runner = R
    M = N = K = 1024
    Au, Bu = synthgen.matmul_uniform(M, K, N)
    ref = on.sgemm(Au, Bu)
    outs = []
    with runner.session(mm.MM_APP_SGEMM, [M, N, K, 2, 16, 1], G=1) as s:
        s.fill(integer=False)
        plan = s.plan(1, rand_profile(mm, 1, 1, 9))
        for graph in (False, False, True, True, True, False):
            s.bufs[(2, 0)].fill_(float("nan"))
            s.run(plan, use_graph=graph)
            outs.append(s.collect(plan, 2).reshape(M, N))
    assert np.max(np.abs(outs[0] - ref) / np.abs(ref)) <= 1e-4
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])


def test_stream_full_size_sampled(R):
    """BASELINE configs[1] size (2^28) in the bench's launch configuration
    (1 logical device, SP-Unified, CUDA graph): sampled outputs vs the oracle
    run on the sampled inputs (STREAM is elementwise)."""
    mm, runner = R
    n = 1 << 28
    idx = np.unique(np.concatenate([np.arange(0, 64), np.arange(n - 64, n),
                                    np.random.default_rng(0).integers(0, n, 4096)]))
    with runner.session(mm.MM_APP_STREAM, [n, 1, 0], G=1) as s:
        prof = s.profile(reps=3)          # profiling runs the kernels: fill afterwards
        s.fill()
        plan = s.plan(2, prof)
        s.run(plan, use_graph=True)
        import torch
        ti = torch.from_numpy(idx).cuda()
        got = [s.bufs[(k, 0)][ti].cpu().numpy() for k in range(3)]
    a0 = np.concatenate([synthgen.uniform(1, synthgen.AID_STREAM_A, -1, 1, start=int(i)) for i in idx])
    b0 = np.concatenate([synthgen.uniform(1, synthgen.AID_STREAM_B, -1, 1, start=int(i)) for i in idx])
    c0 = np.concatenate([synthgen.uniform(1, synthgen.AID_STREAM_C, -1, 1, start=int(i)) for i in idx])
    ra, rb, rc = on.stream_run(a0, b0, c0, 1)
    assert np.array_equal(got[0], ra) and np.array_equal(got[1], rb) and np.array_equal(got[2], rc)


def test_hotspot_full_size_sampled_rows(R):
    """BASELINE configs[2] grid (8192^2) for 6 iterations: sampled rows vs the
    oracle on a row window (the dependency cone after k steps is k rows)."""
    mm, runner = R
    rows = cols = 8192
    iters = 6
    with runner.session(mm.MM_APP_HOTSPOT, [rows, cols, iters], G=1) as s:
        s.fill()
        plan = s.plan(1)
        s.run(plan)
        out = s.bufs[(0, 0)].view(rows, cols)
        sample = [0, 1, 4095, 4096, rows - 1]
        got = {y: out[y].cpu().numpy() for y in sample}
    t_full, p_full = synthgen.hotspot(rows, cols)
    for y in sample:
        lo, hi = max(0, y - iters - 1), min(rows, y + iters + 2)
        # window rows at the cut are wrong after k steps only within k rows of the cut
        ref = on.hotspot_run(t_full[lo:hi], p_full[lo:hi], iters)
        assert np.array_equal(got[y], ref[y - lo]), y


@pytest.mark.parametrize("tb", [4, 8])
def test_hotspot_temporal_block_full_size_sampled_rows(R, tb):
    """BASELINE configs[2] grid (8192^2), 2 temporal blocks, in the launch
    configuration bench.py times: sampled rows (strip and warp-tile seams
    included) vs the oracle on a row window."""
    mm, runner = R
    rows = cols = 8192
    iters = 2 * tb
    with runner.session(mm.MM_APP_HOTSPOT, [rows, cols, iters, 0, 0, tb], G=1) as s:
        s.fill()
        plan = s.plan(1)
        s.run(plan)
        out = s.bufs[(0, 0)].view(rows, cols)
        sample = [0, 1, 2, 127, 128, 255, 256, 4095, 4096, rows - 2, rows - 1]
        got = {y: out[y].cpu().numpy() for y in sample}
    t_full, p_full = synthgen.hotspot(rows, cols)
    for y in sample:
        lo, hi = max(0, y - iters - 1), min(rows, y + iters + 2)
        ref = on.hotspot_run(t_full[lo:hi], p_full[lo:hi], iters)
        assert np.array_equal(got[y], ref[y - lo]), y


def _to_tiles(A, b):
    n = A.shape[0]
    T = n // b
    return A.reshape(T, b, T, b).transpose(0, 2, 1, 3).copy()


def _from_tiles(t, n, b):
    T = n // b
    return t.reshape(T, T, b, b).transpose(0, 2, 1, 3).reshape(n, n)


@pytest.mark.parametrize("nb", [(512, 128), (1024, 256), (2048, 128)])
@pytest.mark.parametrize("strategy", [4, 5, 6])
@pytest.mark.parametrize("G", [1, 2, 3])
def test_cholesky_exact_factor(R, strategy, G, nb):
    """MK-DAG: integer L0 (diag 32..64, band +-1), A = L0 L0^T: every FP32
    operation is exact, so the factor must be L0 bit for bit for any schedule.
    b = 128 runs the FFMA updates, b = 256 the 3xTF32 tcgen05 updates."""
    mm, runner = R
    n, b = nb
    A, L0 = synthgen.cholesky_exact_factor(n)
    with runner.session(mm.MM_APP_CHOLESKY, [n, b], G=G) as s:
        assert s.classify() == mm.MM_MK_DAG
        s.load(0, _to_tiles(A, b))
        plan = s.plan(strategy, rand_profile(mm, G, 4, 7))
        s.run(plan)
        L = _from_tiles(s.collect(plan, 0), n, b)
    assert np.array_equal(np.tril(L), L0)
    T = n // b
    for k in range(T):   # diagonal tiles: strictly upper part zeroed
        blk = L[k * b:(k + 1) * b, k * b:(k + 1) * b]
        assert np.all(np.triu(blk, 1) == 0)


@pytest.mark.parametrize("nb", [(512, 128), (1024, 256), (2048, 256)])
def test_cholesky_random_spd(R, nb):
    mm, runner = R
    n, b = nb
    A = synthgen.spd_random(n)
    ref = on.cholesky(A.astype(np.float64))
    with runner.session(mm.MM_APP_CHOLESKY, [n, b], G=2) as s:
        s.load(0, _to_tiles(A, b))
        plan = s.plan(4, rand_profile(mm, 2, 4, 8))
        s.run(plan, use_graph=True)
        L = np.tril(_from_tiles(s.collect(plan, 0), n, b)).astype(np.float64)
    assert np.max(np.abs(L - ref)) / np.max(np.abs(ref)) <= 1e-4


_CHOL_SCRIPT = r"""
import sys, numpy as np
sys.path.insert(0, {root!r})
import synthgen
from paper_conf_icpp_shenvms15_b200 import mm, runner
n, b = {n}, {b}
A = synthgen.spd_random(n)
T = n // b
At = A.reshape(T, b, T, b).transpose(0, 2, 1, 3).reshape(-1)
rnd = np.random.default_rng(3)
G = 1
prof = mm.make_profile(G, rnd.integers(500, 3000, size=(G, 4)).tolist(),
                       rnd.integers(10 ** 4, 10 ** 6, size=(G, 4)).tolist(), [10 ** 10])
with runner.session(mm.MM_APP_CHOLESKY, [n, b], G=G) as s:
    s.load(0, At)
    plan = s.plan(4, prof)
    s.run(plan)
    np.save({out!r}, s.collect(plan, 0))
"""


@pytest.mark.parametrize("nb", [(1024, 256), (1024, 128), (2048, 128)])
def test_cholesky_random_spd_schedule_invariant(R, nb):
    """on random SPD data (inexact arithmetic) the factor is the
    same bit for bit under every schedule and device count — each tile's
    updates run in the WAW-chain order, and no kernel's arithmetic depends on
    how the runtime batches the tasks of a step."""
    mm, runner = R
    n, b = nb
    A = synthgen.spd_random(n)
    ref = None
    for strategy, G in ((4, 1), (4, 2), (5, 3), (6, 2), (4, 3)):
        with runner.session(mm.MM_APP_CHOLESKY, [n, b], G=G) as s:
            s.load(0, _to_tiles(A, b))
            plan = s.plan(strategy, rand_profile(mm, G, 4, 11 * G + strategy))
            s.run(plan)
            got = s.collect(plan, 0)
        if ref is None:
            ref = got
        assert np.array_equal(got, ref), (strategy, G)


def _chol_subprocess(tmp_path, tag, env_set, n=2048, b=512):
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = str(tmp_path / f"chol_{tag}.npy")
    env = dict(os.environ)
    for key in ("MM_LEAF_WIDE_MIN", "MM_TRSM_COL"):
        env.pop(key, None)
    env.update(env_set)
    code = _CHOL_SCRIPT.format(root=root, n=n, b=b, out=out)
    subprocess.run([sys.executable, "-c", code], check=True, env=env, cwd=root, timeout=600)
    return np.load(out)


def test_cholesky_trsm_leaf_variants_identical(gpu, tmp_path):
    """Leaf path (MM_TRSM_COL=0): the wide (one 256-row CTA per SM, large
    batches) and narrow (64-row CTAs, small batches) TRSM leaves do the same
    arithmetic: forcing the wide leaf for every batch (MM_LEAF_WIDE_MIN=1, a
    fresh process) gives the leaf path's default factor bit for bit."""
    a = _chol_subprocess(tmp_path, "leaf", {"MM_TRSM_COL": "0"})
    w = _chol_subprocess(tmp_path, "wide", {"MM_TRSM_COL": "0", "MM_LEAF_WIDE_MIN": "1"})
    assert np.array_equal(a, w)


def test_cholesky_trsm_column_vs_leaf_path(gpu, tmp_path):
    """The one-launch column TRSM (default, kernels_chol_trsm.cu: left-looking
    over the 128-column leaves, one FP32 accumulation of the earlier leaves'
    3xTF32 products) and the leaf path (right-looking: one subtraction per
    earlier leaf) round differently on random SPD data but agree within the
    3xTF32 tolerance, and both match the FP64 oracle (R28)."""
    n, b = 2048, 512
    col = _chol_subprocess(tmp_path, "col", {})
    leaf = _chol_subprocess(tmp_path, "leaf", {"MM_TRSM_COL": "0"})
    ref = on.cholesky(synthgen.spd_random(n).astype(np.float64))
    for got in (col, leaf):
        L = np.tril(_from_tiles(got, n, b)).astype(np.float64)
        assert np.max(np.abs(L - ref)) / np.max(np.abs(ref)) <= 1e-4


def test_cholesky_device_spd_generator(R):
    mm, runner = R
    n, b = 384, 128
    with runner.session(mm.MM_APP_CHOLESKY, [n, b], G=1) as s:
        s.fill()
        got = s.bufs[(0, 0)].cpu().numpy()
    assert np.array_equal(got, _to_tiles(synthgen.spd_random(n), b).reshape(-1))


@pytest.mark.parametrize("app", ["stream", "hotspot"])
def test_adaptive_dp_perf(R, app):
    """Adaptive DP-Perf (P119: estimates kept and updated at run time): results
    stay bit-exact, and every logged decision is the earliest-finish choice on
    its own snapshot (replayed by the oracle's rule)."""
    mm, runner = R
    from oracle import control as oc
    if app == "stream":
        n, passes = 1 << 20, 2
        ip, G = [n, passes, 1, 32, 1], 3
        a0, b0, c0 = synthgen.stream_random(n)
        ref = on.stream_run(a0, b0, c0, 2 * passes)
        sess = runner.session(mm.MM_APP_STREAM, ip, G=G)
    else:
        rows, cols, iters = 512, 256, 6
        ip, G = [rows, cols, iters, 1, 1], 2
        t0, p = synthgen.hotspot(rows, cols)
        ref = on.hotspot_run(t0, p, 2 * iters)
        sess = runner.session(mm.MM_APP_HOTSPOT, ip, G=G)
    with sess as s:
        prof = s.profile(reps=3)
        s.fill()
        plan = s.plan(4, prof, chunks_per_dev=4)
        s.run(plan, adaptive=True, max_inflight=3)
        s.run(plan, adaptive=True, max_inflight=3)   # continues from the first run's placement
        if app == "stream":
            for k in range(3):
                assert np.array_equal(s.collect(plan, k), ref[k])
        else:
            assert np.array_equal(s.collect(plan, 0).reshape(rows, cols), ref)
        decs = mm.mm_run_decisions(plan)
        info = mm.mm_plan_info(plan)
        assert len(decs) == info.n_tasks
        for dc in decs:
            busy, ready, cost = list(dc.busy_ns[:G]), list(dc.ready_ns[:G]), list(dc.cost_ns[:G])
            chosen, eft = oc.replay_decision(busy, ready, cost)
            assert chosen == dc.chosen and eft == list(dc.eft_ns[:G])
