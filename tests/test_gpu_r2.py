"""Round-2 GPU parity and runtime tests (VERDICT r1 "what's missing" 1, 5, 6):
Cholesky against the oracle at the bench tile, SM-budgeted (green-context)
devices through the whole method (measured profile -> split/schedule -> run),
Glinda's measured transfer term, the CUDA-graph key and the kernel counter."""
import numpy as np
import pytest

import synthgen
from oracle import numeric as on

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def R(gpu):
    from paper_conf_icpp_shenvms15_b200 import mm, runner
    return mm, runner


def _to_tiles(A, b):
    n = A.shape[0]
    T = n // b
    return A.reshape(T, b, T, b).transpose(0, 2, 1, 3).copy()


def _from_tiles(t, n, b):
    T = n // b
    return t.reshape(T, T, b, b).transpose(0, 2, 1, 3).reshape(n, n)


def _prof(mm, G, K):
    rnd = np.random.default_rng(100 + G)
    return mm.make_profile(G, rnd.integers(500, 3000, size=(G, K)).tolist(),
                           rnd.integers(10 ** 4, 10 ** 6, size=(G, K)).tolist(),
                           rnd.integers(10 ** 9, 10 ** 12, size=G).tolist())


# ---------------------------------------------- Cholesky at the bench tile --
@pytest.mark.parametrize("b", [1024, 512])
@pytest.mark.parametrize("strategy,G", [(4, 1), (5, 2), (6, 2)])
def test_cholesky_exact_factor_bench_tile(R, b, strategy, G):
    """SURVEY c12 exact-factor pin at BASELINE configs[4]'s tile (b = 1024)
    and the 512 sweep point, n = 4096: every FP32 operation is exact, so the
    factor is L0 bit for bit (DP-Perf G=1, DP-Dep G=2, SP-Cyclic G=2)."""
    mm, runner = R
    n = 4096
    A, L0 = synthgen.cholesky_exact_factor(n)
    with runner.session(mm.MM_APP_CHOLESKY, [n, b], G=G) as s:
        s.load(0, _to_tiles(A, b))
        plan = s.plan(strategy, _prof(mm, G, 4))
        s.run(plan)
        L = _from_tiles(s.collect(plan, 0), n, b)
    assert np.array_equal(np.tril(L), L0)
    for k in range(n // b):
        assert np.all(np.triu(L[k * b:(k + 1) * b, k * b:(k + 1) * b], 1) == 0)


@pytest.mark.parametrize("b", [2048, 4096, 256])
def test_cholesky_exact_factor_wide_tiles(R, b):
    """The column TRSM's leaf count b/128 at its extremes (2, 16, 32 leaves;
    kernels_chol_trsm.cu kMaxLeaves = 32): n = 2 b (or 8192 for b = 256),
    exact-factor input, the factor is L0 bit for bit."""
    mm, runner = R
    n = 2 * b if b > 256 else 8192
    A, L0 = synthgen.cholesky_exact_factor(n)
    with runner.session(mm.MM_APP_CHOLESKY, [n, b], G=1) as s:
        s.load(0, _to_tiles(A, b))
        plan = s.plan(mm.MM_DP_PERF, _prof(mm, 1, 4))
        s.run(plan)
        L = _from_tiles(s.collect(plan, 0), n, b)
    assert np.array_equal(np.tril(L), L0)


def test_cholesky_random_spd_bench_tile(R):
    """Random SPD n = 4096 at b = 1024 (4 x 4 tiles, the bench's kernels and
    batching) against the FP64 oracle (unblocked Cholesky-Banachiewicz):
    max-norm relative error <= 1e-4 (SURVEY c12 reading)."""
    mm, runner = R
    n, b = 4096, 1024
    A = synthgen.spd_random(n)
    ref = on.cholesky(A.astype(np.float64))
    with runner.session(mm.MM_APP_CHOLESKY, [n, b], G=1) as s:
        s.load(0, _to_tiles(A, b))
        plan = s.plan(4, _prof(mm, 1, 4))
        s.run(plan, use_graph=True)
        L = np.tril(_from_tiles(s.collect(plan, 0), n, b)).astype(np.float64)
    err = np.max(np.abs(L - ref)) / np.max(np.abs(ref))
    assert err <= 1e-4, err


# ------------------------------------------- SM-budgeted (green) devices ----
def test_green_context_sms_granted(R):
    mm, runner = R
    with runner.session(mm.MM_APP_STREAM, [1 << 16, 1, 0, 32, 1], G=2, sm_budgets=[0, 16]) as s:
        big, small = mm.mm_ctx_sm_count(s.ctx, 0), mm.mm_ctx_sm_count(s.ctx, 1)
    assert small >= 16 and big + small <= 148 and big >= 120, (big, small)


def test_green_context_sgemm_sp_single_integer(R):
    """HET-2 (132 + 16 SMs): measured profile -> SP-Single split -> run.  At the
    paper's MatrixMul size (6144 rows, P311; K = 1024 here) both devices get
    several waves of 256 x 256 tile pairs, so the profiled per-row cost ratio
    is that of the SM counts (compute-bound, 132/16 = 8.25) and the fast device
    gets ~89 % of the rows (P329: ~90 %).  Integer inputs: sampled rows (every
    boundary row, both devices) bit-exact against the oracle."""
    mm, runner = R
    M, N, K = 6144, 6144, 1024
    A, B = synthgen.matmul_integer(M, K, N)
    with runner.session(mm.MM_APP_SGEMM, [M, N, K, 2, 16, 1], G=2, sm_budgets=[0, 16]) as s:
        s.fill(integer=True)
        prof = s.profile(reps=3)
        ratio = prof.fs_item[1][0] / prof.fs_item[0][0]
        assert 6.0 <= ratio <= 12.0, (ratio, prof.fs_item[0][0], prof.fs_item[1][0])
        assert mm.mm_classify(s.app) == mm.MM_SK_ONE
        plan = s.plan(mm.MM_SP_SINGLE, prof)
        rng = mm.mm_plan_ranges(plan)
        share = (rng[0][1] - rng[0][0]) / M
        assert 0.80 <= share <= 0.95, (share, rng)
        s.run(plan)
        got = s.collect(plan, 2).reshape(M, N)
    cut = rng[0][1]
    rows = sorted({0, 1, 255, 256, cut - 2, cut - 1, cut, cut + 1, M - 2, M - 1} | set(range(3, M, 997)))
    for r in rows:
        assert np.array_equal(got[r], on.sgemm(A, B, r, r + 1)[r]), r


def test_green_context_dp_perf_stream(R):
    """DP-Perf over a HET-2 pair with a measured profile: bit-exact STREAM, and
    the fast device takes most chunks (P119 performance-aware placement)."""
    mm, runner = R
    n = (1 << 22) + 77
    a0, b0, c0 = synthgen.stream_random(n)
    ra, rb, rc = on.stream_run(a0, b0, c0, 1)
    with runner.session(mm.MM_APP_STREAM, [n, 1, 0, 32, 1], G=2, sm_budgets=[0, 16]) as s:
        prof = s.profile(reps=3)
        s.fill()
        plan = s.plan(mm.MM_DP_PERF, prof, chunks_per_dev=8)
        s.run(plan)
        for slot, ref in ((0, ra), (1, rb), (2, rc)):
            assert np.array_equal(s.collect(plan, slot), ref), slot
        ch = mm.mm_plan_chunks(plan)
    # placement follows the measured estimates: when the 132-SM device's
    # chunks are estimated faster for every kernel, it gets at least half
    fast = sum(1 for c in ch if c.device == 0)
    est = [list(prof.chunk_est_ns[d][:4]) for d in range(2)]
    if all(est[0][k] < est[1][k] for k in range(4)):
        assert fast >= len(ch) // 2, (fast, len(ch), est)


def test_green_context_caller_stream(R):
    """mm_ctx_set_stream on a green-context device: the caller's (primary
    context) stream writes the inputs, mm_run waits for it, and a caller
    kernel after the run reads the result, with no host synchronisation in
    between (the join events are recorded in their own stream's context)."""
    import torch
    mm, runner = R
    n = 1 << 20
    a0, b0, c0 = synthgen.stream_random(n)
    ra, _, _ = on.stream_run(a0, b0, c0, 1)
    with runner.session(mm.MM_APP_STREAM, [n, 1, 0, 32, 1], G=2, sm_budgets=[0, 16]) as s:
        plan = s.plan(mm.MM_SP_UNIFIED, mm.make_profile(2, [[1000] * 4, [8000] * 4], [[1] * 4] * 2,
                                                        [10 ** 11] * 2))
        torch.cuda.synchronize()
        cs = torch.cuda.Stream()
        host = [torch.from_numpy(x).pin_memory() for x in (a0, b0, c0)]
        for d in (0, 1):
            mm.mm_ctx_set_stream(s.ctx, d, cs.cuda_stream)
        with torch.cuda.stream(cs):
            for d in (0, 1):
                for slot in range(3):
                    s.bufs[(slot, d)].copy_(host[slot], non_blocking=True)
        s.run(plan)
        with torch.cuda.stream(cs):
            out = s.bufs[(0, 0)].clone()
            out2 = s.bufs[(0, 1)].clone()
        cs.synchronize()
        rng = mm.mm_plan_ranges(plan)
        got = np.empty(n, np.float32)
        got[rng[0][0]:rng[0][1]] = out.cpu().numpy()[rng[0][0]:rng[0][1]]
        got[rng[1][0]:rng[1][1]] = out2.cpu().numpy()[rng[1][0]:rng[1][1]]
        for d in (0, 1):
            mm.mm_ctx_set_stream(s.ctx, d, 0)
    assert np.array_equal(got, ra)


# ------------------------------------------------ Glinda's transfer term ----
def test_profile_host_link_is_pcie(R):
    """measure_link = host (staged mode): link_Bps is a pinned PCIe copy rate
    (P49's R_GD), far below HBM, and the profile is marked staged so the split
    adds the transfer term; the peer (resident) link of logical devices on one
    GPU is a device-to-device copy (> 100 GB/s)."""
    mm, runner = R
    n = 1 << 22
    with runner.session(mm.MM_APP_STREAM, [n, 1, 0, 32, 1], G=2) as s:
        s.fill()
        ph = s.profile(reps=3, link="host")
        pp = s.profile(reps=3, link="peer")
    assert ph.staged == 1 and pp.staged == 0
    for d in range(2):
        assert 5e9 <= ph.link_Bps[d] <= 100e9, ph.link_Bps[d]
        assert pp.link_Bps[d] >= 100e9, pp.link_Bps[d]


def test_staged_split_moves_with_the_link(R):
    """HET-2 STREAM-Seq: with the host link the SP-Unified split differs from
    the resident one by what the link explains — the per-element transfer
    term (16 B / link_Bps) is added to both devices, so the shares move
    toward equal (the slow device's relative compute handicap shrinks)."""
    mm, runner = R
    n = 1 << 24
    with runner.session(mm.MM_APP_STREAM, [n, 1, 0, 32, 1], G=2, sm_budgets=[0, 16]) as s:
        s.fill()
        pr = s.profile(reps=3, link="peer")
        ph = s.profile(reps=3, link="host")
        rr = mm.mm_split(s.app, pr, mm.MM_SP_UNIFIED)[0][0]
        rh = mm.mm_split(s.app, ph, mm.MM_SP_UNIFIED)[0][0]
    fr = (rr[0][1] - rr[0][0]) / n
    fh = (rh[0][1] - rh[0][0]) / n
    # hand model: c_d = sum_k fs[d][k] + 16 B * 1e15 / link_d fs per element
    c = [sum(ph.fs_item[d][k] for k in range(4)) + 16e15 / ph.link_Bps[d] for d in range(2)]
    want = (1 / c[0]) / (1 / c[0] + 1 / c[1])
    assert abs(fh - want) < 1e-3, (fh, want)
    assert fh < fr, (fh, fr)


# -------------------------------------------------- graph key / counters ----
def test_graph_recaptured_after_scratch_grows(R):
    """a captured graph bakes in the device scratch.  A
    DP-Perf plan (small chunks -> small split scratch) is captured, an
    SP-Single plan then grows the scratch (freeing the old one), and the first
    plan's next graph replay must be re-captured on the new scratch: results
    stay bit-exact (integer inputs)."""
    mm, runner = R
    M, N, K = 2048, 512, 256
    A, B = synthgen.matmul_integer(M, K, N)
    ref = on.sgemm(A, B)
    with runner.session(mm.MM_APP_SGEMM, [M, N, K, 2, 16, 1], G=1) as s:
        s.fill(integer=True)
        small = s.plan(mm.MM_DP_PERF, _prof(mm, 1, 1), chunks_per_dev=8)
        big = s.plan(mm.MM_SP_SINGLE, _prof(mm, 1, 1))
        s.run(small, use_graph=True)
        s.run(big, use_graph=True)
        for p in (small, big, small):
            s.bufs[(2, 0)].fill_(float("nan"))
            s.run(p, use_graph=True)
            assert np.array_equal(s.collect(p, 2).reshape(M, N), ref)


def test_graph_staged_new_host_buffers(R):
    """A staged plan replayed as a graph with a second set of host buffers
    reads and writes the second set (host pointers are part of the key)."""
    import torch
    mm, runner = R
    n = 100000
    sets = []
    for seed in (1, 2):
        a0, b0, c0 = synthgen.stream_random(n, seed=seed)
        sets.append(([torch.from_numpy(x.copy()).pin_memory() for x in (a0, b0, c0)],
                     on.stream_run(a0, b0, c0, 1)))
    with runner.session(mm.MM_APP_STREAM, [n, 1, 0, 32, 1], G=2) as s:
        plan = s.plan(mm.MM_SP_UNIFIED, _prof(mm, 2, 4), staged=True)
        # back to the first set: its arrays now hold run 1's outputs (staged
        # runs write in place), so the expected result is one more pass
        again = ([torch.from_numpy(x.copy()).pin_memory() for x in sets[0][1]], on.stream_run(*sets[0][1], 1))
        for host, ref in sets + [again]:
            st = s.run(plan, host=[h.data_ptr() for h in host], use_graph=True)
            assert st.h2d_bytes == 4 * n and st.d2h_bytes == 12 * n
            for h, r in zip(host, ref):
                assert np.array_equal(h.numpy(), r)


def test_launch_counter_counts_kernels(R):
    """n_launches and mm_kernel_launch_count count kernels, not ops, eagerly
    and per graph replay: the 3xTF32 SGEMM of 1024 x 1024 x 1024 is the B
    split (split_bT) and ONE fused launch (A split in the kernel, in-cluster
    split-K reduction); 2048 x 2048 x 1024 (enough tile pairs, no K split)
    issues the operand split and the GEMM — 2 kernels for one op either way;
    STREAM issues one kernel per op."""
    mm, runner = R
    for (M, N, K), want in (((1024, 1024, 1024), 2), ((2048, 2048, 1024), 2)):
        with runner.session(mm.MM_APP_SGEMM, [M, N, K, 2, 128, 1], G=1) as s:
            s.fill()
            plan = s.plan(mm.MM_SP_SINGLE, _prof(mm, 1, 1))
            c0 = mm.mm_kernel_launch_count()
            st = s.run(plan)
            assert st.n_launches == want and mm.mm_kernel_launch_count() - c0 == want, (M, N, K, st.n_launches)
            s.run(plan, use_graph=True)
            c1 = mm.mm_kernel_launch_count()
            st = s.run(plan, use_graph=True)
            assert st.n_launches == want and mm.mm_kernel_launch_count() - c1 == want
    with runner.session(mm.MM_APP_STREAM, [1 << 20, 1, 0, 32, 1], G=1) as s:
        s.fill()
        plan = s.plan(mm.MM_SP_UNIFIED, _prof(mm, 1, 4))
        assert s.run(plan).n_launches == 4


def test_collect_rejects_bad_destination(R):
    mm, runner = R
    with runner.session(mm.MM_APP_STREAM, [1024, 1, 0, 32, 1], G=2) as s:
        plan = s.plan(mm.MM_SP_UNIFIED, _prof(mm, 2, 4))
        s.run(plan)
        with pytest.raises(mm.MMError):
            mm.mm_collect(s.ctx, plan, s.ptrs(), 0, s.bufs[(0, 0)].data_ptr(), 2)


# ------------------------------------------------ halo overlap split (R33) --
@pytest.mark.parametrize("tb,G", [(1, 3), (8, 3), (4, 2)])
def test_hotspot_halo_split_bit_exact(R, tb, G):
    """SP-Single HotSpot with each device range run interior-first (R33):
    bit-identical to the oracle (same cells, same per-cell arithmetic)."""
    mm, runner = R
    rows, cols, iters = 300, 256, 32   # an even number of launches per run: the result is in slot 0
    t0, p = synthgen.hotspot(rows, cols)
    ref = on.hotspot_run(t0, p, iters)
    with runner.session(mm.MM_APP_HOTSPOT, [rows, cols, iters, 1, 1, tb], G=G) as s:
        s.fill()
        plan = s.plan(mm.MM_SP_SINGLE, _prof(mm, G, 1), halo_split=True)
        n_split = len(mm.mm_plan_chunks(plan))
        assert n_split > (iters // tb) * G   # the ranges were cut
        s.run(plan)
        s.run(plan, use_graph=True)           # steady-state program, second pass from the first's output
        got = s.collect(plan, 0).reshape(rows, cols)
    ref2 = on.hotspot_run(ref, p, iters)
    assert np.array_equal(got, ref2)


def test_stencil_reduction_halo_split(R):
    mm, runner = R
    rows, cols, steps = 200, 96, 5
    t0, p = synthgen.hotspot(rows, cols)
    T, rs = on.stencil_reduction_run(t0, p, steps)
    with runner.session(mm.MM_APP_STENCIL_REDUCTION, [rows, cols, steps, 1, 1, 1], G=3) as s:
        s.fill()
        plan = s.plan(mm.MM_SP_VARIED, _prof(mm, 3, 2), halo_split=True)
        s.run(plan)
        got = s.collect(plan, 1).reshape(rows, cols)
        rowsum = s.collect(plan, 3)
    assert np.array_equal(got, T)
    import math
    assert abs(math.fsum(rowsum) - rs[-1]) <= 1e-12 * abs(rs[-1])


# ------------------------------------------------- repeated runs (mm_run repeat) --
@pytest.mark.parametrize("graph", [False, True])
@pytest.mark.parametrize("timing", [False, True])
def test_run_repeat_equals_sequential_runs(R, graph, timing):
    """mm_run_opts.repeat = 3 runs the op program three times back to back (in
    one CUDA graph with use_graph; kernel-timing events become event nodes of
    that graph): STREAM's arrays evolve as after 3 passes, bit for bit; the
    stats count every run; kernel_ms is the last run's (> 0 when timed)."""
    mm, runner = R
    n = 100003
    a0, b0, c0 = synthgen.stream_random(n)
    ref = on.stream_run(a0, b0, c0, 3)
    with runner.session(mm.MM_APP_STREAM, [n, 1, 1, 32, 1], G=2) as s:
        s.fill()
        prof = mm.make_profile(2, [[1000, 1300, 900, 1100]] * 2, [[10 ** 5] * 4] * 2, [10 ** 11] * 2)
        plan = s.plan(mm.MM_SP_UNIFIED, prof)
        one = s.run(plan)
        s.fill()
        st = s.run(plan, use_graph=graph, time_kernels=timing, repeat=3)
        for slot in range(3):
            assert np.array_equal(s.collect(plan, slot), ref[slot]), slot
        assert st.n_launches == 3 * one.n_launches
        launches = sum(st.kernel_launches[d][k] for d in range(2) for k in range(4))
        assert launches == 3 * sum(one.kernel_launches[d][k] for d in range(2) for k in range(4))
        ms = sum(st.kernel_ms[d][k] for d in range(2) for k in range(4))
        assert (ms > 0) == timing
        assert st.device_ms > 0


_FUSED_SCRIPT = r"""
import sys, numpy as np
sys.path.insert(0, {root!r})
import synthgen
from oracle import numeric as on
from paper_conf_icpp_shenvms15_b200 import mm, runner
M, N, K = {M}, {N}, {K}
out = {{}}
for integer in (True, False):
    A, B = (synthgen.matmul_integer if integer else synthgen.matmul_uniform)(M, K, N)
    ref = on.sgemm(A, B)
    with runner.session(mm.MM_APP_SGEMM, [M, N, K, 2, 16, 1], G=1) as s:
        s.fill(integer=integer)
        plan = s.plan(1, mm.make_profile(1, [[1000]], [[10 ** 5]], [10 ** 10]))
        s.run(plan)
        got = s.collect(plan, 2).reshape(M, N)
    if integer:
        assert np.array_equal(got, ref), "integer"
    else:
        assert np.max(np.abs(got - ref) / np.abs(ref)) <= 1e-4, "uniform"
print("ok")
"""


@pytest.mark.parametrize("variant", ["1", "2", "3"])
@pytest.mark.parametrize("shape", [(1024, 1024, 1024), (300, 520, 768)])
def test_sgemm_fused_variants(gpu, variant, shape):
    """The three small-SGEMM kernels (MM_SGEMM_FUSED = 1 pair tiles, 2 single-SM
    tiles with in-kernel B transposition, 3 split_bT + single-SM tiles; a
    fresh process each): integer inputs bit-exact, uniform within 1e-4 of the
    FP64 oracle, including ragged M and N."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, MM_SGEMM_FUSED=variant)
    M, N, K = shape
    r = subprocess.run([sys.executable, "-c", _FUSED_SCRIPT.format(root=root, M=M, N=N, K=K)], env=env, cwd=root,
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "ok" in r.stdout, r.stderr[-2000:]
