"""Pins of the control-plane oracle (oracle/control.py) against the paper:
Table II classifications, Table I + Propositions 1-3, the printed partition
pairs (P329, P391, P521), footnote 5 rounding, brute-force makespan optima,
closed-form dynamic schedules and per-element re-sync sets.  CPU only."""
import itertools

import pytest

from oracle import apps
from oracle import control as oc


# ------------------------------------------------------ c1 classification ---
def test_table2_classes():
    # Table II (P205-247): MatrixMul, BlackScholes -> SK-One; Nbody, HotSpot ->
    # SK-Loop; STREAM-Seq -> MK-Seq; STREAM-Loop -> MK-Loop.
    assert oc.classify(apps.single("matmul", 6144)) == oc.SK_ONE
    assert oc.classify(apps.single("blackscholes", 80530632)) == oc.SK_ONE
    assert oc.classify(apps.single("nbody", 1 << 20, iters=10)) == oc.SK_LOOP
    assert oc.classify(apps.hotspot(64, 64, 1000)) == oc.SK_LOOP
    assert oc.classify(apps.stream(1000, 1)) == oc.MK_SEQ
    assert oc.classify(apps.stream(1000, 10)) == oc.MK_LOOP
    assert oc.classify(apps.stencil_reduction(64, 64, 100)) == oc.MK_LOOP
    assert oc.classify(apps.cholesky_tasks(4, 2)) == oc.MK_DAG


def test_unstable_sk_loop_becomes_mk_seq():
    # P117: "we can regard each iteration of the kernel as a different kernel,
    # thus turning a SK-Loop application into a MK-Seq application".
    app = apps.hotspot(8, 8, 10)
    app.unstable = True
    assert oc.classify(app) == oc.MK_SEQ


def test_partial_loop_is_unrolled():
    # P115: a loop over some kernels of an MK app does not change its class.
    app = apps.stream(100, 1)
    app.loop = (1, 2, 5)
    assert oc.classify(app) == oc.MK_SEQ


def _brute_class(k, edges, iters):
    # Independent statement of Fig 3: one kernel -> I/II by loop; several ->
    # sequence (every kernel has <=1 successor and <=1 predecessor and they are
    # all connected in one line) -> III/IV by loop, else V.
    if k == 1:
        return oc.SK_LOOP if iters > 1 else oc.SK_ONE
    for perm in itertools.permutations(range(k)):
        line = {(perm[i], perm[i + 1]) for i in range(k - 1)}
        if set(e for e in edges if e[0] != e[1]) == line:
            return oc.MK_LOOP if iters > 1 else oc.MK_SEQ
    return oc.MK_DAG


@pytest.mark.parametrize("k", [1, 2, 3])
def test_classify_exhaustive_small(k):
    pairs = [(a, b) for a in range(k) for b in range(k) if a != b]
    for r in range(len(pairs) + 1):
        for es in itertools.combinations(pairs, r):
            if not es and k > 1:
                continue  # R1: no edges = implicit id-order sequence (tested below)
            for iters in (1, 3):
                app = oc.App(buffers=[(4, 4)], kernels=[oc.Kernel(f"k{i}", 4) for i in range(k)],
                             edges=list(es), loop=(0, k - 1, iters) if iters > 1 else None)
                assert oc.classify(app) == _brute_class(k, list(es), iters), (k, es, iters)


def test_implicit_sequence():
    app = oc.App(buffers=[(4, 4)], kernels=[oc.Kernel("a", 4), oc.Kernel("b", 4)])
    assert oc.classify(app) == oc.MK_SEQ


# ------------------------------------------------------------- c2 ranking ---
def _before(lst, a, b):
    return lst.index(a) < lst.index(b)


def test_ranking_props():
    for cls in (oc.SK_ONE, oc.SK_LOOP, oc.MK_SEQ, oc.MK_LOOP, oc.MK_DAG):
        for s in (False, True):
            r = oc.rank(cls, s)
            # Proposition 1: DP-Perf >= DP-Dep for all classes.
            assert _before(r, oc.DP_PERF, oc.DP_DEP)
    for cls in (oc.SK_ONE, oc.SK_LOOP):   # Proposition 2
        assert oc.rank(cls, False) == [oc.SP_SINGLE, oc.DP_PERF, oc.DP_DEP]
    for cls in (oc.MK_SEQ, oc.MK_LOOP):   # Proposition 3 (1) and (2)
        assert oc.rank(cls, False) == [oc.SP_UNIFIED, oc.DP_PERF, oc.DP_DEP, oc.SP_VARIED]
        assert oc.rank(cls, True) == [oc.SP_VARIED, oc.DP_PERF, oc.DP_DEP, oc.SP_UNIFIED]
    # P201: for MK-DAG "we recommend the use of dynamic partitioning".
    assert oc.rank(oc.MK_DAG, False) == [oc.DP_PERF, oc.DP_DEP]


# ---------------------------------------------------------- c3 split model --
def _beta(r_gc, r_gd, n=10 ** 6, g=32):
    # device 0 = "GPU": t_G = 1000 ps, x_G = R_GD t_G; device 1 = "CPU": t_C = R_GC t_G
    tg = 10 ** 6
    cost = [tg + int(round(r_gd * tg)), int(round(r_gc * tg))]
    rng = oc.split_items(n, g, cost, 1)
    return (rng[0][1] - rng[0][0]) / n


def test_glinda_pairs_blackscholes():
    # P391: transfer = 37.5x kernel (R_GD = 37.5) and 59% on the GPU; the
    # closed form beta = R_GC/(1+R_GC+R_GD) then needs R_GC = 55.40.
    assert abs(_beta(55.40, 37.5) - 0.59) < 1e-3


def test_glinda_pairs_stream():
    # P521: transfer ~88% of GPU time (R_GD = 0.88/0.12 = 7.33), 44% on GPU.
    r_gd = 0.88 / 0.12
    r_gc = 0.44 * (1 + r_gd) / (1 - 0.44)
    assert abs(r_gc - 6.55) < 0.01
    assert abs(_beta(r_gc, r_gd) - 0.44) < 1e-3


def test_glinda_pairs_matrixmul():
    # P329: ~90% on the GPU with a negligible transfer (R_GD ~ 0) <-> R_GC = 9.
    assert abs(_beta(9.0, 0.0) - 0.9) < 1e-3


def test_footnote5_two_device_rounding():
    # P379 fn 5: n_g rounded UP to a multiple of the warp size, n_c = n - n_g.
    n, g = 1000, 32
    cost = [10 ** 6, 3 * 10 ** 6]          # beta = 0.75 -> 750 -> round up 768
    r = oc.split_items(n, g, cost, 1)
    assert r[0] == (0, 768) and r[1] == (768, 1000)


def test_equal_profile_stream_8gpu():
    r = oc.split_items(1 << 28, 32, [1000] * 8, 1)
    assert [e - b for b, e in r] == [33554432] * 8


def _makespan(shares, cost):
    return max(s * c for s, c in zip(shares, cost))


@pytest.mark.parametrize("G", [1, 2, 3])
def test_split_near_bruteforce_optimum(G):
    g = 4
    for n in (1, 7, 64, 127, 255):
        for cost in itertools.product((3, 5, 11), repeat=G):
            r = oc.split_items(n, g, list(cost), 1)
            shares = [e - b for b, e in r]
            assert sum(shares) == n
            best = None
            units = -(-n // g)
            for parts in itertools.product(range(units + 1), repeat=G - 1):
                s = [p * g for p in parts]
                if sum(s) > n:
                    continue
                s.append(n - sum(s))
                m = _makespan(s, cost)
                best = m if best is None else min(best, m)
            assert _makespan(shares, cost) <= best + max(g * c for c in cost)


def test_split_invariants_random():
    import random
    rnd = random.Random(7)
    for _ in range(500):
        G = rnd.randint(1, 8)
        g = rnd.choice([1, 4, 32, 128])
        n = rnd.randint(0, 10 ** 7)
        cost = [rnd.randint(1, 10 ** 9) for _ in range(G)]
        r = oc.split_items(n, g, cost, 1)
        shares = [e - b for b, e in r]
        assert sum(shares) == n
        used = [d for d in range(G) if shares[d] > 0]
        assert all(shares[d] % g == 0 for d in used[:-1])
        # contiguous in id order
        pos = 0
        for d in used:
            assert r[d][0] == pos
            pos = r[d][1]


def test_split_decision_drops_slow_device():
    # P49 decision: a share below one wave drops the slowest device; config[0]
    # (1024 rows, 128-row granule, one wave = 1024 rows) resolves to one GPU.
    r = oc.split_items(1024, 128, [100, 100], 1024)
    assert r == [(0, 1024), (0, 0)]
    r = oc.split_items(1024, 128, [300, 100], 600)
    assert r == [(0, 0), (0, 1024)]


def test_sp_unified_vs_varied():
    app = apps.stream(1 << 12, 1)
    prof = oc.Profile(G=2, fs_item=[[10, 20, 30, 40], [20, 20, 20, 20]],
                      chunk_est_ns=[[1] * 4] * 2, link_Bps=[10 ** 9] * 2)
    u = oc.sp_split(app, prof, oc.SP_UNIFIED)
    assert all(r == u[0] for r in u)
    v = oc.sp_split(app, prof, oc.SP_VARIED)
    # copy: device 0 twice as fast -> ~2/3; triad: device 1 twice as fast -> ~1/3
    assert v[0][0][1] > v[3][0][1]
    with pytest.raises(ValueError):
        oc.sp_split(app, prof, oc.SP_SINGLE)


def test_staged_unified_mk_loop_drops_transfer():
    # P549: "the data transfer is not profiled" for MK-Loop SP-Unified.
    seq, loop = apps.stream(1 << 12, 1), apps.stream(1 << 12, 10)
    prof = oc.Profile(G=2, fs_item=[[10] * 4, [40] * 4], chunk_est_ns=[[1] * 4] * 2,
                      link_Bps=[10 ** 9, 10 ** 15], staged=True)
    s = oc.sp_split(seq, prof, oc.SP_UNIFIED)[0]
    l = oc.sp_split(loop, prof, oc.SP_UNIFIED)[0]
    assert s[0][1] < l[0][1]


# ------------------------------------------------------------- c4 DP-Perf --
def test_dp_perf_identical_devices_round_robin():
    app = apps.single("bs", 1 << 14)
    prof = oc.Profile(G=4, fs_item=[[1]] * 4, chunk_est_ns=[[1000]] * 4, link_Bps=[10 ** 9] * 4)
    tasks, dev, _ = oc.dp_perf(app, prof, 8)
    assert len(tasks) == 32
    assert dev == [i % 4 for i in range(32)]


def test_dp_perf_slow_device_gets_nothing():
    # P329: DP-Perf assigns all MatrixMul task instances to the (much faster) GPU.
    app = apps.single("mm", 6144, granule=1)
    prof = oc.Profile(G=2, fs_item=[[1], [1]], chunk_est_ns=[[1000], [10 ** 9]], link_Bps=[1] * 2)
    _, dev, _ = oc.dp_perf(app, prof, 8)
    assert set(dev) == {0}


def test_dp_perf_ratio_matches_sp_single():
    # P387: "DP-Perf detects similar partitioning as SP-Single".
    n, k = 1 << 16, 16
    for ratio in (2, 3, 5):
        app = apps.single("bs", n)
        prof = oc.Profile(G=2, fs_item=[[100], [100 * ratio]],
                          chunk_est_ns=[[1000], [1000 * ratio]], link_Bps=[10 ** 9] * 2)
        _, dev, _ = oc.dp_perf(app, prof, k)
        cs = oc.chunk_size(n, 32, 2 * k)
        sp = oc.sp_split(app, prof, oc.SP_SINGLE)[0]
        assert abs(dev.count(0) * cs - (sp[0][1] - sp[0][0])) <= cs


def test_dp_perf_respects_dependencies_hand_schedule():
    # 2 devices, STREAM with 2 chunks per kernel (k=1); est 10 ns per chunk,
    # link so slow that moving data never pays: each chain stays put.
    app = apps.stream(64, 1)
    prof = oc.Profile(G=2, fs_item=[[1] * 4] * 2, chunk_est_ns=[[10] * 4] * 2, link_Bps=[1, 1])
    tasks, dev, fin = oc.dp_perf(app, prof, 1)
    assert dev == [0, 1] * 4
    assert fin == [10, 10, 20, 20, 30, 30, 40, 40]


# -------------------------------------------------------------- c5 DP-Dep --
def test_dp_dep_stream_chains():
    G, k = 4, 2
    app = apps.stream(1024, 3)
    tasks, dev = oc.dp_dep(app, G, k)
    C = G * k
    for t, task in enumerate(tasks):
        chunk = (task.begin // oc.chunk_size(1024, 32, C))
        assert dev[t] == chunk % G


def test_dp_dep_sk_one_round_robin():
    _, dev = oc.dp_dep(apps.single("x", 1000), 3, 4)
    assert dev == [i % 3 for i in range(len(dev))]


def test_dp_dep_halo_does_not_chain():
    # A stencil chunk chains to the same chunk of the previous iteration (WAW on
    # its own rows), never to the halo neighbours.
    app = apps.hotspot(64, 8, 4)
    tasks, dev = oc.dp_dep(app, 2, 2)
    per_iter = 4
    for t in range(per_iter, len(tasks)):
        assert dev[t] == dev[t - 2 * per_iter] if t >= 2 * per_iter else True
    # iterations 0 and 1 write different buffers (ping-pong): round-robin seeds both
    assert dev[:8] == [0, 1, 0, 1, 0, 1, 0, 1]


def test_dp_dep_cholesky_tile_ownership():
    app = apps.cholesky_tasks(4, 1)
    tasks, dev = oc.dp_dep(app, 2)
    last = {}
    for t, task in enumerate(tasks):
        w = [a for a in task.accesses if a.mode & oc.WRITE][0].lo
        if w in last:
            assert dev[t] == last[w]
        last[w] = dev[t]


# --------------------------------------------------- c6 op program / re-sync --
def _interval_resync(P, Q, halo, nb):
    # c6 transfer set {(e -> d, P_e ∩ Q_d^h)}: independent interval arithmetic.
    out = []
    for d, (qb, qe) in enumerate(Q):
        if qe <= qb:
            continue
        lo, hi = max(0, qb - halo), min(nb, qe + halo)
        for e, (pb, pe) in enumerate(P):
            if e == d:
                continue
            a, b = max(lo, pb), min(hi, pe)
            if a < b:
                out.append((e, d, a, b))
    return sorted(out)


def test_sp_varied_resync_matches_interval_formula():
    n = 1000
    app = apps.stream(n, 1)
    prof = oc.Profile(G=3, fs_item=[[10, 30, 20, 10], [20, 10, 20, 30], [30, 20, 10, 20]],
                      chunk_est_ns=[[1] * 4] * 3, link_Bps=[10 ** 9] * 3)
    ranges = oc.sp_split(app, prof, oc.SP_VARIED)
    tasks, dev = oc.sp_tasks(app, ranges)
    ops = oc.op_program(app, 3, tasks, dev, oc.SP_VARIED)
    x = sorted((o[2], o[1], o[4], o[5]) for o in ops if o[0] == oc.OP_XFER and o[3] == 2)
    # buffer c: written by copy (ranges[0]) read by scale (ranges[1]); rewritten
    # by add (ranges[2]) read by triad (ranges[3]).
    want = _interval_resync(ranges[0], ranges[1], 0, n) + _interval_resync(ranges[2], ranges[3], 0, n)
    assert x == sorted(want)
    assert sum(1 for o in ops if o[0] == oc.OP_BARRIER) == 3


def test_sp_unified_no_transfers():
    app = apps.stream(1000, 3)
    prof = oc.Profile(G=4, fs_item=[[7, 9, 11, 13]] * 4, chunk_est_ns=[[1] * 4] * 4,
                      link_Bps=[10 ** 9] * 4)
    ranges = oc.sp_split(app, prof, oc.SP_UNIFIED)
    tasks, dev = oc.sp_tasks(app, ranges)
    ops = oc.op_program(app, 4, tasks, dev, oc.SP_UNIFIED)
    assert not any(o[0] in (oc.OP_XFER, oc.OP_BARRIER) for o in ops)
    assert sum(1 for o in ops if o[0] == oc.OP_KERNEL) == 4 * 4 * 3


def test_hotspot_halo_rows():
    rows, cols, iters, G = 40, 8, 5, 4
    app = apps.hotspot(rows, cols, iters)
    prof = oc.Profile(G=G, fs_item=[[5]] * G, chunk_est_ns=[[1]] * G, link_Bps=[10 ** 9] * G)
    ranges = oc.sp_split(app, prof, oc.SP_SINGLE)
    assert [e - b for b, e in ranges[0]] == [10] * 4
    tasks, dev = oc.sp_tasks(app, ranges)
    ops = oc.op_program(app, G, tasks, dev, oc.SP_SINGLE)
    xs = [o for o in ops if o[0] == oc.OP_XFER]
    # iterations 1..4 each move one ghost row per internal boundary per direction
    assert len(xs) == (iters - 1) * 2 * (G - 1)
    assert all(o[5] - o[4] == cols for o in xs)


def test_replay_decision_rule():
    # earliest finish wins; a busier device loses; ties go to the lowest id
    assert oc.replay_decision([0, 0], [0, 0], [10, 5])[0] == 1
    assert oc.replay_decision([100, 0], [0, 0], [10, 50])[0] == 1
    assert oc.replay_decision([0, 0], [0, 0], [7, 7])[0] == 0
    assert oc.replay_decision([0, 0], [30, 0], [10, 25]) == (1, [40, 25])
