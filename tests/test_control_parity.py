"""The C++ control plane (libmm.so through its C ABI) against the oracle:
classification, ranking, splits, DP schedules and the op program must be
bit-identical.  Host-only calls: runs on CPU (no GPU needed)."""
import random

import pytest

from oracle import apps as oa
from oracle import control as oc

mm = pytest.importorskip("paper_conf_icpp_shenvms15_b200.mm")


# ------------------------------------------------------------ app builders --
def stream_pair(n, passes=1, sync=0, granule=32, min_items=1):
    app = mm.mm_app_builtin(mm.MM_APP_STREAM, [n, passes, sync, granule, min_items])
    return app, oa.stream(n, passes, sync, granule, min_items)


def hotspot_pair(rows, cols, iters, granule=1, min_items=1, tb=1):
    app = mm.mm_app_builtin(mm.MM_APP_HOTSPOT, [rows, cols, iters, granule, min_items, tb])
    return app, oa.hotspot(rows, cols, iters, granule, min_items, tb)


def stencil_pair(rows, cols, steps, sync=1, granule=1):
    app = mm.mm_app_builtin(mm.MM_APP_STENCIL_REDUCTION, [rows, cols, steps, sync, granule, 1])
    return app, oa.stencil_reduction(rows, cols, steps, sync, granule)


def bs_pair(n, granule=32):
    app = mm.mm_app_builtin(mm.MM_APP_BLACKSCHOLES, [n, granule, 1])
    k = oc.Kernel("bs", n, granule, 1, [oc.Access(0, oc.READ), oc.Access(1, oc.READ), oc.Access(2, oc.READ),
                                        oc.Access(3, oc.WRITE), oc.Access(4, oc.WRITE)])
    return app, oc.App(buffers=[(4, n)] * 5, kernels=[k])


def sgemm_pair(M, N, K, granule=16):
    app = mm.mm_app_builtin(mm.MM_APP_SGEMM, [M, N, K, 1, granule, 1])
    k = oc.Kernel("sgemm", M, granule, 1, [oc.Access(0, oc.READ, K), oc.Access(1, oc.READ, 0),
                                           oc.Access(2, oc.WRITE, N)])
    return app, oc.App(buffers=[(4, M * K), (4, K * N), (4, M * N)], kernels=[k])


def chol_pair(T, b):
    app = mm.mm_app_builtin(mm.MM_APP_CHOLESKY, [T * b, b])
    return app, oa.cholesky_tasks(T, b)


def rand_profile(rnd, G, K, equal=False):
    ps = [[rnd.randint(100, 5000) for _ in range(K)] for _ in range(G)]
    est = [[rnd.randint(1000, 10 ** 6) for _ in range(K)] for _ in range(G)]
    link = [rnd.randint(10 ** 8, 10 ** 12) for _ in range(G)]
    if equal:
        ps = [ps[0]] * G
        est = [est[0]] * G
        link = [link[0]] * G
    po = oc.Profile(G=G, fs_item=ps, chunk_est_ns=est, link_Bps=link)
    pc = mm.make_profile(G, ps, est, link)
    return pc, po


def ops_as_tuples(plan):
    out = []
    for o in mm.mm_plan_ops(plan):
        if o.kind == mm.MM_OPK_KERNEL:
            out.append((oc.OP_KERNEL, o.device, o.kernel, o.iter, o.r.begin, o.r.end))
        elif o.kind == mm.MM_OPK_XFER:
            out.append((oc.OP_XFER, o.device, o.src, o.buffer, o.r.begin, o.r.end))
        elif o.kind == mm.MM_OPK_BARRIER:
            out.append((oc.OP_BARRIER,))
        else:
            out.append((oc.OP_FLUSH, o.device, o.buffer, o.r.begin, o.r.end))
    return out


def oracle_plan(oapp, po, strategy, kpd=8, staged=False, one_shot=True):
    G = po.G
    if strategy in (oc.SP_SINGLE, oc.SP_UNIFIED, oc.SP_VARIED):
        ranges = oc.sp_split(oapp, po, strategy)
        tasks, dev = oc.sp_tasks(oapp, ranges)
        fin = [0] * len(tasks)
    elif strategy == oc.DP_PERF:
        tasks, dev, fin = oc.dp_perf(oapp, po, kpd)
    elif strategy == oc.DP_DEP:
        tasks, dev = oc.dp_dep(oapp, G, kpd)
        fin = [0] * len(tasks)
    elif strategy == oc.DP_STATIC:
        tasks, dev = oc.dp_static(oapp, po, kpd)
        fin = [0] * len(tasks)
    else:
        tasks, dev = oc.sp_cyclic(oapp, G)
        fin = [0] * len(tasks)
    if staged or one_shot:
        ops = oc.op_program(oapp, G, tasks, dev, strategy, staged)
    else:
        ops = oc.steady_program(oapp, G, tasks, dev, strategy)
    return tasks, dev, fin, ops


def check_plan(capp, oapp, pc, po, strategy, kpd=8, staged=False):
    for one_shot in (True, False):
        _check_plan(capp, oapp, pc, po, strategy, kpd, staged, one_shot)


def _check_plan(capp, oapp, pc, po, strategy, kpd, staged, one_shot):
    plan = mm.mm_plan_build(capp, pc, mm.plan_opts(strategy, chunks_per_dev=kpd, staged=staged,
                                                   one_shot=one_shot))
    try:
        tasks, dev, fin, ops = oracle_plan(oapp, po, strategy, kpd, staged, one_shot)
        ch = mm.mm_plan_chunks(plan)
        assert len(ch) == len(tasks)
        assert [c.device for c in ch] == dev
        assert [c.kernel for c in ch] == [t.kernel for t in tasks]
        assert [(c.items.begin, c.items.end) for c in ch] == [(t.begin, t.end) for t in tasks]
        if strategy == oc.DP_PERF:
            assert [c.finish_ns for c in ch] == fin
        assert ops_as_tuples(plan) == ops
        info = mm.mm_plan_info(plan)
        assert info.xfer_bytes == oc.transfer_bytes(oapp, [o for o in ops if o[0] == oc.OP_XFER and o[2] >= 0])
    finally:
        mm.mm_plan_destroy(plan)


# ------------------------------------------------------------------ tests --
def test_abi_struct_sizes_match_header():
    import ctypes
    assert mm.mm_abi_sizes() == [ctypes.sizeof(s) for s in mm.ABI_STRUCTS]


def test_exports_every_declared_symbol():
    import re
    import subprocess
    hdr = open(mm.LIB_PATH.replace("paper_conf_icpp_shenvms15_b200/libmm.so", "include/mm.h")).read()
    declared = set(re.findall(r"^(?:mm_status|void|const char\*|int64_t)\s+(mm_[a-z0-9_]+)\(", hdr, re.M))
    assert len(declared) > 30
    syms = subprocess.run(["nm", "-D", "--defined-only", mm.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (mm_[a-z0-9_]+)", syms))
    assert declared <= exported, declared - exported
    assert set(mm.EXPORTS) <= exported


def test_classify_and_rank_builtin_apps():
    cases = [(stream_pair(100, 1), oc.MK_SEQ), (stream_pair(100, 5), oc.MK_LOOP),
             (hotspot_pair(8, 8, 10), oc.SK_LOOP), (hotspot_pair(8, 8, 1), oc.SK_ONE),
             (stencil_pair(8, 8, 3), oc.MK_LOOP), (bs_pair(64), oc.SK_ONE), (sgemm_pair(64, 8, 8), oc.SK_ONE),
             (chol_pair(3, 2), oc.MK_DAG)]
    for (capp, oapp), cls in cases:
        assert mm.mm_classify(capp) == oc.classify(oapp) == cls
        ns = mm.mm_needs_sync(capp)
        assert ns == oc.needs_sync(oapp)
        assert mm.mm_rank(cls, ns) == oc.rank(cls, ns)
        mm.mm_app_destroy(capp)


def test_classify_custom_flows():
    rnd = random.Random(3)
    for _ in range(300):
        k = rnd.randint(1, 4)
        app = mm.mm_app_create()
        b = mm.mm_app_add_buffer(app, 4, 16)
        for i in range(k):
            mm.mm_app_add_kernel(app, mm.kernel_desc(f"k{i}", mm.MM_OP_STREAM_COPY, 16, [(b, mm.MM_READ, 1, 0)]))
        edges = [(rnd.randrange(k), rnd.randrange(k)) for _ in range(rnd.randint(0, 4))]
        for a, c in edges:
            mm.mm_app_add_edge(app, a, c)
        loop = None
        if rnd.random() < 0.5:
            f = rnd.randrange(k)
            l = rnd.randrange(f, k)
            it = rnd.randint(1, 4)
            mm.mm_app_set_loop(app, f, l, it)
            loop = (f, l, it) if it > 1 else None
        unstable = rnd.random() < 0.2
        mm.mm_app_set_unstable(app, unstable)
        oapp = oc.App(buffers=[(4, 16)], kernels=[oc.Kernel(f"k{i}", 16) for i in range(k)], edges=edges,
                      loop=loop, unstable=unstable)
        assert mm.mm_classify(app) == oc.classify(oapp), (k, edges, loop, unstable)
        mm.mm_app_destroy(app)


def test_split_random_profiles_bit_exact():
    rnd = random.Random(11)
    for trial in range(200):
        G = rnd.randint(1, 8)
        n = rnd.choice([0, 1, 31, 32, 1000, 4099, 1 << 20, (1 << 28) + 5])
        g = rnd.choice([1, 4, 32, 128])
        mn = rnd.choice([1, 1, 64, 100000])
        capp, oapp = stream_pair(n, 1, 0, g, mn)
        pc, po = rand_profile(rnd, G, 4, equal=(trial % 5 == 0))
        for s in (oc.SP_UNIFIED, oc.SP_VARIED):
            got, _ = mm.mm_split(capp, pc, s)
            assert got == oc.sp_split(oapp, po, s), (trial, s)
        mm.mm_app_destroy(capp)


def test_split_stream_2_28_over_8():
    capp, _ = stream_pair(1 << 28, 1, 0, 32, 1)
    pc = mm.make_profile(8, [[1000] * 4] * 8, [[1] * 4] * 8, [1] * 8)
    got, used = mm.mm_split(capp, pc, mm.MM_SP_UNIFIED)
    assert used == 8 and [e - b for b, e in got[0]] == [33554432] * 8
    mm.mm_app_destroy(capp)


def test_matmul_1024_resolves_to_one_gpu():
    # BASELINE configs[0]: 1024^2 fills less than one wave per device -> 1 GPU (P49 decision)
    capp = mm.mm_app_builtin(mm.MM_APP_SGEMM, [1024, 1024, 1024])
    pc = mm.make_profile(8, [[1000]] * 8, [[1]] * 8, [1] * 8)
    got, used = mm.mm_split(capp, pc, mm.MM_SP_SINGLE)
    assert used == 1 and got[0][0] == (0, 1024)
    mm.mm_app_destroy(capp)


@pytest.mark.parametrize("strategy", [oc.SP_UNIFIED, oc.SP_VARIED, oc.DP_PERF, oc.DP_DEP])
@pytest.mark.parametrize("sync", [0, 1, 2])
def test_plan_stream(strategy, sync):
    rnd = random.Random(100 + strategy * 7 + sync)
    for trial in range(6):
        G = rnd.randint(1, 5)
        n = rnd.choice([64, 1000, 4099])
        passes = rnd.choice([1, 2])
        capp, oapp = stream_pair(n, passes, sync, rnd.choice([1, 32]), 1)
        pc, po = rand_profile(rnd, G, 4)
        check_plan(capp, oapp, pc, po, strategy, kpd=rnd.choice([1, 2, 4]))
        mm.mm_app_destroy(capp)


@pytest.mark.parametrize("strategy", [oc.SP_SINGLE, oc.DP_PERF, oc.DP_DEP])
def test_plan_hotspot(strategy):
    rnd = random.Random(7 + strategy)
    for trial in range(5):
        G = rnd.randint(1, 4)
        capp, oapp = hotspot_pair(rnd.randint(8, 40), rnd.choice([4, 7]), rnd.randint(1, 4))
        pc, po = rand_profile(rnd, G, 1)
        check_plan(capp, oapp, pc, po, strategy, kpd=rnd.choice([1, 2, 3]))
        mm.mm_app_destroy(capp)


@pytest.mark.parametrize("strategy", [oc.SP_SINGLE, oc.DP_PERF, oc.DP_DEP])
def test_plan_hotspot_temporal_block(strategy):
    """Temporal blocking: halo tb rows, iters/tb launches."""
    rnd = random.Random(70 + strategy)
    for trial in range(5):
        G = rnd.randint(1, 4)
        tb = rnd.choice([2, 3, 4])
        capp, oapp = hotspot_pair(rnd.randint(8, 40), rnd.choice([4, 8]), tb * rnd.randint(1, 3), tb=tb)
        pc, po = rand_profile(rnd, G, 1)
        check_plan(capp, oapp, pc, po, strategy, kpd=rnd.choice([1, 2, 3]))
        mm.mm_app_destroy(capp)


def test_plan_dp_static_all_range_apps():
    """§V conversion (P565): chunk counts from the static ratio, consecutive
    chunks per device; bit-exact plans (chunks, devices, op program) for
    SK-One, SK-Loop, MK-Seq/MK-Loop (with and without sync) and MK-Loop
    stencil+reduction under random heterogeneous profiles."""
    rnd = random.Random(565)
    makers = [lambda: bs_pair(rnd.randint(50, 900)), lambda: sgemm_pair(rnd.randint(20, 90), 6, 5),
              lambda: hotspot_pair(rnd.randint(8, 40), 4, rnd.randint(1, 3)),
              lambda: stream_pair(rnd.choice([64, 1000, 4099]), rnd.choice([1, 2]), rnd.choice([0, 1, 2]),
                                  rnd.choice([1, 32]), 1),
              lambda: stencil_pair(rnd.randint(8, 30), 5, rnd.randint(1, 3), rnd.choice([0, 1]))]
    for trial in range(12):
        for mk in makers:
            capp, oapp = mk()
            G = rnd.randint(1, 5)
            K = mm.mm_app_info(capp)[0]
            pc, po = rand_profile(rnd, G, K)
            check_plan(capp, oapp, pc, po, oc.DP_STATIC, kpd=rnd.choice([1, 2, 3, 8]))
            mm.mm_app_destroy(capp)


def test_dp_static_counts_follow_the_static_ratio():
    """Worked case: MatrixMul-like SK-One with a 9:1 cost ratio between two
    devices (P329: SP-Single puts ~90% on the GPU) and 10 chunks: the slow
    device gets 1 instance, the fast one 9 (P565 step 2); with 20 chunks, 2
    and 18; the fast device's chunks come first (P565 step 3)."""
    app = oa.single("mm", 1000, granule=1)
    for kpd, want in ((5, (9, 1)), (10, (18, 2))):
        prof = oc.Profile(G=2, fs_item=[[1000], [9000]], chunk_est_ns=[[1], [1]], link_Bps=[1, 1])
        tasks, dev = oc.dp_static(app, prof, kpd)
        assert (dev.count(0), dev.count(1)) == want
        assert dev == sorted(dev)


def test_dp_static_rejects_dag():
    capp = mm.mm_app_builtin(mm.MM_APP_CHOLESKY, [256, 64])
    try:
        with pytest.raises(mm.MMError):
            mm.mm_plan_build(capp, mm.make_profile(2, [[1000] * 4] * 2, [[1000] * 4] * 2, [10 ** 9] * 2),
                             mm.plan_opts(mm.MM_DP_STATIC))
    finally:
        mm.mm_app_destroy(capp)


@pytest.mark.parametrize("ip", [[64, 8, 7, 1, 1, 2], [64, 6, 8, 1, 1, 2], [64, 8, 10, 1, 1, 5]])
def test_hotspot_temporal_block_rejected(ip):
    """iterations % tb != 0, cols % 4 != 0, or an unsupported tb: MM_EINVAL."""
    with pytest.raises(mm.MMError):
        mm.mm_app_builtin(mm.MM_APP_HOTSPOT, ip)


@pytest.mark.parametrize("strategy", [oc.SP_UNIFIED, oc.SP_VARIED, oc.DP_PERF, oc.DP_DEP])
def test_plan_stencil_reduction(strategy):
    rnd = random.Random(17 + strategy)
    for trial in range(4):
        G = rnd.randint(1, 4)
        capp, oapp = stencil_pair(rnd.randint(8, 30), 5, rnd.randint(1, 3), rnd.choice([0, 1, 2]))
        pc, po = rand_profile(rnd, G, 2)
        check_plan(capp, oapp, pc, po, strategy, kpd=2)
        mm.mm_app_destroy(capp)


@pytest.mark.parametrize("strategy", [oc.SP_SINGLE, oc.DP_PERF, oc.DP_DEP])
def test_plan_blackscholes_sgemm(strategy):
    rnd = random.Random(5 + strategy)
    for mk in (lambda: bs_pair(rnd.randint(50, 500)), lambda: sgemm_pair(rnd.randint(20, 90), 6, 5)):
        G = rnd.randint(1, 4)
        capp, oapp = mk()
        pc, po = rand_profile(rnd, G, 1)
        check_plan(capp, oapp, pc, po, strategy, kpd=2)
        mm.mm_app_destroy(capp)


@pytest.mark.parametrize("strategy", [oc.DP_PERF, oc.DP_DEP, oc.SP_CYCLIC])
def test_plan_cholesky(strategy):
    rnd = random.Random(23 + strategy)
    for G in (1, 2, 4, 6):
        capp, oapp = chol_pair(rnd.randint(2, 5), 2)
        pc, po = rand_profile(rnd, G, 4)
        check_plan(capp, oapp, pc, po, strategy)
        mm.mm_app_destroy(capp)


@pytest.mark.parametrize("P", [2, 3, 8])
def test_plan_staged_pipeline(P):
    rnd = random.Random(90 + P)
    for trial in range(4):
        G = rnd.randint(1, 3)
        capp, oapp = stream_pair(rnd.choice([100, 777, 4099]), rnd.choice([1, 2]), 0, 32, 1)
        pc, po = rand_profile(rnd, G, 4)
        plan = mm.mm_plan_build(capp, pc, mm.plan_opts(oc.SP_UNIFIED, staged=True, pipeline=P))
        ranges = oc.sp_split(oapp, po, oc.SP_UNIFIED)
        tasks, dev, flush = oc.sp_tasks_pipelined(oapp, ranges, P)
        ops = oc.op_program(oapp, G, tasks, dev, oc.SP_UNIFIED, True, None, flush)
        ch = mm.mm_plan_chunks(plan)
        assert [c.device for c in ch] == dev
        assert [(c.items.begin, c.items.end) for c in ch] == [(t.begin, t.end) for t in tasks]
        assert ops_as_tuples(plan) == ops
        # every written element is flushed exactly once
        fl = [o for o in ops if o[0] == oc.OP_FLUSH]
        assert sum(o[4] - o[3] for o in fl) == 3 * oapp.kernels[0].n_items
        mm.mm_plan_destroy(plan)
        mm.mm_app_destroy(capp)


@pytest.mark.parametrize("strategy", [oc.SP_UNIFIED, oc.SP_VARIED, oc.DP_PERF])
def test_plan_staged(strategy):
    rnd = random.Random(31 + strategy)
    for trial in range(4):
        G = rnd.randint(1, 4)
        capp, oapp = stream_pair(rnd.choice([100, 777]), rnd.choice([1, 2]), rnd.choice([0, 1]), 32, 1)
        pc, po = rand_profile(rnd, G, 4)
        check_plan(capp, oapp, pc, po, strategy, kpd=2, staged=True)
        mm.mm_app_destroy(capp)


def test_errors_are_status_codes():
    with pytest.raises(mm.MMError) as e:
        mm.mm_rank(99, 0)
    assert e.value.status == mm.MM_EINVAL
    capp, _ = stream_pair(100, 1)
    pc = mm.make_profile(2, [[0] * 4] * 2, [[1] * 4] * 2, [1, 1])
    with pytest.raises(mm.MMError):
        mm.mm_split(capp, pc, mm.MM_SP_UNIFIED)   # zero cost
    with pytest.raises(mm.MMError):
        mm.mm_split(capp, mm.make_profile(2, [[1] * 4] * 2), mm.MM_SP_SINGLE)  # 4 kernels
    mm.mm_app_destroy(capp)


def test_het_k_instance_assignment_matches_p329():
    """HET-k: one fast device + 3 slow ones (6x per-item
    cost), SK-One app, one task instance per device (kpd = 1).  P329:
    DP-Dep "does not take into account their different hardware
    capabilities ... only one task instance is assigned to the GPU";
    DP-Perf "assigns all the task instances to the GPU"; SP-Single splits by
    the capability ratio (6 : 1 : 1 : 1 -> 2/3 on the fast device); DP-Static
    converts that ratio into instance counts (P565)."""
    n, G = 4096, 4
    capp, oapp = bs_pair(n)
    ps = [[1000]] + [[6000]] * 3
    est = [[10 ** 5]] + [[6 * 10 ** 5]] * 3
    link = [10 ** 12] * G
    pc = mm.make_profile(G, ps, est, link)
    po = oc.Profile(G=G, fs_item=ps, chunk_est_ns=est, link_Bps=link)
    try:
        for strategy, kpd in ((oc.DP_DEP, 1), (oc.DP_PERF, 1), (oc.SP_SINGLE, 1), (oc.DP_STATIC, 3)):
            check_plan(capp, oapp, pc, po, strategy, kpd=kpd)
        _, dev = oc.dp_dep(oapp, G, 1)
        assert dev.count(0) == 1                       # one instance on the fast device
        _, dev, _ = oc.dp_perf(oapp, po, 1)
        assert dev.count(0) == len(dev)                # all instances on the fast device
        r = oc.sp_split(oapp, po, oc.SP_SINGLE)[0]
        share = (r[0][1] - r[0][0]) / n
        assert abs(share - 2 / 3) < 0.01
        # SP-Single items [2752, 480, 480, 384] (granule 32); 12 instances:
        # quotas 12*items/n = [8.06, 1.41, 1.41, 1.13] -> floors [8, 1, 1, 1],
        # the one left over to the largest remainder (tie d1/d2 -> d1)
        assert [b - a for a, b in r] == [2752, 480, 480, 384]
        _, dev = oc.dp_static(oapp, po, 3)
        assert [dev.count(d) for d in range(G)] == [8, 2, 1, 1]
        assert dev == sorted(dev)
    finally:
        mm.mm_app_destroy(capp)
