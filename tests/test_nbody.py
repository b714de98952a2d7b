"""Nbody (the paper's second SK-Loop app, Table II P223-227, P319): control
plane against the oracle on CPU, CUDA path against the oracle on GPU."""
import numpy as np
import pytest

import synthgen
from oracle import apps as oa
from oracle import control as oc
from oracle import numeric as on

mm = pytest.importorskip("paper_conf_icpp_shenvms15_b200.mm")


def _pair(n, iters):
    return mm.mm_app_builtin(mm.MM_APP_NBODY, [n, iters, 32, 1]), oa.nbody(n, iters, 32, 1)


@pytest.mark.parametrize("strategy", [oc.SP_SINGLE, oc.DP_PERF, oc.DP_DEP])
def test_nbody_plan_matches_oracle(strategy):
    from test_control_parity import check_plan, rand_profile
    import random
    rnd = random.Random(strategy)
    for G in (1, 2, 3):
        capp, oapp = _pair(rnd.randint(40, 300), rnd.randint(1, 3))
        assert mm.mm_classify(capp) == oc.classify(oapp)
        pc, po = rand_profile(rnd, G, 1)
        check_plan(capp, oapp, pc, po, strategy, kpd=2)
        mm.mm_app_destroy(capp)


def test_nbody_all_gather_volume():
    # SP-Single on G devices: every iteration after the first pulls all the
    # positions a device does not own (an all-gather through the directory).
    n, iters, G = 256, 3, 4
    capp, oapp = _pair(n, iters)
    prof = mm.make_profile(G, [[1000]] * G, [[1]] * G, [10 ** 9] * G)
    plan = mm.mm_plan_build(capp, prof, mm.plan_opts(mm.MM_SP_SINGLE, one_shot=True))
    info = mm.mm_plan_info(plan)
    assert info.xfer_bytes == (iters - 1) * G * (n - n // G) * 16
    mm.mm_plan_destroy(plan)
    mm.mm_app_destroy(capp)


@pytest.mark.gpu
@pytest.mark.parametrize("strategy", [1, 4, 5])
@pytest.mark.parametrize("G", [1, 3])
def test_nbody_gpu_vs_oracle(gpu, strategy, G):
    from paper_conf_icpp_shenvms15_b200 import runner
    n, iters = 2048 + 33, 3
    pos, vel = synthgen.nbody(n)
    rp, rv = on.nbody_run(pos, vel, iters)
    with runner.session(mm.MM_APP_NBODY, [n, iters, 32, 1], G=G) as s:
        s.fill()
        assert np.array_equal(s.bufs[(0, 0)].cpu().numpy().reshape(n, 4), pos)   # device generator
        prof = mm.make_profile(G, [[1000 + 300 * d] for d in range(G)], [[10 ** 5]] * G, [10 ** 11] * G)
        plan = s.plan(strategy, prof, chunks_per_dev=2)
        s.run(plan)
        slot_p, slot_v = (1, 3) if iters % 2 else (0, 2)
        gp = s.collect(plan, slot_p).reshape(n, 4)
        gv = s.collect(plan, slot_v).reshape(n, 4)
    # Element by element: FP32 (rsqrt.approx, FMA, summation over n bodies)
    # vs the FP64 oracle.  The error of a sum is bounded relative to the sum
    # of the ABSOLUTE values of its terms, not to its value (which cancels), so
    # each component's tolerance scales with |v| + dt * A_i, where A_i =
    # sum_j m_j |d_ij| / (|d_ij|^2 + eps^2)^{3/2} (per component, FP64, from
    # the initial state), and for positions with |x| + dt |v| + dt^2 A_i.
    dt, eps2 = on.NBODY_DT, on.NBODY_EPS2
    P = pos.astype(np.float64)
    Aabs = np.zeros((n, 3))
    for i0 in range(0, n, 256):
        d = P[None, :, :3] - P[i0:i0 + 256, None, :3]
        r2 = (d * d).sum(-1) + eps2
        Aabs[i0:i0 + 256] = (np.abs(d) * (P[None, :, 3] / r2 ** 1.5)[..., None]).sum(1)
    sv = np.abs(rv[:, :3]) + dt * iters * Aabs
    sp = np.abs(rp[:, :3]) + dt * iters * np.abs(rv[:, :3]) + dt * dt * iters * Aabs
    ev = np.abs(gv[:, :3] - rv[:, :3]) / sv
    ep = np.abs(gp[:, :3] - rp[:, :3]) / sp
    assert ev.max() <= 2e-5 and ep.max() <= 2e-6, (ev.max(), ep.max())
    assert np.array_equal(gp[:, 3], pos[:, 3]) and np.all(gv[:, 3] == 0)


@pytest.mark.gpu
def test_nbody_partition_invariance(gpu):
    """A body's sum runs over all j in the same order on every device, so any
    partitioning gives bit-identical results."""
    from paper_conf_icpp_shenvms15_b200 import runner
    n, iters = 3000, 2
    outs = []
    for G, strategy in ((1, 1), (3, 1), (2, 5), (3, 4)):
        with runner.session(mm.MM_APP_NBODY, [n, iters, 32, 1], G=G) as s:
            s.fill()
            prof = mm.make_profile(G, [[1000 + 500 * d] for d in range(G)], [[10 ** 5]] * G, [10 ** 11] * G)
            plan = s.plan(strategy, prof, chunks_per_dev=3)
            s.run(plan)
            outs.append(s.collect(plan, 0))
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])


@pytest.mark.parametrize("eps2", [-1.0, 1e-40])
def test_nbody_rejects_non_normal_softening(eps2):
    """The kernel's rsqrt.approx.ftz equals rsqrtf only for normal d2 >= eps2
    (include/mm.h MM_APP_NBODY): a negative or denormal eps^2 is MM_EINVAL."""
    with pytest.raises(mm.MMError):
        mm.mm_app_builtin(mm.MM_APP_NBODY, [64, 1, 32, 1], [1e-3, eps2])
