"""C-ABI calls around the app description and the context:
mm_app_finalize (CPU), mm_buffer_register and mm_ctx_set_stream (GPU)."""
import numpy as np
import pytest

import synthgen
from oracle import numeric as on
from paper_conf_icpp_shenvms15_b200 import mm


def _stream_app():
    return mm.mm_app_builtin(mm.MM_APP_STREAM, [1024, 1, 0, 32, 1])


def test_finalize_freezes_the_description():
    app = _stream_app()
    cls = mm.mm_classify(app)
    mm.mm_app_finalize(app)
    mm.mm_app_finalize(app)                       # idempotent
    assert mm.mm_classify(app) == cls == mm.MM_MK_SEQ
    for call in (lambda: mm.mm_app_set_sync(app, 0, mm.MM_SYNC_BARRIER),
                 lambda: mm.mm_app_add_edge(app, 0, 1),
                 lambda: mm.mm_app_set_loop(app, 0, 3, 2),
                 lambda: mm.mm_app_set_unstable(app, 1)):
        with pytest.raises(mm.MMError) as e:
            call()
        assert e.value.status == mm.MM_ESTATE
    mm.mm_app_destroy(app)


def test_finalize_rejects_an_empty_app():
    app = mm.mm_app_create()
    with pytest.raises(mm.MMError) as e:
        mm.mm_app_finalize(app)
    assert e.value.status == mm.MM_EINVAL
    mm.mm_app_destroy(app)


@pytest.fixture(scope="module")
def R():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_icpp_shenvms15_b200 import runner
    return mm, runner


@pytest.mark.gpu
@pytest.mark.parametrize("strategy", [mm.MM_SP_UNIFIED, mm.MM_SP_VARIED, mm.MM_DP_PERF])
def test_registered_buffers(R, strategy):
    """mm_run / mm_collect with buffers = NULL use the registered pointers."""
    _, runner = R
    n = 100003
    a0, b0, c0 = synthgen.stream_random(n)
    ref = on.stream_run(a0, b0, c0, 1)
    with runner.session(mm.MM_APP_STREAM, [n, 1, 0, 32, 1], G=2, register=False) as s:
        s.fill()
        for slot in range(3):
            assert mm.mm_buffer_register(s.ctx, 4, n, [s.bufs[(slot, d)].data_ptr() for d in range(2)]) == slot
        prof = mm.make_profile(2, [[1000, 2000, 1000, 3000], [2000, 1000, 3000, 1000]],
                               [[10 ** 5] * 4] * 2, [10 ** 11] * 2)
        plan = s.plan(strategy, prof, chunks_per_dev=2)
        mm.mm_run(s.ctx, plan, None)
        import torch
        for slot in range(3):
            out = torch.empty(n, dtype=torch.float32, pin_memory=True)
            mm.mm_collect(s.ctx, plan, None, slot, out.data_ptr(), -1)
            assert np.array_equal(out.numpy(), ref[slot])


@pytest.mark.gpu
def test_registered_buffer_shape_mismatch(R):
    _, runner = R
    with runner.session(mm.MM_APP_STREAM, [4096, 1, 0, 32, 1], G=1, register=False) as s:
        for slot in range(3):
            mm.mm_buffer_register(s.ctx, 4, 4096 if slot < 2 else 1024, [s.bufs[(slot, 0)].data_ptr()])
        plan = s.plan(mm.MM_SP_UNIFIED)
        with pytest.raises(mm.MMError) as e:
            mm.mm_run(s.ctx, plan, None)
        assert e.value.status == mm.MM_EINVAL


@pytest.mark.gpu
def test_set_stream_orders_runs_with_a_torch_stream(R):
    """Inputs written by torch on the caller's stream right before mm_run (no
    host synchronisation) are what the run reads, and a torch op queued on
    that stream after mm_run sees the run's results."""
    import torch
    _, runner = R
    n = 1 << 24
    a0, b0, c0 = synthgen.stream_random(n)
    ref = on.stream_run(a0, b0, c0, 1)
    with runner.session(mm.MM_APP_STREAM, [n, 1, 0, 32, 1], G=1) as s:
        plan = s.plan(mm.MM_SP_UNIFIED)
        user = torch.cuda.Stream()
        mm.mm_ctx_set_stream(s.ctx, 0, user.cuda_stream)
        host = [torch.from_numpy(x).pin_memory() for x in (a0, b0, c0)]
        torch.cuda.synchronize()
        for rep in range(2):
            with torch.cuda.stream(user):
                for slot in range(3):
                    s.bufs[(slot, 0)].fill_(float("nan"))        # long queue ahead of the copies
                    s.bufs[(slot, 0)].copy_(host[slot], non_blocking=True)
            s.run(plan)
            with torch.cuda.stream(user):
                got = [s.bufs[(slot, 0)].clone() for slot in range(3)]
            user.synchronize()
            for slot in range(3):
                assert np.array_equal(got[slot].cpu().numpy(), ref[slot]), (rep, slot)
        mm.mm_ctx_set_stream(s.ctx, 0, 0)
