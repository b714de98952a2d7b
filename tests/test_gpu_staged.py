"""Staged (host-resident) execution on the GPU: the pipelined plan (sub-chunks
with H2D / kernels / D2H on separate streams) must give the oracle's results
bit for bit in host memory, and overlap must not change a single byte."""
import numpy as np
import pytest

import synthgen
from oracle import numeric as on

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("P", [1, 4, 8])
@pytest.mark.parametrize("G", [1, 2])
def test_stream_staged_pipeline(gpu, P, G):
    import torch
    from paper_conf_icpp_shenvms15_b200 import mm, runner
    n, passes = (1 << 20) + 96, 2
    a0, b0, c0 = synthgen.stream_random(n)
    ref = on.stream_run(a0, b0, c0, passes)
    with runner.session(mm.MM_APP_STREAM, [n, passes, 0, 32, 1], G=G) as s:
        prof = mm.make_profile(G, [[1000 + 100 * d] * 4 for d in range(G)], [[10 ** 5] * 4] * G, [10 ** 10] * G)
        plan = s.plan(mm.MM_SP_UNIFIED, prof, staged=True, pipeline=P)
        for rep in range(2):                      # inputs re-uploaded every run
            host = [torch.from_numpy(x.copy()).pin_memory() for x in (a0, b0, c0)]
            st = s.run(plan, host=[h.data_ptr() for h in host])
            for h, r in zip(host, ref):
                assert np.array_equal(h.numpy(), r), (P, G, rep)
            assert st.d2h_bytes == 3 * 4 * n
