"""Host-side cost of one bench step (MatrixMul 1024^2, SP-Single) broken
down per call: wall time per call averaged over many steps (GPU box)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_icpp_shenvms15_b200 import mm, runner  # noqa: E402


def main(n=300):
    s = runner.session(mm.MM_APP_SGEMM, [1024, 1024, 1024, 0], G=1)
    prof = s.profile(reps=3)
    s.fill()
    plan = s.plan(mm.MM_SP_SINGLE, prof)
    T = {}

    def tm(name, f):
        a = time.perf_counter_ns()
        r = f()
        T[name] = T.get(name, 0) + time.perf_counter_ns() - a
        return r

    for _ in range(10):
        s.run(plan, time_kernels=True)
    torch.cuda.synchronize()
    for _ in range(n):
        c = tm("classify", lambda: mm.mm_classify(s.app))
        ns = tm("needs_sync", lambda: mm.mm_needs_sync(s.app))
        tm("rank", lambda: mm.mm_rank(c, ns))
        tm("split", lambda: mm.mm_split(s.app, prof, mm.MM_SP_SINGLE))
        p = tm("ptrs", lambda: s.ptrs())
        st = tm("mm_run(timed)", lambda: mm.mm_run(s.ctx, plan, p, time_kernels=True))
        tm("stats", lambda: [st.kernel_ms[0][0], st.n_launches])
    for _ in range(n):
        tm("mm_run(untimed)", lambda: mm.mm_run(s.ctx, plan, p))
        tm("mm_run(graph)", lambda: mm.mm_run(s.ctx, plan, p, use_graph=True))
    torch.cuda.synchronize()
    for _ in range(n):   # the bench's timed steps: registered buffers, graph, enqueue only
        tm("mm_run(graph,no_wait)", lambda: mm.mm_run(s.ctx, plan, None, use_graph=True, no_wait=True))
    torch.cuda.synchronize()
    for k, v in T.items():
        print(f"{k:18s} {v / n / 1000:8.2f} us")
    print("device ms (last timed run)", st.device_ms, "kernel ms", st.kernel_ms[0][0])


if __name__ == "__main__":
    main()
