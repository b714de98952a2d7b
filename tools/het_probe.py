import numpy as np, torch, sys, time
sys.path.insert(0, __import__('os').path.dirname(__import__('os').path.dirname(__import__('os').path.abspath(__file__))))
import synthgen
from oracle import numeric as on
from paper_conf_icpp_shenvms15_b200 import mm, runner
n = 1 << 24
a0, b0, c0 = synthgen.stream_random(n)
ref = on.stream_run(a0, b0, c0, 1)
try:
    s = runner.session(mm.MM_APP_STREAM, [n, 1, 0, 32, 1], G=2, sm_budgets=[0, 16])
except Exception as e:
    print("ctx fail", e); raise
print("sms", mm.mm_ctx_sm_count(s.ctx, 0), mm.mm_ctx_sm_count(s.ctx, 1))
s.fill()
prof = s.profile(reps=3)
print("ps", [list(prof.fs_item[d][:4]) for d in range(2)], "est", [list(prof.chunk_est_ns[d][:4]) for d in range(2)], "link", list(prof.link_Bps[:2]))
for strat in (2, 3, 4, 5):
    s.fill()
    p = s.plan(strat, prof)
    st = s.run(p)
    ok = all(np.array_equal(s.collect(p, k), ref[k]) for k in range(3))
    info = mm.mm_plan_info(p)
    print(mm.mm_strategy_name(strat), "ok" if ok else "MISMATCH", "ms", st.device_ms, "ranges", mm.mm_plan_ranges(p)[:2], "items d0/d1", info.items[0][0], info.items[1][0])
s.close()
