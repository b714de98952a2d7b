import time, statistics, torch
from paper_conf_icpp_shenvms15_b200 import mm, runner
s = runner.session(mm.MM_APP_CHOLESKY, [32768, 1024], G=1)
prof = s.equal_profile()
s.fill()
plan = s.plan(mm.MM_DP_PERF, prof)
for _ in range(2): s.run(plan)
torch.cuda.synchronize()
st_ = s.stream(0)
for tk in (False, True):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    walls, devs = [], []
    e0.record(st_)
    for _ in range(3):
        a = time.perf_counter()
        r = s.run(plan, time_kernels=tk)
        walls.append((time.perf_counter() - a) * 1e3); devs.append(r.device_ms)
    e1.record(st_); torch.cuda.synchronize()
    print("time_kernels", tk, "region/step", e0.elapsed_time(e1) / 3, "wall", [round(x, 2) for x in walls], "device", [round(x, 2) for x in devs], "run.wall_ms", round(r.wall_ms, 2))
