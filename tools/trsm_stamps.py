"""Per-leaf timeline of the column TRSM (MM_TRSM_STAMPS): one eager
Cholesky run, then per step the median over CTAs of each phase (us from the
CTA's start).  Development tool."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def run(n, b, path):
    os.environ["MM_TRSM_STAMPS"] = path
    import synthgen
    from paper_conf_icpp_shenvms15_b200 import mm, runner
    T = n // b
    with runner.session(mm.MM_APP_CHOLESKY, [n, b], G=1) as s:
        s.fill()
        prof = mm.make_profile(1, [[1000] * 4], [[10 ** 5] * 4], [10 ** 10])
        plan = s.plan(mm.MM_DP_PERF, prof)
        s.run(plan)


def summary(path):
    rows = [l.strip().split(",") for l in open(path) if l.strip()]
    by = {}
    for r in rows:
        by.setdefault(int(r[0]), []).append([float(x) for x in r[2:]])
    for k in sorted(by):
        a = np.array(by[k])
        med = np.median(a, axis=0)
        ls, le, ms, mt, mc = med[0:8], med[8:16], med[16:24], med[24:32], med[32:40]
        print(f"k={k:2d} ctas={len(a):3d} end={med[40]:7.1f}  leaf start/end: " +
              " ".join(f"{x:5.1f}/{y:5.1f}" for x, y in zip(ls, le)))
        print("      mma start/ts/commit: " + " ".join(f"{x:5.1f}/{y:5.1f}/{z:5.1f}" for x, y, z in zip(ms, mt, mc)))


if __name__ == "__main__":
    path = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/trsm_stamps.csv"
    if os.path.exists(path):
        os.remove(path)
    run(int(os.environ.get("N", 8192)), 1024, path)
    summary(path)
