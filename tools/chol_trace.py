"""Summarise an MM_TRACE timeline of one Cholesky run: per step k, the
lane-1 critical path (POTRF, TRSM) and the lane-0 updates (SYRK, GEMM)."""
import collections
import sys


def main(path):
    rows = [l.strip().split(",") for l in open(path) if l.strip()]
    # keep the last run only: start times restart near 0
    runs, cur, last = [], [], -1.0
    for r in rows:
        t0 = float(r[6])
        if cur and t0 < last - 1.0 and t0 < 1.0:
            runs.append(cur)
            cur = []
        cur.append(r)
        last = t0
    runs.append(cur)
    run = runs[-1]
    end = max(float(r[7]) for r in run)
    per = collections.defaultdict(lambda: collections.defaultdict(float))
    span = collections.defaultdict(lambda: [1e30, 0.0])
    for name, i, j, k, dev, ntask, a, z in run:
        k = int(k)
        a, z = float(a), float(z)
        per[k][name] += z - a
        s = span[k]
        s[0], s[1] = min(s[0], a), max(s[1], z)
    print(f"run end {end:.2f} ms; {len(run)} launches")
    print(" k   start     end   potrf   trsm   syrk   gemm")
    for k in sorted(per):
        p = per[k]
        print(f"{k:2d} {span[k][0]:7.2f} {span[k][1]:7.2f} {p['potrf']:7.3f} {p['trsm']:6.3f} {p['syrk']:6.3f} {p['gemm']:6.3f}")


if __name__ == "__main__":
    main(sys.argv[1])
