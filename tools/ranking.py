"""E6: does the paper's Table I ranking hold on B200?  (PAPER.md P549, P565)

Runs every Table I strategy of each application class on
  * HET-2: two logical devices on one B200, a "GPU" of 132 SMs and a "CPU" of
    16 SMs (CUDA green contexts) — 148/16 = 9.25, the K20m/E5-2620 SP peak
    ratio of Table III is 3519.3/384 = 9.16 (P277-281);
  * HOMO-2: two logical devices of the whole GPU each (identical processors),
in resident mode (inputs in HBM) and, for the transfer-dominated MK apps,
staged mode (inputs on the host, P119 H2D/D2H in the run; the paper's regime).

Writes one JSON document (default profiles/r1_ranking.json): per config the
median device time of every strategy, the devices' item shares, and whether
the measured order satisfies Propositions 1-3 (ties within 3% count as "=").

    python tools/ranking.py [--out FILE] [--reps 3] [--quick]
"""
import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_icpp_shenvms15_b200 import mm, runner  # noqa: E402

TOL = 0.03

# (name, builtin id, iparam) — paper sizes where they fit (P311, P319, P473)
APPS = [
    ("MatrixMul 6144^2 (SK-One)", mm.MM_APP_SGEMM, [6144, 6144, 6144, 0, 128, 128]),
    ("BlackScholes 80,530,632 (SK-One)", mm.MM_APP_BLACKSCHOLES, [80530632, 32, 4096]),
    ("HotSpot 8192^2 x 100 (SK-Loop)", mm.MM_APP_HOTSPOT, [8192, 8192, 100, 1, 64]),
    ("STREAM-Seq 62,914,560 w/o sync (MK-Seq)", mm.MM_APP_STREAM, [62914560, 1, 0, 32, 4096]),
    ("STREAM-Seq 62,914,560 w sync (MK-Seq)", mm.MM_APP_STREAM, [62914560, 1, 1, 32, 4096]),
    ("STREAM-Loop x10 w/o sync (MK-Loop)", mm.MM_APP_STREAM, [62914560, 10, 0, 32, 4096]),
    ("STREAM-Loop x10 w sync (MK-Loop)", mm.MM_APP_STREAM, [62914560, 10, 1, 32, 4096]),
    ("stencil+reduction 8192^2 x 20 w sync (MK-Loop)", mm.MM_APP_STENCIL_REDUCTION, [8192, 8192, 20, 2, 1, 64]),
    ("Cholesky 8192^2 tile 512 (MK-DAG)", mm.MM_APP_CHOLESKY, [8192, 512]),
]


# SM budgets per logical device (0 = the rest of the GPU).  HET-k (SURVEY
# §8(f) f2): one fast device + m slow ones, the paper's GPU + CPU-worker mix
# (P329: DP-Dep "uses all the CPU cores and the GPU" as equal workers).
# PART-k: k equal green contexts with disjoint SMs (the GPU's remaining SMs
# idle) — identical processors that, unlike HOMO-k, do not share SMs; only
# HBM is still shared.
PLATFORMS = {"HET-2": [0, 16], "HOMO-2": [0, 0], "HET-4": [0, 16, 16, 16], "HOMO-4": [0, 0, 0, 0],
             "HET-8": [0, 8, 8, 8, 8, 8, 8, 8],
             "PART-2": [72, 72], "PART-4": [32, 32, 32, 32], "PART-8": [16] * 8}


def expected_order(cls, sync):
    return mm.mm_rank(cls, sync)


def verdict(order, times):
    """Every adjacent pair of the expected order must satisfy t[a] <= t[b]*(1+TOL)."""
    ok = True
    pairs = []
    for a, b in zip(order, order[1:]):
        ta, tb = times.get(a), times.get(b)
        if ta is None or tb is None:
            continue
        holds = ta <= tb * (1 + TOL)
        pairs.append({"better": mm.mm_strategy_name(a), "worse": mm.mm_strategy_name(b),
                      "ms": [round(ta, 4), round(tb, 4)], "holds": holds})
        ok &= holds
    return ok, pairs


MEM_BOUND = (mm.MM_APP_STREAM, mm.MM_APP_BLACKSCHOLES, mm.MM_APP_HOTSPOT, mm.MM_APP_STENCIL_REDUCTION)


def emulation_note(budgets, cls, app_id):
    """Where a platform of logical devices on ONE B200 distorts an ordering."""
    notes = []
    if len(budgets) > 1 and all(b == 0 for b in budgets):
        notes.append("HOMO: every logical device claims the whole GPU, so concurrent devices contend for the "
                     "same SMs and HBM; sharding adds transfers without adding hardware (single-GPU artefact)")
        if cls == mm.MM_MK_DAG:
            notes.append("MK-DAG: a strategy that keeps the DAG on one device wins by construction here; "
                         "on separate GPUs it would leave the others idle")
    elif len(set(budgets)) == 1 and app_id in MEM_BOUND:
        notes.append("PART: equal SM partitions of one GPU share its HBM, so a memory-bound kernel on one "
                     "device runs faster while the others idle (single-GPU artefact)")
    elif app_id in MEM_BOUND:
        notes.append("HET: SMs are partitioned (green contexts) but HBM bandwidth is shared, so memory-bound "
                     "kernels of the small devices steal bandwidth from the big one (single-GPU artefact)")
    return "; ".join(notes) or None


def run_config(name, app_id, ip, budgets, staged, reps):
    G = len(budgets)
    s = runner.session(app_id, ip, G=G, sm_budgets=budgets)
    try:
        cls = s.classify()
        ns = mm.mm_needs_sync(s.app)
        order = expected_order(cls, ns)
        # Glinda's transfer metric (P49) measured on the link the data crosses:
        # the pinned host link for staged runs (sets prof.staged), the
        # device-to-device exchange link for resident ones
        prof = s.profile(reps=3, link="host" if staged else "peer")
        s.fill()
        host = None
        if staged:
            host = []
            for slot in range(s.nbuf):
                eb, n = mm.mm_app_buffer_info(s.app, slot)
                h = torch.empty(max(n, 1), dtype=runner._DT[eb], pin_memory=True)
                h.copy_(s.bufs[(slot, 0)].cpu())
                host.append(h)
        # MK-DAG factors A in place: every run starts from the same SPD matrix
        # (restored outside the library's device-timed span)
        pristine = ({d: s.bufs[(0, d)].clone() for d in range(G) if s.mine[d]}
                    if cls == mm.MM_MK_DAG else {})

        def restore():
            for d, t in pristine.items():
                s.bufs[(0, d)].copy_(t)
            if pristine and host is not None:
                host[0].copy_(pristine[min(pristine)])
            if pristine:
                torch.cuda.synchronize()

        times, shares, instances = {}, {}, {}
        adaptive_ms, ad_share = None, None
        # comparators outside Table I: SP-Cyclic (MK-DAG, P201); DP-Static,
        # §V's conversion of dynamic into static partitioning (P565)
        strategies = list(order) + ([mm.MM_SP_CYCLIC] if cls == mm.MM_MK_DAG else [mm.MM_DP_STATIC])
        for st in strategies:
            p = s.plan(st, prof, staged=staged)
            kw = {"host": [h.data_ptr() for h in host]} if staged else {}
            restore()
            s.run(p, **kw)
            ts = []
            for _ in range(reps):
                restore()
                r = s.run(p, **kw)
                ts.append(r.device_ms)
            times[st] = statistics.median(ts)
            if st == mm.MM_DP_PERF and not staged:
                # adaptive DP-Perf (estimates updated at run time) beside the frozen schedule
                restore()
                s.run(p, adaptive=True)
                ta = []
                for _ in range(reps):
                    restore()
                    ta.append(s.run(p, adaptive=True).device_ms)
                adaptive_ms = statistics.median(ta)
                decs = mm.mm_run_decisions(p)
                ad_share = [sum(1 for dc in decs if dc.chosen == d) / max(1, len(decs)) for d in range(G)]
            info = mm.mm_plan_info(p)
            tot = [sum(info.items[d][k] for k in range(s.K)) for d in range(G)]
            if st in (mm.MM_DP_PERF, mm.MM_DP_DEP, mm.MM_DP_STATIC):
                ch = mm.mm_plan_chunks(p)
                instances[mm.mm_strategy_name(st)] = [sum(1 for c in ch if c.device == d) for d in range(G)]
            shares[mm.mm_strategy_name(st)] = [round(x / max(1, sum(tot)), 4) for x in tot]
        ok, pairs = verdict(order, times)
        table = {k: v for k, v in times.items() if k in order}
        top_ok = times[order[0]] <= min(table.values()) * (1 + TOL)
        return {"app": name, "class": mm.mm_class_name(cls), "needs_sync": ns, "mode": "staged" if staged else "resident",
                "sms": [mm.mm_ctx_sm_count(s.ctx, d) for d in range(G)],
                "expected_order": [mm.mm_strategy_name(x) for x in order],
                "ms": {mm.mm_strategy_name(k): round(v, 4) for k, v in times.items()},
                "measured_order": [mm.mm_strategy_name(k) for k, _ in sorted(times.items(), key=lambda kv: kv[1])],
                "share_per_device": shares, "task_instances_per_device": instances,
                "ranking_holds": ok, "top_choice_holds": top_ok, "pairs": pairs,
                "dp_perf_adaptive_ms": None if adaptive_ms is None else round(adaptive_ms, 4),
                "dp_perf_adaptive_task_share": ad_share,
                "profile_link_Bps": [int(prof.link_Bps[d]) for d in range(G)],
                "profile_link_lat_ns": [int(prof.link_lat_ns[d]) for d in range(G)],
                "emulation_note": emulation_note(budgets, cls, app_id),
                "profile_fs_item": [[int(prof.fs_item[d][k]) for k in range(s.K)] for d in range(G)],
                "profile_chunk_est_ns": [[int(prof.chunk_est_ns[d][k]) for k in range(s.K)] for d in range(G)]}
    finally:
        s.close()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r2_ranking.json"))
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--only", default="", help="run only the apps whose name contains this string")
    ap.add_argument("--platforms", default="HET-2,HOMO-2",
                    help="comma list of " + ",".join(PLATFORMS))
    args = ap.parse_args()
    torch.cuda.set_device(0)
    plats = [(n, PLATFORMS[n]) for n in args.platforms.split(",")]
    res = {"platforms": {n: b for n, b in plats}, "tolerance": TOL, "configs": []}
    t0 = time.time()
    for pname, budgets in plats:
        for name, app_id, ip in APPS:
            if args.only and args.only not in name:
                continue
            modes = [False]
            if app_id == mm.MM_APP_STREAM and not args.quick:
                modes.append(True)
            for staged in modes:
                try:
                    r = run_config(name, app_id, ip, budgets, staged, args.reps)
                except Exception as e:  # report, never hide
                    r = {"app": name, "mode": "staged" if staged else "resident", "error": str(e)[:300]}
                r["platform"] = pname
                res["configs"].append(r)
                print(json.dumps({k: r.get(k) for k in ("platform", "app", "mode", "ms", "ranking_holds", "top_choice_holds",
                                                         "dp_perf_adaptive_ms", "share_per_device", "error")}),
                      flush=True)
    res["wall_s"] = round(time.time() - t0, 1)
    held = [c.get("ranking_holds") for c in res["configs"] if "ranking_holds" in c]
    top = [c.get("top_choice_holds") for c in res["configs"] if "top_choice_holds" in c]
    res["summary"] = {"configs": len(res["configs"]), "ranking_holds": sum(bool(h) for h in held),
                      "ranking_violated": sum(not h for h in held),
                      "top_choice_holds": sum(bool(h) for h in top), "top_choice_violated": sum(not h for h in top)}
    with open(args.out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps(res["summary"]))


if __name__ == "__main__":
    main()
