"""Benchmark of the matchmaking hot path on B200 (driver contract: one JSON line).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--app stream|stream-loop|hotspot|stencil|blackscholes|sgemm]

Workload (default): BASELINE.json configs[1] — MK-Seq STREAM copy/scale/add/
triad on 2^28 FP32 elements, one STREAM-Seq pass per step.  A step is the whole
hot path: classify -> rank (Table I) -> split -> run the best-ranked strategy
(SP-Unified for MK-Seq without sync).  Profiling (Glinda's probes, the DP
warm-up) is excluded from timing as in the paper (P311).  Inputs are 1 GiB per
array (> 126 MB L2), generated in place; no L2 flush is needed (the apps
whose inputs fit in L2, MatrixMul 1024^2 and Nbody, flush it before every
timed step with a 1 GiB write, outside the step's timed span).

value = algorithmic bytes of the step (40 B/element/pass) / device time, summed
over all ranks' work and divided by the max-over-ranks time (whole job).
Under torchrun (N>1) every rank owns one GPU = one logical device; exchanges
go through the library's NCCL communicator.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "per-app exec time & speedup vs 1 GPU per strategy at 1/2/4/8 B200; HBM % peak"

# apps whose resident inputs fit in L2: timed steps flush it first
L2_RESIDENT = ("matmul1k", "nbody")

APPS = {
    # name: (builtin id, iparam, algorithmic bytes per step as fn(iparam), description)
    "stream": ("MM_APP_STREAM", [1 << 28, 1, 0], lambda p: 40 * p[0] * p[1],
               "MK-Seq STREAM-Seq copy/scale/add/triad, 2^28 FP32 (BASELINE configs[1])"),
    "stream-loop": ("MM_APP_STREAM", [1 << 28, 10, 0], lambda p: 40 * p[0] * p[1],
                    "MK-Loop STREAM-Loop x10, 2^28 FP32"),
    "hotspot": ("MM_APP_HOTSPOT", [8192, 8192, 1000], lambda p: p[0] * p[1] * p[2],
                "SK-Loop HotSpot 8192^2 x 1000 iterations (BASELINE configs[2])"),
    "stencil": ("MM_APP_STENCIL_REDUCTION", [16384, 16384, 100, 1], lambda p: 20 * p[0] * p[1] * p[2],
                "MK-Loop stencil + FP64 residual 16384^2 x 100 steps, w-sync (BASELINE configs[3])"),
    "blackscholes": ("MM_APP_BLACKSCHOLES", [80530632], lambda p: 20 * p[0],
                     "SK-One BlackScholes 80,530,632 options (P311)"),
    "sgemm": ("MM_APP_SGEMM", [6144, 6144, 6144, 0], lambda p: 2 * p[0] * p[1] * p[2],
              "SK-One MatrixMul 6144^2 FP32 (P311)"),
    "matmul1k": ("MM_APP_SGEMM", [1024, 1024, 1024, 0], lambda p: 2 * p[0] * p[1] * p[2],
                 "SK-One MatrixMul 1024^2 FP32 (BASELINE configs[0])"),
    "cholesky": ("MM_APP_CHOLESKY", [32768, 1024], lambda p: p[0] ** 3 / 3,
                 "MK-DAG tiled Cholesky 32768^2 FP32, tile 1024 (BASELINE configs[4])"),
    "nbody": ("MM_APP_NBODY", [1048576, 1], lambda p: 20 * p[0] * p[0] * p[1],
              "SK-Loop Nbody 1,048,576 bodies, 1 step (P319; 20 flop/interaction)"),
}
FLOP_APPS = ("sgemm", "matmul1k", "cholesky", "nbody")
# HotSpot with temporal blocking moves 12 B per cell per h iterations, so a
# "bytes per iteration" rate is not a bandwidth: report cell updates per second
CELL_APPS = ("hotspot",)
# HotSpot temporal block: iterations per launch in the bench
# step (1000 % HOTSPOT_TB == 0); the result is bit-identical for every value
HOTSPOT_TB = 8
# FP32 lane-ops per HotSpot cell update (R16: 9 add/sub + 5 mul)
HOT_FLOPS = 14
# kernel whose roofline is reported, and its algorithmic bytes per item
DOMINANT = {"stream": ("triad", 12), "stream-loop": ("triad", 12), "hotspot": ("hotspot", None),
            "stencil": ("stencil", None), "blackscholes": ("blackscholes", 20), "sgemm": ("sgemm", None),
            "matmul1k": ("sgemm", None), "cholesky": ("gemm", None), "nbody": ("nbody", None)}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get("hbm_gbs", 6650.0), d.get("bf16_tflops", 1590.0), "measured"
    except Exception:
        return 6650.0, 1590.0, "fallback"


def load_sustained_bf16():
    """Sustained dense bf16 TF/s (back-to-back GEMMs under the power cap):
    the denominator for a contraction timed inside a long step."""
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        if "bf16_tflops_sustained" in d:
            return d["bf16_tflops_sustained"], "measured sustained (MEASURED_PEAKS.json bf16_tflops_sustained)"
    except Exception:
        pass
    return None, None


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "20"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(r[1]) for r in self.rows if len(r) > 2 and r[1].replace('.', '').isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) > 2 and r[2].replace('.', '').isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for i, nm in enumerate(names):
                if len(r) > 5 + i and r[5 + i].lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows)}


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def unit_of(app: str):
    if app in FLOP_APPS:
        return "TFLOP/s", 1e12
    if app in CELL_APPS:
        return "Gcell-updates/s", 1e9
    return "GB/s", 1e9


def cpu_baseline(app: str, seconds: float = 10.0):
    """The oracle, as it stands, single-threaded on a bounded sample."""
    import numpy as np

    import synthgen
    from oracle import numeric as on
    if app.startswith("stream"):
        n = 1 << 24
        a, b, c = synthgen.stream_random(n)
        t0 = time.perf_counter()
        passes = 0
        while time.perf_counter() - t0 < seconds:
            on.lib().or_stream_run(a, b, c, n, 3.0, 1)
            passes += 1
        dt = time.perf_counter() - t0
        return {"value": 40 * n * passes / dt / 1e9, "unit": "GB/s", "cores": 1, "kind": "oracle",
                "sample": f"{passes} STREAM-Seq passes over 2^24 of the 2^28 elements (single thread, C -O2)"}
    if app == "hotspot" or app == "stencil":
        rows, cols = 1024, 8192
        t, p = synthgen.hotspot(rows, cols)
        out = np.empty_like(t)
        t0 = time.perf_counter()
        it = 0
        while time.perf_counter() - t0 < seconds:
            on.hotspot_rows(t, p, out)
            t, out = out, t
            it += 1
        dt = time.perf_counter() - t0
        if app == "hotspot":
            return {"value": rows * cols * it / dt / 1e9, "unit": "Gcell-updates/s", "cores": 1, "kind": "oracle",
                    "sample": f"{it} HotSpot iterations over 1024 of the 8192 rows"}
        return {"value": 12 * rows * cols * it / dt / 1e9, "unit": "GB/s", "cores": 1, "kind": "oracle",
                "sample": f"{it} HotSpot iterations over 1024 of the 8192 rows"}
    if app == "blackscholes":
        n = 1 << 22
        S, X, T = synthgen.blackscholes(n)
        t0 = time.perf_counter()
        k = 0
        while time.perf_counter() - t0 < seconds:
            on.blackscholes(S, X, T)
            k += 1
        dt = time.perf_counter() - t0
        return {"value": 20 * n * k / dt / 1e9, "unit": "GB/s", "cores": 1, "kind": "oracle",
                "sample": f"{k} passes over 2^22 options"}
    if app == "cholesky":
        n = 768
        A = synthgen.spd_random(n).astype(np.float64)
        t0 = time.perf_counter()
        k = 0
        while time.perf_counter() - t0 < seconds:
            on.cholesky(A)
            k += 1
        dt = time.perf_counter() - t0
        return {"value": n ** 3 / 3 * k / dt / 1e12, "unit": "TFLOP/s", "cores": 1, "kind": "oracle",
                "sample": f"{k} unblocked FP64 Cholesky factorizations of a 768^2 SPD matrix (n^3/3 flop each)"}
    if app == "nbody":
        n = 1 << 20
        pos, vel = synthgen.nbody(n)
        t0 = time.perf_counter()
        k = 0
        while time.perf_counter() - t0 < seconds:
            on.nbody_step_bodies(pos, vel, list(range(k % n, k % n + 256)))
            k += 256
        dt = time.perf_counter() - t0
        return {"value": 20 * n * k / dt / 1e12, "unit": "TFLOP/s", "cores": 1, "kind": "oracle",
                "sample": f"{k} bodies of the 2^20-body step, each summed over all 2^20 bodies (20 flop/interaction)"}
    n = 512
    A, B = synthgen.matmul_uniform(n, n, n)
    t0 = time.perf_counter()
    k = 0
    while time.perf_counter() - t0 < seconds:
        on.sgemm(A, B)
        k += 1
    dt = time.perf_counter() - t0
    return {"value": 2 * n ** 3 * k / dt / 1e12, "unit": "TFLOP/s", "cores": 1, "kind": "oracle",
            "sample": f"{k} 512^3 products"}


def run_reference(args):
    world, rank, local = dist_env()
    if rank != 0:
        return
    unit = unit_of(args.app)[0]
    # each step = a bounded sample of the workload on the oracle (host cores)
    vals = []
    for i in range(args.warmup + args.steps):
        cb = cpu_baseline(args.app, seconds=max(2.0, 20.0 / max(1, args.steps)))
        if i >= args.warmup:
            vals.append(cb)
    v = statistics.median([c["value"] for c in vals])
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": unit, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": APPS[args.app][3], "sample": vals[0]["sample"]},
            "cpu_baseline": {"value": v, "unit": unit, "cores": 1, "kind": "oracle", "sample": vals[0]["sample"]},
            "e2e": {"value": v, "unit": unit, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--app", default="stream", choices=sorted(APPS))
    ap.add_argument("--tb", type=int, default=None,
                    help="HotSpot temporal block h (iterations per launch; default 4 for --app hotspot)")
    ap.add_argument("--chol-tile", type=int, default=None, help="Cholesky tile b (default 1024)")
    ap.add_argument("--chol-n", type=int, default=None, help="Cholesky order n (default 32768)")
    ap.add_argument("--pipeline", type=int, default=32,
                    help="e2e staged pipeline sub-chunks per device (R24; 8: 171.5, 16: 174.1, 32: 176.4, 64: 175.4 GB/s STREAM)")
    ap.add_argument("--halo-split", default="auto", choices=["auto", "on", "off"],
                    help="R33: SP ranges of halo-reading kernels run interior-first so the interior overlaps "
                         "the halo pulls (auto = on when the job spans more than one device)")
    ap.add_argument("--one-graph", action="store_true",
                    help="time the K steps as ONE mm_run with repeat = K (one graph of K copies of the op "
                         "program); measured no faster than K replays, and slower with kernel timing, whose "
                         "event nodes then sit in every copy")
    ap.add_argument("--no-graph", action="store_true",
                    help="timed steps issue the op program eagerly instead of replaying a CUDA graph")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-strategies", action="store_true")
    ap.add_argument("--no-e2e", action="store_true", help="skip the staged (host-buffer) e2e pass")
    ap.add_argument("--no-profile", action="store_true",
                    help="use an equal synthetic profile instead of measuring one (ncu runs)")
    ap.add_argument("--kernel-timing", default="last", choices=["all", "last", "none"],
                    help="per-kernel CUDA events in the timed steps: every step, the last step, or none")
    ap.add_argument("--share-gpu", action="store_true",
                    help="ranks share GPUs (rank r on cuda:r %% count): exercises the multi-process "
                         "IPC path on a box with fewer GPUs than ranks; not a scaling measurement")
    ap.add_argument("--logical", type=int, default=0,
                    help="virtual mode: run G logical devices on this one GPU (G = --logical)")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist

    from paper_conf_icpp_shenvms15_b200 import mm, runner

    world, rank, local = dist_env()
    have = torch.cuda.device_count()
    if args.gpus > 1 and world == 1:
        # --gpus N without a launcher: one rank per GPU needs N visible GPUs
        # (or --share-gpu); never time fewer GPUs than asked for
        if have < args.gpus and not args.share_gpu:
            print(json.dumps({"error": f"--gpus {args.gpus} but only {have} CUDA device(s) visible",
                              "n_gpus": have}), flush=True)
            sys.exit(2)
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", "--master-port", str(29500 + os.getpid() % 1000)] + sys.argv
        sys.exit(subprocess.call(cmd))
    if world > 1 and world != args.gpus:
        print(json.dumps({"error": f"WORLD_SIZE={world} but --gpus {args.gpus}"}), flush=True)
        sys.exit(2)
    if world > have and not args.share_gpu:
        print(json.dumps({"error": f"{world} ranks but only {have} CUDA device(s) visible"}), flush=True)
        sys.exit(2)
    if args.share_gpu:   # exercising the multi-process path on fewer GPUs than ranks
        local = local % have
    torch.cuda.set_device(local)
    if world > 1:
        # rank 0 names the context: the IPC rendezvous id (default transport:
        # CUDA IPC pulls + device-memory flags) or an NCCL id (MM_TRANSPORT=nccl)
        dist.init_process_group("gloo")
        nccl = os.environ.get("MM_TRANSPORT") == "nccl"
        nid = [(mm.mm_nccl_unique_id() if nccl else mm.mm_rendezvous_id()) if rank == 0 else None]
        dist.broadcast_object_list(nid, src=0)
        nccl_id = nid[0]
    else:
        nccl_id = None
    G = world if world > 1 else max(1, args.logical)
    app_id = getattr(mm, APPS[args.app][0])
    iparam = list(APPS[args.app][1])
    tb = 1
    if args.app == "hotspot":
        tb = args.tb if args.tb is not None else HOTSPOT_TB
        iparam = iparam + [0, 0, tb]
    if args.app == "cholesky":
        iparam = [args.chol_n or iparam[0], args.chol_tile or iparam[1]]
    algo_bytes = APPS[args.app][2](iparam)
    sess = runner.session(app_id, iparam, G=G, cuda_devices=[local] * G, rank=rank, world=world,
                          nccl_id=nccl_id)
    hbm_peak, tf_peak, peak_kind = load_peaks()

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    # --- setup (excluded from timing, P311): profile, then generate inputs ---
    prof = sess.equal_profile() if args.no_profile else sess.profile(reps=3)
    sess.fill()
    cls = mm.mm_classify(sess.app)
    ranked = mm.mm_rank(cls, mm.mm_needs_sync(sess.app))
    best = ranked[0]
    halo_split = args.halo_split == "on" or (args.halo_split == "auto" and G > 1)
    plan = sess.plan(best, prof, halo_split=halo_split)
    info = mm.mm_plan_info(plan)
    K = sess.K

    def step(p, **kw):
        # the hot path: classify -> rank -> split (pure, host) -> partitioned run
        c = mm.mm_classify(sess.app)
        mm.mm_rank(c, mm.mm_needs_sync(sess.app))
        if best in (mm.MM_SP_SINGLE, mm.MM_SP_UNIFIED, mm.MM_SP_VARIED):
            mm.mm_split(sess.app, prof, best)
        return sess.run(p, **kw)

    # MK-DAG factors A in place: every step starts from the same SPD matrix,
    # restored from a pristine copy between steps, outside the timed spans
    # (each step is then bracketed by its own barrier + synchronize); the
    # other apps' steps are timed back to back
    pristine = {}
    if args.app == "cholesky":
        pristine = {d: sess.bufs[(0, d)].clone() for d in range(G) if sess.mine[d]}

    # apps whose inputs fit in the 126 MB L2 (MatrixMul 1024^2: 12 MB; Nbody
    # 2^20 bodies: 32 MB) run every timed step from a cold L2: a 1 GiB buffer
    # is written on the step's stream just before the step's start event; the
    # timed span of a step is its start -> end event pair.  (1 GiB, not just
    # > 126 MB: the ~170 us write also keeps the host's issue of the next step
    # ahead of the GPU, so no host latency falls inside a span — with 256 MB
    # the MatrixMul span still held ~3 us of it.)
    flush_l2 = args.app in L2_RESIDENT
    l2_junk = torch.empty(256 << 20, dtype=torch.float32, device=f"cuda:{local}") if flush_l2 else None

    def restore():
        for d, t in pristine.items():
            sess.bufs[(0, d)].copy_(t)
        if pristine:
            torch.cuda.synchronize()

    def flush():
        if l2_junk is not None:
            with torch.cuda.stream(stream):
                l2_junk.fill_(1.0)

    # timed steps: the op program replayed as one CUDA graph, enqueued without
    # a host round trip per step (mm_run no_wait; steps are ordered on the
    # library's streams); the last step runs eagerly with CUDA events around
    # every kernel for the roofline (--kernel-timing)
    graph_ok = world == 1 or os.environ.get("MM_TRANSPORT") != "nccl"
    fast = dict(use_graph=graph_ok and not args.no_graph, no_wait=True)
    # apps that do not restore their input between steps run all K timed steps
    # as ONE mm_run with repeat = K (see the timed loop); its graph is captured
    # in the last warm-up step, outside the timed region
    one_graph = (not pristine and not flush_l2 and fast["use_graph"] and args.one_graph
                 and args.kernel_timing != "all")
    for w in range(args.warmup):
        restore()
        if w == 0:
            step(plan, time_kernels=True)
        elif one_graph and w == args.warmup - 1:
            step(plan, use_graph=True, time_kernels=args.kernel_timing != "none", repeat=args.steps)
        else:
            step(plan, **fast)
    barrier()
    l0 = mm.mm_kernel_launch_count()
    stream = sess.stream(rank if world > 1 else 0)
    kms = [[0.0] * K for _ in range(G)]
    launches = 0
    spans = []
    # --kernel-timing last: the final timed step carries CUDA events around every
    # kernel; it runs eagerly and blocks once (the other steps are graph replays
    # enqueued back to back), so timing more steps would add host round trips
    # to the measured region
    n_last = 1
    # one_graph: one CUDA graph holding K copies of the op program
    # (kernel-timing events are event nodes of that graph, read for the last
    # copy), so the steps pay one launch instead of K
    with ClockSampler(local) as clk:
        if one_graph:
            barrier()
            ev0 = torch.cuda.Event(enable_timing=True)
            ev0.record(stream)
            for _ in range(args.steps - 1):   # the host control plane of every step
                c = mm.mm_classify(sess.app)
                mm.mm_rank(c, mm.mm_needs_sync(sess.app))
                if best in (mm.MM_SP_SINGLE, mm.MM_SP_UNIFIED, mm.MM_SP_VARIED):
                    mm.mm_split(sess.app, prof, best)
            st = step(plan, use_graph=True, time_kernels=args.kernel_timing != "none", repeat=args.steps)
            for d in range(G):
                for k in range(K):
                    kms[d][k] += st.kernel_ms[d][k]
            launches += st.n_launches
            ev1 = torch.cuda.Event(enable_timing=True)
            ev1.record(stream)
            barrier()
            spans.append((ev0, ev1))
        for i in range(0 if not one_graph else args.steps, args.steps):
            if pristine or i == 0:
                restore()
                barrier()
            if pristine or flush_l2 or i == 0:
                # L2-resident apps: flush + start event enqueued behind the
                # previous step without a host round trip, so neither the host's
                # issue of this step nor the flush falls inside its span
                flush()
                ev0 = torch.cuda.Event(enable_timing=True)
                ev0.record(stream)
            kt = args.kernel_timing == "all" or (args.kernel_timing == "last" and i >= args.steps - n_last)
            st = step(plan, time_kernels=True) if kt else step(plan, **fast)
            if kt:
                for d in range(G):
                    for k in range(K):
                        kms[d][k] += st.kernel_ms[d][k]
            launches += st.n_launches
            if pristine or flush_l2 or i == args.steps - 1:
                ev1 = torch.cuda.Event(enable_timing=True)
                ev1.record(stream)
                if pristine or i == args.steps - 1:
                    barrier()
                spans.append((ev0, ev1))
    ms_total = sum(a.elapsed_time(b) for a, b in spans)
    gpu_launches = mm.mm_kernel_launch_count() - l0
    if world > 1:
        t = torch.tensor([ms_total], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_total = float(t.item())
        lt = torch.tensor([gpu_launches], dtype=torch.int64)
        dist.all_reduce(lt)
        gpu_launches = int(lt.item())
    ms_step = ms_total / args.steps
    unit, scale = unit_of(args.app)
    value = algo_bytes / (ms_step * 1e-3) / scale

    # --- roofline of the dominant kernel (event-timed inside the timed region)
    dom, bpi = DOMINANT[args.app]
    # kernel ids of the builtin apps in program order
    kname_map = {"stream": ["copy", "scale", "add", "triad"], "stream-loop": ["copy", "scale", "add", "triad"],
                 "hotspot": ["hotspot"], "stencil": ["stencil", "residual"], "blackscholes": ["blackscholes"],
                 "sgemm": ["sgemm"], "matmul1k": ["sgemm"],
                 "cholesky": ["potrf", "trsm", "syrk", "gemm"], "nbody": ["nbody"]}[args.app]
    kid = kname_map.index(dom)
    my = [d for d in range(G) if sess.mine[d]]
    dom_ms = sum(kms[d][kid] for d in my)
    timed_steps = {"all": args.steps, "last": n_last, "none": 0}[args.kernel_timing]
    dom_launch = sum(st.kernel_launches[d][kid] for d in my) * timed_steps
    items = sum(info.items[d][kid] for d in my)
    if args.app == "cholesky":
        # the trailing update = SYRK + GEMM tasks; a step's SYRKs and GEMMs share
        # launches (timed under the batch head's kernel), so time both together
        ks = kname_map.index("syrk")
        dom_ms += sum(kms[d][ks] for d in my)
        dom_launch += sum(st.kernel_launches[d][ks] for d in my) * timed_steps
        syrk_items = sum(info.items[d][ks] for d in my)
    if bpi is None:
        bpi = {"hotspot": 12 * iparam[1], "stencil": 12 * iparam[1]}.get(args.app)
    roof = None
    if dom_launch and dom_ms > 0:
        per_launch_ms = dom_ms / dom_launch
        launches_per_step = dom_launch / timed_steps
        if args.app == "nbody":
            # FP32-pipe-bound all-pairs: 20 flop per interaction (usual count);
            # the kernel needs 12 FP32 lane-ops per interaction, so the ceiling
            # is 148 SMs x 128 lanes x 1.965 GHz / 12 interactions/s x 20 flop
            n_b = iparam[0]
            ach = 20 * n_b * items * timed_steps / (dom_ms * 1e-3) / 1e12
            pk = 148 * 128 * 1.965e9 / 12 * 20 / 1e12
            roof = {"bound": "alu", "achieved": ach, "peak": pk, "unit": "TFLOP/s", "frac": ach / pk,
                    "traffic": None, "kernel": "nbody (all pairs, smem tiles, 2 bodies/thread in f32x2)",
                    "peak_kind": "derived: 148 SMs x 128 FP32 lanes/clk (measured, tools/pipe_rates.cu) x "
                                 "1.965 GHz / 12 FP32 lane-ops per interaction x 20 flop"}
        elif args.app == "cholesky":
            # trailing GEMM updates on tcgen05 (3xTF32): FP32-equivalent flops vs
            # measured bf16 x 0.5 (tf32) / 3
            # (the step runs ~75 ms back to back under the power cap, so the
            # denominator is the sustained figure; burst reported beside it)
            # algorithmic flops: 2 b^3 per GEMM task, b^3 per SYRK task
            b = iparam[1]
            ach = (2 * items + syrk_items) * b ** 3 * timed_steps / (dom_ms * 1e-3) / 1e12
            sus, sus_kind = load_sustained_bf16()
            burst = tf_peak * 0.5 / 3.0
            pk = sus * 0.5 / 3.0 if sus else burst
            roof = {"bound": "tensor", "achieved": ach, "peak": pk, "unit": "TFLOP/s", "frac": ach / pk,
                    "traffic": None, "kernel": "SYRK + GEMM tile updates (3xTF32 tcgen05, batched per step)",
                    "peak_kind": (sus_kind if sus else peak_kind) + " bf16_tflops x 0.5 (tf32) / 3 (3xTF32)",
                    "peak_burst": burst, "frac_of_burst": ach / burst}
        elif args.app in ("sgemm", "matmul1k"):
            # 3xTF32: FP32-equivalent flops; peak = measured bf16 x 0.5 (nominal
            # tf32/bf16 dense ratio) / 3 (three tf32 MMAs per FP32 product)
            fl = 2 * iparam[1] * iparam[2] * items / launches_per_step
            ach = fl / (per_launch_ms * 1e-3) / 1e12
            pk = tf_peak * 0.5 / 3.0
            roof = {"bound": "tensor", "achieved": ach, "peak": pk, "unit": "TFLOP/s", "frac": ach / pk,
                    "traffic": None, "kernel": "sgemm (3xTF32 tcgen05, incl. operand split)",
                    "peak_kind": peak_kind + " bf16_tflops x 0.5 (tf32) / 3 (3xTF32)",
                    "avg_launch_ms": per_launch_ms}
        elif args.app == "hotspot" and tb > 1:
            # temporal block: per launch 12 B per cell (read T, read P, write T)
            # for tb updates per cell.  Two ceilings: HBM (12 B / tb per update)
            # and the FP32 pipe (14 lane-ops per update, 128 lanes/clk/SM,
            # tools/pipe_rates.cu); the lower one bounds the kernel
            byts = bpi * items / launches_per_step
            upd = tb * items * iparam[1] / launches_per_step
            ach_gbs = byts / (per_launch_ms * 1e-3) / 1e9
            alu_peak_upd = 148 * 128 * 1.965e9 / HOT_FLOPS
            hbm_peak_upd = hbm_peak * 1e9 / (12.0 / tb)
            if hbm_peak_upd <= alu_peak_upd:
                roof = {"bound": "hbm", "achieved": ach_gbs, "peak": hbm_peak, "unit": "GB/s",
                        "frac": ach_gbs / hbm_peak, "traffic": None, "kernel": f"hotspot_tb<{tb}>",
                        "peak_kind": peak_kind + " (MEASURED_PEAKS.json hbm_gbs)"}
            else:
                ach_tf = upd * HOT_FLOPS / (per_launch_ms * 1e-3) / 1e12
                pk = alu_peak_upd * HOT_FLOPS / 1e12
                roof = {"bound": "alu", "achieved": ach_tf, "peak": pk, "unit": "TFLOP/s", "frac": ach_tf / pk,
                        "traffic": None, "kernel": f"hotspot_tb<{tb}>",
                        "peak_kind": "derived: 148 SMs x 128 FP32 lanes/clk x 1.965 GHz; 14 FP32 ops per cell update"}
            roof.update({"algorithmic_bytes_per_launch": byts, "avg_launch_ms": per_launch_ms,
                         "cell_updates_per_s": upd / (per_launch_ms * 1e-3),
                         "ceilings_updates_per_s": {"hbm": hbm_peak_upd, "fp32": alu_peak_upd}})
        else:
            byts = bpi * items / launches_per_step
            ach = byts / (per_launch_ms * 1e-3) / 1e9
            roof = {"bound": "hbm", "achieved": ach, "peak": hbm_peak, "unit": "GB/s", "frac": ach / hbm_peak,
                    "traffic": None, "kernel": dom, "peak_kind": peak_kind + " (MEASURED_PEAKS.json hbm_gbs)",
                    "algorithmic_bytes_per_launch": byts, "avg_launch_ms": per_launch_ms}
        tr = os.path.join(ROOT, "profiles", "ncu_traffic.json")
        if os.path.exists(tr):
            try:
                roof["traffic"] = json.load(open(tr)).get(f"{args.app}:{dom}")
            except Exception:
                pass

    # --- e2e: same step through the C ABI with HOST buffers (staged mode) ----
    e2e = None
    try:
        if args.no_e2e:
            raise RuntimeError("skipped (--no-e2e)")
        import numpy as np
        nbuf = sess.nbuf
        host = []
        for s in range(nbuf):
            eb, n = mm.mm_app_buffer_info(sess.app, s)
            h = torch.empty(max(n, 1), dtype=runner._DT[eb], pin_memory=True)
            src = pristine[my[0]] if (s == 0 and pristine) else sess.bufs[(s, my[0])]
            if n <= (1 << 29) or pristine:
                h[:n].copy_(src[:n])
            host.append(h)

        def restore_host():   # MK-DAG: the staged run writes L back over host A
            if pristine:
                host[0].copy_(pristine[my[0]])
                torch.cuda.synchronize()
        # staged pipeline (R24): sub-chunks overlap H2D, kernels and D2H on
        # separate streams (applies to pointwise apps; ignored otherwise)
        splan = sess.plan(best, prof, staged=True, pipeline=args.pipeline)
        restore_host()
        step(splan, host=[h.data_ptr() for h in host])  # warm-up
        barrier()
        e0 = time.perf_counter()
        tot = []
        hb = db = 0
        for _ in range(max(1, min(args.steps, 5))):
            restore_host()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            st = step(splan, host=[h.data_ptr() for h in host])
            torch.cuda.synchronize()
            tot.append(time.perf_counter() - t0)
            hb, db = st.h2d_bytes, st.d2h_bytes
        ms_e2e = statistics.median(tot) * 1e3
        if world > 1:
            t = torch.tensor([ms_e2e], dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms_e2e = float(t.item())
        ev = algo_bytes / (ms_e2e * 1e-3) / scale
        e2e = {"value": ev, "unit": unit, "h2d_bytes_per_step": int(hb), "d2h_bytes_per_step": int(db),
               "ms_per_step": ms_e2e, "mode": f"staged (pinned host inputs; H2D / kernels / D2H pipelined over {args.pipeline} sub-chunks per device)"}
        del host
    except Exception as ex:  # report, never hide
        e2e = {"value": None, "unit": unit, "error": str(ex)[:200]}
    # comparators outside Table I: SP-Cyclic for MK-DAG (P201; BASELINE
    # configs[4]); §V's DP-Static conversion (P565) for the range apps
    extras = [mm.MM_SP_CYCLIC] if args.app == "cholesky" else [mm.MM_DP_STATIC]
    if args.app == "cholesky":
        ranked = list(ranked) + [mm.MM_SP_CYCLIC]

    # --- every Table I strategy for this class, w/o and w/ sync (ranking) ----
    strategies = {}
    strategies_graph = {}
    if not args.no_strategies:
        for s_id in list(ranked) + [x for x in extras if x not in ranked]:
            try:
                p = sess.plan(s_id, prof)
                restore()
                step(p)
                barrier()
                ts = []
                for _ in range(3):
                    restore()
                    st = sess.run(p)
                    ts.append(st.device_ms)
                ms = statistics.median(ts)
                if world == 1:   # the same op program captured once and replayed as a CUDA graph
                    restore()
                    sess.run(p, use_graph=True)
                    tg = []
                    for _ in range(3):
                        restore()
                        tg.append(sess.run(p, use_graph=True).device_ms)
                    strategies_graph[mm.mm_strategy_name(s_id)] = round(statistics.median(tg), 4)
                if world > 1:
                    t = torch.tensor([ms], dtype=torch.float64)
                    dist.all_reduce(t, op=dist.ReduceOp.MAX)
                    ms = float(t.item())
                strategies[mm.mm_strategy_name(s_id)] = round(ms, 4)
            except mm.MMError as ex:
                strategies[mm.mm_strategy_name(s_id)] = f"error: {ex}"[:120]

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(args.app)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": unit, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": APPS[args.app][3], "app": args.app, "class": mm.mm_class_name(cls),
                       "strategy": mm.mm_strategy_name(best), "logical_devices": G,
                       "l2": ("L2 flushed before every timed step (a 1 GiB buffer written on the stream between "
                              "steps, outside each step's start/end events; value = summed step spans; "
                              "this app's inputs fit in the 126 MB L2)" if flush_l2 else
                              "inputs larger than L2 (>= 151 MB per array); no flush"),
                       "kernel_timing": {"all": "per-kernel CUDA events in every timed step",
                                         "last": f"per-kernel CUDA events in the last {n_last} of {args.steps} timed steps"
                                                 + (" (graph event nodes)" if one_graph else ""),
                                         "none": "no per-kernel events"}[args.kernel_timing],
                       "issue": ("all timed steps in ONE CUDA graph (mm_run repeat = K: K copies of the op program, "
                                 "kernel-timing events as graph nodes, read for the last copy)" if one_graph else
                                 "other timed steps: the op program replayed as a CUDA graph, enqueued back to back"
                                 if fast["use_graph"] else "other timed steps: eager issue, enqueued back to back"),
                       "split": mm.mm_plan_ranges(plan)[:G], "parallelism": f"row/element split over {G}",
                       "halo_split": halo_split,
                       **({"temporal_block": tb} if args.app == "hotspot" else {})},
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": gpu_launches,
            "clocks": clk.summary(), "strategies_ms": strategies, "strategies_graph_ms": strategies_graph,
            "kernel_ms_per_step": {kname_map[k]: round(sum(kms[d][k] for d in my) / max(1, timed_steps), 4)
                                   for k in range(K)},
            "ranking": [mm.mm_strategy_name(s) for s in ranked],
        }
        print(json.dumps(line), flush=True)
    sess.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
