"""Multi-process (N>1) host path on CPU with gloo, world size 2.

1. Every rank builds the plan independently through the C ABI; the op
   programs must be identical (the executor relies on it: each rank walks the
   same global op list and the NCCL send/recv pairs match by order).
2. A CPU emulation of the multi-process executor — each rank owns one logical
   device (its own full-size copies), runs its KERNEL ops with the oracle's
   kernels, and turns every XFER into a gloo send/recv in global order —
   reproduces the unpartitioned oracle bit for bit.  This checks that the op
   program moves every element a rank needs (re-sync, halos, DP chunk inputs).
"""
import hashlib
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

import synthgen
from oracle import numeric as on

mm = pytest.importorskip("paper_conf_icpp_shenvms15_b200.mm")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _plan_digest(plan):
    h = hashlib.sha256()
    for o in mm.mm_plan_ops(plan):
        h.update(bytes(o))
    return h.hexdigest()


def _emulate(rank, world, app_id, iparam, strategy, prof_seed):
    import torch
    app = mm.mm_app_builtin(app_id, iparam)
    rnd = np.random.default_rng(prof_seed)
    K = mm.mm_app_info(app)[0]
    prof = mm.make_profile(world, rnd.integers(500, 3000, size=(world, K)).tolist(),
                           rnd.integers(10 ** 4, 10 ** 6, size=(world, K)).tolist(),
                           rnd.integers(10 ** 9, 10 ** 12, size=world).tolist())
    plan = mm.mm_plan_build(app, prof, mm.plan_opts(strategy, chunks_per_dev=2))
    # 1. identical plans on every rank
    dig = [None] * world
    dist.all_gather_object(dig, _plan_digest(plan))
    assert len(set(dig)) == 1
    # 2. emulated execution: this rank's full-size copies
    nbuf = mm.mm_app_info(app)[1]
    bufs = []
    for s in range(nbuf):
        eb, n = mm.mm_app_buffer_info(app, s)
        bufs.append(np.zeros(n, np.float32 if eb == 4 else np.float64))
    if app_id == mm.MM_APP_STREAM:
        a, b, c = synthgen.stream_random(iparam[0])
        bufs[0][:], bufs[1][:], bufs[2][:] = a, b, c
    else:
        t, p = synthgen.hotspot(iparam[0], iparam[1])
        bufs[0][:] = t.reshape(-1)
        bufs[2][:] = p.reshape(-1)
    chunks = mm.mm_plan_chunks(plan)
    cols = iparam[1] if app_id != mm.MM_APP_STREAM else 1
    for o in mm.mm_plan_ops(plan):
        if o.kind == mm.MM_OPK_BARRIER:
            dist.barrier()
        elif o.kind == mm.MM_OPK_XFER:
            lo, hi = o.r.begin, o.r.end
            if o.device == rank:
                t = torch.empty(hi - lo, dtype=torch.float32)
                dist.recv(t, src=o.src)
                bufs[o.buffer][lo:hi] = t.numpy()
            elif o.src == rank:
                dist.send(torch.from_numpy(bufs[o.buffer][lo:hi].copy()), dst=o.device)
        elif o.kind == mm.MM_OPK_KERNEL and o.device == rank:
            b0, e0 = o.r.begin, o.r.end
            if app_id == mm.MM_APP_STREAM:
                A, B, Cc = bufs
                [lambda: on.stream_copy(A, Cc, b0, e0), lambda: on.stream_scale(B, Cc, 3.0, b0, e0),
                 lambda: on.stream_add(A, B, Cc, b0, e0), lambda: on.stream_triad(A, B, Cc, 3.0, b0, e0)][o.kernel]()
            else:
                src, dst = (0, 1) if o.iter % 2 == 0 else (1, 0)
                rows = iparam[0]
                tb = iparam[5] if len(iparam) > 5 and iparam[5] > 1 else 1
                if tb > 1:   # temporal block: tb iterations per kernel, halo tb rows
                    on.hotspot_block_rows(bufs[src].reshape(rows, cols), bufs[2].reshape(rows, cols),
                                          bufs[dst].reshape(rows, cols), b0, e0, tb)
                else:
                    on.hotspot_rows(bufs[src].reshape(rows, cols), bufs[2].reshape(rows, cols),
                                    bufs[dst].reshape(rows, cols), b0, e0)
    # assemble on rank 0 from the final owners
    results = {}
    for s in range(3):
        owners = mm.mm_plan_owners(plan, s)
        full = np.zeros_like(bufs[s])
        for (lo, hi, d) in owners:
            if d == rank:
                full[lo:hi] = bufs[s][lo:hi]
        t = torch.from_numpy(full)
        mask = torch.from_numpy(np.concatenate([np.full(hi - lo, d == rank) for lo, hi, d in owners]
                                               ).astype(np.float32))
        dist.all_reduce(t)  # disjoint ownership: sum = assembly
        dist.all_reduce(mask)
        assert torch.all(mask == 1)
        results[s] = t.numpy()
    del chunks
    mm.mm_plan_destroy(plan)
    mm.mm_app_destroy(app)
    return results


def _worker(rank, world, port, cases, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        out = []
        for case in cases:
            res = _emulate(rank, world, *case)
            if rank == 0:
                out.append(res)
        if rank == 0:
            q.put(("ok", out))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put(("err", f"rank {rank}: {e!r}"))
        raise
    finally:
        dist.destroy_process_group()


CASES = [
    (mm.MM_APP_STREAM, [4099, 2, 0, 32, 1], mm.MM_SP_UNIFIED, 1),
    (mm.MM_APP_STREAM, [4099, 1, 1, 32, 1], mm.MM_SP_VARIED, 2),
    (mm.MM_APP_STREAM, [3000, 2, 0, 32, 1], mm.MM_DP_PERF, 3),
    (mm.MM_APP_STREAM, [3000, 1, 2, 32, 1], mm.MM_DP_DEP, 4),
    (mm.MM_APP_HOTSPOT, [41, 16, 5, 1, 1], mm.MM_SP_SINGLE, 5),
    (mm.MM_APP_HOTSPOT, [41, 16, 4, 1, 1], mm.MM_DP_PERF, 6),
    (mm.MM_APP_HOTSPOT, [41, 16, 3, 1, 1], mm.MM_DP_DEP, 7),
    (mm.MM_APP_HOTSPOT, [41, 16, 6, 1, 1, 2], mm.MM_SP_SINGLE, 8),   # temporal block 2
    (mm.MM_APP_HOTSPOT, [41, 16, 9, 1, 1, 3], mm.MM_DP_DEP, 9),      # temporal block 3
]


def test_two_rank_emulation_matches_oracle():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, CASES, q)) for r in range(2)]
    for p in procs:
        p.start()
    status, out = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
    assert status == "ok", out
    for (app_id, ip, strategy, _), res in zip(CASES, out):
        if app_id == mm.MM_APP_STREAM:
            ref = on.stream_run(*synthgen.stream_random(ip[0]), ip[1])
            for s in range(3):
                assert np.array_equal(res[s], ref[s]), (strategy, s)
        else:
            t, p = synthgen.hotspot(ip[0], ip[1])
            ref = on.hotspot_run(t, p, ip[2])
            tb = ip[5] if len(ip) > 5 and ip[5] > 1 else 1
            slot = 0 if (ip[2] // tb) % 2 == 0 else 1
            assert np.array_equal(res[slot].reshape(ip[0], ip[1]), ref), strategy
