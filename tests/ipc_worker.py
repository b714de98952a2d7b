"""One rank of a multi-process run through the C ABI (world > 1, IPC transport).

    python tests/ipc_worker.py RANK WORLD ID_HEX CASE OUT.npz [graph] [runs]

Every rank builds the same app and plan, fills its own full-size input copies
(resident inputs are replicated, R12), runs the plan, and saves the element
ranges whose final value it holds (mm_plan_owners) so the test can assemble
the result.  All ranks may share one GPU (cuda:LOCAL % device_count)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_icpp_shenvms15_b200 import mm, runner  # noqa: E402

CASES = {
    # name: (app id, iparam, strategy, output slots, chunks_per_dev)
    "stream_varied": (mm.MM_APP_STREAM, [100003, 2, 0, 32, 1], mm.MM_SP_VARIED, (0, 1, 2), 2),
    "stream_varied_flush": (mm.MM_APP_STREAM, [65536 + 11, 1, 2, 32, 1], mm.MM_SP_VARIED, (0, 1, 2), 2),
    "stream_dp_perf": (mm.MM_APP_STREAM, [100003, 1, 1, 32, 1], mm.MM_DP_PERF, (0, 1, 2), 3),
    "hotspot": (mm.MM_APP_HOTSPOT, [257, 256, 7, 1, 1], mm.MM_SP_SINGLE, (1,), 2),
    "hotspot_tb4": (mm.MM_APP_HOTSPOT, [300, 64, 24, 1, 1, 4], mm.MM_SP_SINGLE, (0,), 2),
    "hotspot_dp_dep": (mm.MM_APP_HOTSPOT, [200, 128, 6, 1, 1], mm.MM_DP_DEP, (0,), 2),
    "hotspot_split": (mm.MM_APP_HOTSPOT, [300, 64, 24, 1, 1, 4], mm.MM_SP_SINGLE, (0,), 2),
    "stencil": (mm.MM_APP_STENCIL_REDUCTION, [200, 96, 5, 1, 1, 1], mm.MM_SP_VARIED, (1, 3), 2),
    "chol": (mm.MM_APP_CHOLESKY, [1024, 256], mm.MM_DP_DEP, (0,), 1),
    "chol_cyclic": (mm.MM_APP_CHOLESKY, [1024, 256], mm.MM_SP_CYCLIC, (0,), 1),
    "profile": (mm.MM_APP_STREAM, [1 << 20, 1, 0, 32, 1], mm.MM_DP_PERF, (0,), 2),
    "stream_staged": (mm.MM_APP_STREAM, [100003, 1, 0, 32, 1], mm.MM_SP_UNIFIED, (0, 1, 2), 2),
    "stream_staged_dp": (mm.MM_APP_STREAM, [100003, 1, 1, 32, 1], mm.MM_DP_PERF, (0, 1, 2), 2),
}


def main():
    rank, world, idhex, case, out = int(sys.argv[1]), int(sys.argv[2]), sys.argv[3], sys.argv[4], sys.argv[5]
    graph = len(sys.argv) > 6 and sys.argv[6] == "graph"
    runs = int(sys.argv[7]) if len(sys.argv) > 7 else 1
    dev = rank % torch.cuda.device_count()
    torch.cuda.set_device(dev)
    app_id, ip, strategy, slots, kpd = CASES[case]
    G = world
    # device d's per-kernel cost: rank-dependent, so SP-Varied ranges differ per kernel
    K = 4
    fs = [[1000 + 700 * ((d + k) % G) for k in range(K)] for d in range(G)]
    prof = mm.make_profile(G, fs, [[10 ** 5 + 3 * 10 ** 4 * d] * K for d in range(G)], [10 ** 11] * G)
    with runner.session(app_id, ip, G=G, cuda_devices=[dev] * G, rank=rank, world=world,
                        nccl_id=bytes.fromhex(idhex)) as s:
        if app_id == mm.MM_APP_CHOLESKY:
            import synthgen
            n, b = ip
            A, _ = synthgen.cholesky_exact_factor(n)
            T = n // b
            s.load(0, A.reshape(T, b, T, b).transpose(0, 2, 1, 3).copy())
        else:
            s.fill()
        if case == "profile":   # collective mm_profile_run: every rank returns the same profile
            p = s.profile(reps=2)
            np.savez(out, fs=np.array([[p.fs_item[d][k] for k in range(4)] for d in range(G)]),
                     link=np.array([p.link_Bps[d] for d in range(G)]),
                     lat=np.array([p.link_lat_ns[d] for d in range(G)]))
            print(f"rank {rank} ok", flush=True)
            return
        if case.startswith("stream_staged"):
            # staged (P119): inputs in this rank's pinned host memory, the run
            # copies them in and flushes the outputs this rank produced back
            import synthgen
            n = ip[0]
            host = [torch.from_numpy(x.copy()).pin_memory() for x in synthgen.stream_random(n)]
            plan = s.plan(strategy, prof, chunks_per_dev=kpd, staged=True)
            st = s.run(plan, host=[h.data_ptr() for h in host], use_graph=graph)
            torch.cuda.synchronize()
            res = {"xfer": np.array([st.xfer_bytes]), "h2d": np.array([st.h2d_bytes])}
            for slot in slots:
                segs = [(b0, e0) for (b0, e0, o) in mm.mm_plan_owners(plan, slot) if o == rank]
                hv = host[slot].numpy()
                res[f"r{slot}"] = np.array(segs, dtype=np.int64).reshape(-1, 2)
                res[f"v{slot}"] = np.concatenate([hv[b0:e0] for b0, e0 in segs]) if segs else hv[:0]
            np.savez(out, **res)
            print(f"rank {rank} ok", flush=True)
            return
        plan = s.plan(strategy, prof, chunks_per_dev=kpd, halo_split=case.endswith("_split"))
        for _ in range(runs):
            if app_id == mm.MM_APP_CHOLESKY and runs > 1:
                s.load(0, A.reshape(T, b, T, b).transpose(0, 2, 1, 3).copy())
                torch.cuda.synchronize()
            st = s.run(plan, use_graph=graph)
        torch.cuda.synchronize()
        res = {"xfer": np.array([st.xfer_bytes]), "launches": np.array([st.n_launches])}
        for slot in slots:
            host = s.bufs[(slot, rank)].cpu().numpy()
            segs = [(b0, e0) for (b0, e0, o) in mm.mm_plan_owners(plan, slot) if o == rank]
            res[f"r{slot}"] = np.array(segs, dtype=np.int64).reshape(-1, 2)
            res[f"v{slot}"] = np.concatenate([host[b0:e0] for b0, e0 in segs]) if segs else host[:0]
        np.savez(out, **res)
    print(f"rank {rank} ok", flush=True)


if __name__ == "__main__":
    main()
