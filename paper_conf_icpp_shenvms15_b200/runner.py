"""Session: device memory (torch tensors) + the C-ABI calls for one app.

Plumbing only: torch allocates one full-size tensor per (buffer slot, logical
device) and provides host pinned memory; every step of the method (classify,
rank, profile, split/schedule, run, exchanges, input generation) is a call
into libmm.so through :mod:`.mm`.
"""
from __future__ import annotations

from typing import Dict, List, Optional, Sequence

import torch

import synthgen
from . import mm

_DT = {1: torch.uint8, 2: torch.float16, 4: torch.float32, 8: torch.float64}

# Input recipes per builtin app: slot -> (array_id, lo, hi) of synthgen.uniform,
# or ("int", array_id, lo, hi) for synthgen.integers.  Mirrors synthgen's
# per-app helpers (same ids and ranges).
RECIPES = {
    mm.MM_APP_STREAM: {0: (synthgen.AID_STREAM_A, -1.0, 1.0), 1: (synthgen.AID_STREAM_B, -1.0, 1.0),
                       2: (synthgen.AID_STREAM_C, -1.0, 1.0)},
    mm.MM_APP_HOTSPOT: {0: (synthgen.AID_HOT_T, 323.15, 343.15), 2: (synthgen.AID_HOT_P, 0.0, 1e-3)},
    mm.MM_APP_STENCIL_REDUCTION: {0: (synthgen.AID_HOT_T, 323.15, 343.15),
                                  2: (synthgen.AID_HOT_P, 0.0, 1e-3)},
    mm.MM_APP_BLACKSCHOLES: {0: (synthgen.AID_BS_S, 5.0, 30.0), 1: (synthgen.AID_BS_X, 1.0, 100.0),
                             2: (synthgen.AID_BS_T, 0.25, 10.0)},
    mm.MM_APP_SGEMM: {0: (synthgen.AID_MM_A, 0.0, 1.0), 1: (synthgen.AID_MM_B, 0.0, 1.0)},
}
RECIPES_INT = {
    mm.MM_APP_SGEMM: {0: ("int", synthgen.AID_MM_A, -4, 4), 1: ("int", synthgen.AID_MM_B, -4, 4)},
}


class Session:
    """One app on G logical devices of this process."""

    def __init__(self, app: int, G: int = 1, cuda_devices: Optional[Sequence[int]] = None,
                 sm_budgets: Optional[Sequence[int]] = None, rank: int = 0, world: int = 1,
                 nccl_id: Optional[bytes] = None, owned: Optional[Sequence[int]] = None,
                 app_id: int = 0, register: bool = True):
        self.app = app
        self.app_id = app_id
        self.G = G
        self.K, self.nbuf, _ = mm.mm_app_info(app)
        cuda_devices = list(cuda_devices) if cuda_devices is not None else [0] * G
        sm_budgets = list(sm_budgets) if sm_budgets is not None else [0] * G
        if world == 1:
            ranks = [0] * G
        else:
            ranks = list(range(G))
        self.ranks = ranks
        self.rank = rank
        self.world = world
        self.ctx = mm.mm_ctx_create([(cuda_devices[d], sm_budgets[d], ranks[d]) for d in range(G)],
                                    my_rank=rank, world=world, nccl_id=nccl_id)
        self.mine = [ranks[d] == rank for d in range(G)]
        self.cuda_devices = cuda_devices
        self.bufs: Dict[tuple, torch.Tensor] = {}
        for s in range(self.nbuf):
            eb, n = mm.mm_app_buffer_info(app, s)
            for d in range(G):
                if self.mine[d]:
                    self.bufs[(s, d)] = torch.empty(max(n, 1), dtype=_DT[eb],
                                                    device=f"cuda:{cuda_devices[d]}")
        # register the buffers once (mm_buffer_register): runs then pass no
        # pointer array (mm_run with buffers == NULL)
        # (register=False: the caller registers, or passes pointers per run)
        ptrs = self.ptrs()
        for slot in range(self.nbuf if register else 0):
            eb, n = mm.mm_app_buffer_info(app, slot)
            mm.mm_buffer_register(self.ctx, eb, n, ptrs[slot * G:(slot + 1) * G])
        self.registered = register
        self.plans: List[int] = []
        self.tile = 0   # Cholesky tile size (set by session())

    # -- memory ------------------------------------------------------------
    def ptrs(self) -> List[int]:
        out = []
        for s in range(self.nbuf):
            for d in range(self.G):
                t = self.bufs.get((s, d))
                out.append(t.data_ptr() if t is not None else 0)
        return out

    def fill(self, integer: bool = False, seed: int = synthgen.SEED, recipe=None):
        """Generate the app's inputs in place on every owned device (resident
        mode) with the device counter hash (= synthgen)."""
        if self.app_id == mm.MM_APP_NBODY and recipe is None:
            # synthgen.nbody: positions U[-1,1)^3 with masses U[0.5,1) in w,
            # velocities U[-0.01,0.01)^3 with w = 0 (strided fills of the float4s)
            _, n4 = mm.mm_app_buffer_info(self.app, 0)
            n = n4 // 4
            for d in range(self.G):
                if not self.mine[d]:
                    continue
                p, v = self.bufs[(0, d)], self.bufs[(2, d)]
                mm.mm_fill_uniform(self.ctx, d, p.data_ptr(), n4, seed, synthgen.AID_NB_P, 0, -1.0, 1.0)
                mm.mm_fill_uniform(self.ctx, d, v.data_ptr(), n4, seed, synthgen.AID_NB_V, 0, -0.01, 0.01)
                m = torch.empty(n, dtype=torch.float32, device=p.device)
                mm.mm_fill_uniform(self.ctx, d, m.data_ptr(), n, seed, synthgen.AID_NB_P + 100, 0, 0.5, 1.0)
                p.view(n, 4)[:, 3].copy_(m)
                v.view(n, 4)[:, 3].zero_()
            torch.cuda.synchronize()
            return
        if self.app_id == mm.MM_APP_CHOLESKY and recipe is None:
            _, nn = mm.mm_app_buffer_info(self.app, 0)
            n = int(round(nn ** 0.5))
            for d in range(self.G):
                if self.mine[d]:
                    mm.mm_fill_spd_tiles(self.ctx, d, self.bufs[(0, d)].data_ptr(), n, self.tile, seed,
                                         synthgen.AID_CHOL_S)
            return
        rec = recipe or (RECIPES_INT if integer else RECIPES).get(self.app_id, {})
        for slot, r in rec.items():
            for d in range(self.G):
                if not self.mine[d]:
                    continue
                t = self.bufs[(slot, d)]
                _, n = mm.mm_app_buffer_info(self.app, slot)
                if r[0] == "int":
                    mm.mm_fill_integers(self.ctx, d, t.data_ptr(), n, seed, r[1], 0, r[2], r[3])
                else:
                    mm.mm_fill_uniform(self.ctx, d, t.data_ptr(), n, seed, r[0], 0, r[1], r[2])

    def load(self, slot: int, host_array):
        """Copy a host array into every owned copy of a slot (tests)."""
        src = torch.from_numpy(host_array.reshape(-1))
        for d in range(self.G):
            if self.mine[d]:
                self.bufs[(slot, d)][: src.numel()].copy_(src)

    # -- method --------------------------------------------------------------
    def classify(self) -> int:
        return mm.mm_classify(self.app)

    def rank_strategies(self) -> List[int]:
        return mm.mm_rank(self.classify(), mm.mm_needs_sync(self.app))

    def profile(self, **kw) -> mm.mm_profile:
        return mm.mm_profile_run(self.ctx, self.app, self.ptrs(), **kw)

    def equal_profile(self, ps: int = 1000, est_ns: int = 100000, link: int = 10 ** 12) -> mm.mm_profile:
        return mm.make_profile(self.G, [[ps] * mm.MM_MAX_K] * self.G, [[est_ns] * mm.MM_MAX_K] * self.G,
                               [link] * self.G)

    def plan(self, strategy: int, prof: Optional[mm.mm_profile] = None, **opts) -> int:
        prof = prof if prof is not None else self.equal_profile()
        p = mm.mm_plan_build(self.app, prof, mm.plan_opts(strategy, **opts))
        self.plans.append(p)
        return p

    def run(self, plan: int, **kw) -> mm.mm_run_stats:
        return mm.mm_run(self.ctx, plan, None if self.registered else self.ptrs(), **kw)

    def tune_chunks(self, strategy: int, prof: mm.mm_profile, candidates=(1, 2, 4, 8, 16, 32), reps: int = 3,
                    **opts):
        """Task-size auto-tuning (P565) through mm_tune_chunks -> (best, ms per candidate)."""
        return mm.mm_tune_chunks(self.ctx, self.app, prof, mm.plan_opts(strategy, **opts), list(candidates),
                                 self.ptrs(), reps)

    def stream(self, d: int = 0) -> torch.cuda.Stream:
        return torch.cuda.ExternalStream(mm.mm_ctx_stream(self.ctx, d), device=f"cuda:{self.cuda_devices[d]}")

    def collect(self, plan: int, slot: int):
        """Assembled final contents of a buffer slot as a host numpy array."""
        eb, n = mm.mm_app_buffer_info(self.app, slot)
        out = torch.empty(max(n, 1), dtype=_DT[eb], pin_memory=True)
        mm.mm_collect(self.ctx, plan, self.ptrs(), slot, out.data_ptr(), -1)
        return out[:n].numpy().copy()

    def close(self):
        for p in self.plans:
            mm.mm_plan_destroy(p)
        self.plans = []
        if self.ctx:
            torch.cuda.synchronize()
            mm.mm_ctx_destroy(self.ctx)
            self.ctx = 0
        if self.app:
            mm.mm_app_destroy(self.app)
            self.app = 0
        self.bufs.clear()

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def builtin(app_id: int, iparam: Sequence[int] = (), fparam: Sequence[float] = ()) -> int:
    return mm.mm_app_builtin(app_id, iparam, fparam)


def session(app_id: int, iparam: Sequence[int] = (), fparam: Sequence[float] = (), **kw) -> Session:
    s = Session(builtin(app_id, iparam, fparam), app_id=app_id, **kw)
    if app_id == mm.MM_APP_CHOLESKY:
        s.tile = int(iparam[1]) if len(iparam) > 1 and iparam[1] else 1024
    return s
