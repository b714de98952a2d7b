"""ctypes binding of ``include/mm.h`` (libmm.so): same names, marshalling only.

Every ``mm_*`` function here converts Python arguments to the C types of the
header, calls the C entry point of the same name and raises :class:`MMError`
on a non-zero status.  No step of the method runs in Python.  The library is
loaded from this package directory; if it is missing the import fails loudly
(there is no fallback).
"""
from __future__ import annotations

import ctypes as C
import os
from typing import List, Optional, Sequence, Tuple

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libmm.so")

MM_MAX_DEV, MM_MAX_K, MM_MAX_ACCESS, MM_MAX_BUF, MM_MAX_PARAM = 8, 16, 8, 32, 8

(MM_OK, MM_EINVAL, MM_ENOMEM, MM_ECUDA, MM_ENCCL, MM_ESTATE, MM_ENOTSUP,
 MM_ERANGE) = 0, -1, -2, -3, -4, -5, -6, -7
MM_SK_ONE, MM_SK_LOOP, MM_MK_SEQ, MM_MK_LOOP, MM_MK_DAG = 1, 2, 3, 4, 5
MM_SP_SINGLE, MM_SP_UNIFIED, MM_SP_VARIED, MM_DP_PERF, MM_DP_DEP, MM_SP_CYCLIC, MM_DP_STATIC = 1, 2, 3, 4, 5, 6, 7
MM_SYNC_NONE, MM_SYNC_BARRIER, MM_SYNC_FLUSH = 0, 1, 2
MM_READ, MM_WRITE, MM_RW = 1, 2, 3
MM_LINK_PEER, MM_LINK_HOST = 1, 2
(MM_OP_CUSTOM, MM_OP_STREAM_COPY, MM_OP_STREAM_SCALE, MM_OP_STREAM_ADD, MM_OP_STREAM_TRIAD,
 MM_OP_HOTSPOT, MM_OP_ROW_RESIDUAL, MM_OP_BLACKSCHOLES, MM_OP_SGEMM, MM_OP_CHOL_POTRF,
 MM_OP_CHOL_TRSM, MM_OP_CHOL_SYRK, MM_OP_CHOL_GEMM, MM_OP_NBODY) = range(14)
MM_OPK_KERNEL, MM_OPK_XFER, MM_OPK_BARRIER, MM_OPK_FLUSH = 1, 2, 3, 4
(MM_APP_STREAM, MM_APP_HOTSPOT, MM_APP_STENCIL_REDUCTION, MM_APP_BLACKSCHOLES, MM_APP_SGEMM,
 MM_APP_CHOLESKY, MM_APP_NBODY) = 1, 2, 3, 4, 5, 6, 7

STRATEGY_NAMES = {MM_SP_SINGLE: "SP-Single", MM_SP_UNIFIED: "SP-Unified", MM_SP_VARIED: "SP-Varied",
                  MM_DP_PERF: "DP-Perf", MM_DP_DEP: "DP-Dep", MM_SP_CYCLIC: "SP-Cyclic",
                  MM_DP_STATIC: "DP-Static"}
CLASS_NAMES = {MM_SK_ONE: "SK-One", MM_SK_LOOP: "SK-Loop", MM_MK_SEQ: "MK-Seq",
               MM_MK_LOOP: "MK-Loop", MM_MK_DAG: "MK-DAG"}


class MMError(RuntimeError):
    def __init__(self, status: int, fn: str, msg: str):
        super().__init__(f"{fn} -> {status}: {msg}")
        self.status = status


# ----------------------------------------------------------------- structs --
class mm_range(C.Structure):
    _fields_ = [("begin", C.c_int64), ("end", C.c_int64)]


class mm_access(C.Structure):
    _fields_ = [("buffer", C.c_int32), ("mode", C.c_int32), ("elems_per_item", C.c_int64),
                ("halo_items", C.c_int64)]


mm_launch_fn = C.CFUNCTYPE(C.c_int32, C.c_void_p, C.c_int32, mm_range, C.POINTER(C.c_void_p), C.c_void_p)


class mm_kernel_desc(C.Structure):
    _fields_ = [("name", C.c_char_p), ("op", C.c_int32), ("n_items", C.c_int64), ("granule", C.c_int64),
                ("min_items_per_dev", C.c_int64), ("access", mm_access * MM_MAX_ACCESS),
                ("n_access", C.c_int32), ("fparam", C.c_double * MM_MAX_PARAM),
                ("iparam", C.c_int64 * MM_MAX_PARAM), ("launch", mm_launch_fn), ("user", C.c_void_p)]


class mm_task_access(C.Structure):
    _fields_ = [("buffer", C.c_int32), ("mode", C.c_int32), ("lo", C.c_int64), ("hi", C.c_int64)]


class mm_task_desc(C.Structure):
    _fields_ = [("kernel", C.c_int32), ("iparam", C.c_int64 * 4), ("access", mm_task_access * 4),
                ("n_access", C.c_int32), ("lane", C.c_int32)]


class mm_app_params(C.Structure):
    _fields_ = [("iparam", C.c_int64 * MM_MAX_PARAM), ("fparam", C.c_double * MM_MAX_PARAM)]


class mm_profile(C.Structure):
    _fields_ = [("G", C.c_int32), ("K", C.c_int32), ("staged", C.c_int32), ("_pad", C.c_int32),
                ("fs_item", (C.c_uint64 * MM_MAX_K) * MM_MAX_DEV),
                ("chunk_est_ns", (C.c_uint64 * MM_MAX_K) * MM_MAX_DEV),
                ("link_Bps", C.c_uint64 * MM_MAX_DEV), ("link_lat_ns", C.c_uint64 * MM_MAX_DEV)]


class mm_plan_opts(C.Structure):
    _fields_ = [("strategy", C.c_int32), ("chunks_per_dev", C.c_int32), ("staged", C.c_int32),
                ("grid_rows", C.c_int32), ("one_shot", C.c_int32), ("pipeline", C.c_int32),
                ("split", C.POINTER(mm_range)), ("halo_split", C.c_int32), ("_pad2", C.c_int32)]


class mm_chunk(C.Structure):
    _fields_ = [("kernel", C.c_int32), ("device", C.c_int32), ("iter", C.c_int64), ("items", mm_range),
                ("finish_ns", C.c_uint64)]


class mm_op_rec(C.Structure):
    _fields_ = [("kind", C.c_int32), ("device", C.c_int32), ("src", C.c_int32), ("kernel", C.c_int32),
                ("buffer", C.c_int32), ("_pad", C.c_int32), ("task", C.c_int64), ("iter", C.c_int64),
                ("r", mm_range)]


class mm_plan_info_t(C.Structure):
    _fields_ = [("cls", C.c_int32), ("strategy", C.c_int32), ("G", C.c_int32), ("devices_used", C.c_int32),
                ("n_tasks", C.c_int64), ("n_ops", C.c_int64), ("n_kernel_ops", C.c_int64),
                ("n_xfer_ops", C.c_int64), ("n_barriers", C.c_int64), ("n_flush_ops", C.c_int64),
                ("xfer_bytes", C.c_int64), ("flush_bytes", C.c_int64), ("h2d_bytes", C.c_int64),
                ("items", (C.c_int64 * MM_MAX_K) * MM_MAX_DEV)]


class mm_device_spec(C.Structure):
    _fields_ = [("cuda_device", C.c_int32), ("sm_budget", C.c_int32), ("rank", C.c_int32),
                ("_pad", C.c_int32)]


class mm_profile_opts(C.Structure):
    _fields_ = [("probe_items", C.c_int64), ("reps", C.c_int32), ("dp_warmup_chunks", C.c_int32),
                ("chunks_per_dev", C.c_int32), ("measure_link", C.c_int32)]


class mm_run_opts(C.Structure):
    _fields_ = [("use_graph", C.c_int32), ("time_kernels", C.c_int32), ("adaptive", C.c_int32),
                ("max_inflight", C.c_int32), ("host", C.POINTER(C.c_void_p)), ("no_wait", C.c_int32),
                ("repeat", C.c_int32)]


class mm_decision(C.Structure):
    _fields_ = [("task", C.c_int64), ("chosen", C.c_int32), ("kernel", C.c_int32), ("now_ns", C.c_uint64),
                ("busy_ns", C.c_uint64 * MM_MAX_DEV), ("ready_ns", C.c_uint64 * MM_MAX_DEV),
                ("cost_ns", C.c_uint64 * MM_MAX_DEV), ("eft_ns", C.c_uint64 * MM_MAX_DEV)]


class mm_run_stats(C.Structure):
    _fields_ = [("wall_ms", C.c_double), ("device_ms", C.c_double),
                ("kernel_ms", (C.c_double * MM_MAX_K) * MM_MAX_DEV),
                ("kernel_launches", (C.c_int64 * MM_MAX_K) * MM_MAX_DEV),
                ("n_launches", C.c_int64), ("xfer_bytes", C.c_int64), ("h2d_bytes", C.c_int64),
                ("d2h_bytes", C.c_int64)]


ABI_STRUCTS = [mm_range, mm_access, mm_kernel_desc, mm_task_access, mm_task_desc, mm_app_params,
               mm_profile, mm_plan_opts, mm_chunk, mm_op_rec, mm_plan_info_t, mm_device_spec,
               mm_profile_opts, mm_run_opts, mm_run_stats, mm_decision]

# ---------------------------------------------------------------- loading --
if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with `python -m "
                      "paper_conf_icpp_shenvms15_b200.build` (no fallback exists)")
lib = C.CDLL(LIB_PATH)

_P = C.c_void_p
_SIGS = {
    "mm_app_create": [C.POINTER(_P)],
    "mm_app_add_buffer": [_P, C.c_int32, C.c_int64, C.POINTER(C.c_int32)],
    "mm_app_add_kernel": [_P, C.POINTER(mm_kernel_desc), C.POINTER(C.c_int32)],
    "mm_app_add_edge": [_P, C.c_int32, C.c_int32],
    "mm_app_set_loop": [_P, C.c_int32, C.c_int32, C.c_int64],
    "mm_app_set_sync": [_P, C.c_int32, C.c_int32],
    "mm_app_set_swap": [_P, C.c_int32, C.c_int32],
    "mm_app_set_unstable": [_P, C.c_int32],
    "mm_app_set_lane": [_P, C.c_int32, C.c_int32],
    "mm_app_add_task": [_P, C.POINTER(mm_task_desc)],
    "mm_app_builtin": [C.c_int32, C.POINTER(mm_app_params), C.POINTER(_P)],
    "mm_app_info": [_P, C.POINTER(C.c_int32), C.POINTER(C.c_int32), C.POINTER(C.c_int64)],
    "mm_app_buffer_info": [_P, C.c_int32, C.POINTER(C.c_int32), C.POINTER(C.c_int64)],
    "mm_classify": [_P, C.POINTER(C.c_int32)],
    "mm_needs_sync": [_P, C.POINTER(C.c_int32)],
    "mm_rank": [C.c_int32, C.c_int32, C.POINTER(C.c_int32), C.c_int32, C.POINTER(C.c_int32)],
    "mm_split": [_P, C.POINTER(mm_profile), C.c_int32, C.POINTER(mm_range), C.c_int32, C.POINTER(C.c_int32)],
    "mm_schedule": [_P, C.POINTER(mm_profile), C.POINTER(mm_plan_opts), C.POINTER(mm_chunk), C.c_int64,
                    C.POINTER(C.c_int64)],
    "mm_plan_build": [_P, C.POINTER(mm_profile), C.POINTER(mm_plan_opts), C.POINTER(_P)],
    "mm_plan_info": [_P, C.POINTER(mm_plan_info_t)],
    "mm_plan_ranges": [_P, C.POINTER(mm_range), C.c_int32, C.POINTER(C.c_int32)],
    "mm_plan_chunks": [_P, C.POINTER(mm_chunk), C.c_int64, C.POINTER(C.c_int64)],
    "mm_plan_ops": [_P, C.POINTER(mm_op_rec), C.c_int64, C.POINTER(C.c_int64)],
    "mm_plan_owners": [_P, C.c_int32, C.POINTER(mm_range), C.POINTER(C.c_int32), C.c_int64,
                       C.POINTER(C.c_int64)],
    "mm_nccl_unique_id": [C.c_void_p],
    "mm_rendezvous_id": [C.c_void_p],
    "mm_ctx_create": [C.POINTER(mm_device_spec), C.c_int32, C.c_int32, C.c_int32, C.c_void_p, C.POINTER(_P)],
    "mm_ctx_stream": [_P, C.c_int32, C.POINTER(_P)],
    "mm_ctx_sm_count": [_P, C.c_int32, C.POINTER(C.c_int32)],
    "mm_ctx_set_stream": [_P, C.c_int32, C.c_void_p],
    "mm_buffer_register": [_P, C.c_int32, C.c_int64, C.POINTER(_P), C.POINTER(C.c_int32)],
    "mm_app_finalize": [_P],
    "mm_fill_uniform": [_P, C.c_int32, C.c_void_p, C.c_int64, C.c_uint64, C.c_int32, C.c_int64, C.c_float,
                        C.c_float],
    "mm_fill_integers": [_P, C.c_int32, C.c_void_p, C.c_int64, C.c_uint64, C.c_int32, C.c_int64, C.c_int32,
                         C.c_int32],
    "mm_fill_spd_tiles": [_P, C.c_int32, C.c_void_p, C.c_int64, C.c_int64, C.c_uint64, C.c_int32],
    "mm_profile_run": [_P, _P, C.POINTER(_P), C.POINTER(mm_profile_opts), C.POINTER(mm_profile)],
    "mm_run": [_P, _P, C.POINTER(_P), C.POINTER(mm_run_opts), C.POINTER(mm_run_stats)],
    "mm_collect": [_P, _P, C.POINTER(_P), C.c_int32, C.c_void_p, C.c_int32],
    "mm_run_decisions": [_P, C.POINTER(mm_decision), C.c_int64, C.POINTER(C.c_int64)],
    "mm_tune_chunks": [_P, _P, C.POINTER(mm_profile), C.POINTER(mm_plan_opts), C.POINTER(C.c_int32), C.c_int32,
                       C.POINTER(_P), C.c_int32, C.POINTER(C.c_int32), C.POINTER(C.c_double)],
    "mm_abi_sizes": [C.POINTER(C.c_int64), C.c_int32, C.POINTER(C.c_int32)],
}
for _name, _args in _SIGS.items():
    _f = getattr(lib, _name)
    _f.argtypes = _args
    _f.restype = C.c_int32
for _name in ("mm_app_destroy", "mm_plan_destroy", "mm_ctx_destroy"):
    getattr(lib, _name).argtypes = [_P]
    getattr(lib, _name).restype = None
lib.mm_last_error.restype = C.c_char_p
lib.mm_strategy_name.restype = C.c_char_p
lib.mm_strategy_name.argtypes = [C.c_int32]
lib.mm_class_name.restype = C.c_char_p
lib.mm_class_name.argtypes = [C.c_int32]
lib.mm_kernel_launch_count.restype = C.c_int64

# Every symbol the header declares (the CPU suite checks the export list).
EXPORTS = sorted(list(_SIGS) + ["mm_app_destroy", "mm_plan_destroy", "mm_ctx_destroy", "mm_last_error",
                                "mm_strategy_name", "mm_class_name", "mm_kernel_launch_count"])


def _check(st: int, fn: str):
    if st != MM_OK:
        raise MMError(st, fn, (lib.mm_last_error() or b"").decode())


_FN = {}


def _call(fn: str, *args):
    f = _FN.get(fn)
    if f is None:
        f = _FN[fn] = getattr(lib, fn)
    st = f(*args)
    if st:
        _check(st, fn)


# --------------------------------------------------------- same-name calls --
def mm_last_error() -> str:
    return (lib.mm_last_error() or b"").decode()


def mm_abi_sizes() -> List[int]:
    out = (C.c_int64 * 32)()
    n = C.c_int32()
    _call("mm_abi_sizes", out, 32, C.byref(n))
    return list(out[:n.value])


def mm_app_create() -> int:
    h = _P()
    _call("mm_app_create", C.byref(h))
    return h.value


def mm_app_destroy(app: int):
    lib.mm_app_destroy(app)


def mm_app_add_buffer(app: int, elem_bytes: int, n_elems: int) -> int:
    s = C.c_int32()
    _call("mm_app_add_buffer", app, elem_bytes, n_elems, C.byref(s))
    return s.value


def kernel_desc(name: str, op: int, n_items: int, accesses: Sequence[Tuple[int, int, int, int]],
                granule: int = 32, min_items: int = 1, fparam=(), iparam=()) -> mm_kernel_desc:
    """Marshal a kernel descriptor; accesses = [(buffer, mode, elems_per_item, halo)]."""
    d = mm_kernel_desc()
    d.name = name.encode()
    d.op = op
    d.n_items = n_items
    d.granule = granule
    d.min_items_per_dev = min_items
    for i, (b, m, e, h) in enumerate(accesses):
        d.access[i] = mm_access(b, m, e, h)
    d.n_access = len(accesses)
    for i, v in enumerate(fparam):
        d.fparam[i] = v
    for i, v in enumerate(iparam):
        d.iparam[i] = v
    return d


def mm_app_add_kernel(app: int, desc: mm_kernel_desc) -> int:
    k = C.c_int32()
    _call("mm_app_add_kernel", app, C.byref(desc), C.byref(k))
    return k.value


def mm_app_add_edge(app: int, a: int, b: int):
    _call("mm_app_add_edge", app, a, b)


def mm_app_set_loop(app: int, first: int, last: int, iterations: int):
    _call("mm_app_set_loop", app, first, last, iterations)


def mm_app_set_sync(app: int, kernel: int, sync: int):
    _call("mm_app_set_sync", app, kernel, sync)


def mm_app_set_swap(app: int, a: int, b: int):
    _call("mm_app_set_swap", app, a, b)


def mm_app_set_unstable(app: int, unstable: bool):
    _call("mm_app_set_unstable", app, int(unstable))


def mm_app_set_lane(app: int, kernel: int, lane: int):
    _call("mm_app_set_lane", app, kernel, lane)


def mm_app_add_task(app: int, kernel: int, iparam: Sequence[int],
                    accesses: Sequence[Tuple[int, int, int, int]], lane: int = 0):
    t = mm_task_desc()
    t.kernel = kernel
    t.lane = lane
    for i, v in enumerate(iparam):
        t.iparam[i] = v
    for i, (b, m, lo, hi) in enumerate(accesses):
        t.access[i] = mm_task_access(b, m, lo, hi)
    t.n_access = len(accesses)
    _call("mm_app_add_task", app, C.byref(t))


def mm_app_builtin(app_id: int, iparam: Sequence[int] = (), fparam: Sequence[float] = ()) -> int:
    p = mm_app_params()
    for i, v in enumerate(iparam):
        p.iparam[i] = int(v)
    for i, v in enumerate(fparam):
        p.fparam[i] = float(v)
    h = _P()
    _call("mm_app_builtin", app_id, C.byref(p), C.byref(h))
    return h.value


def mm_app_info(app: int) -> Tuple[int, int, int]:
    k, b, t = C.c_int32(), C.c_int32(), C.c_int64()
    _call("mm_app_info", app, C.byref(k), C.byref(b), C.byref(t))
    return k.value, b.value, t.value


def mm_app_buffer_info(app: int, slot: int) -> Tuple[int, int]:
    eb, n = C.c_int32(), C.c_int64()
    _call("mm_app_buffer_info", app, slot, C.byref(eb), C.byref(n))
    return eb.value, n.value


def mm_classify(app: int) -> int:
    c = C.c_int32()
    _call("mm_classify", app, C.byref(c))
    return c.value


def mm_needs_sync(app: int) -> bool:
    c = C.c_int32()
    _call("mm_needs_sync", app, C.byref(c))
    return bool(c.value)


def mm_rank(cls: int, needs_sync: bool) -> List[int]:
    out = (C.c_int32 * 8)()
    n = C.c_int32()
    _call("mm_rank", cls, int(needs_sync), out, 8, C.byref(n))
    return list(out[:n.value])


def make_profile(G: int, fs_item, chunk_est_ns=None, link_Bps=None, staged: bool = False,
                 link_lat_ns=None) -> mm_profile:
    """Marshal a profile from nested lists fs_item[d][k] (fs), chunk_est_ns[d][k], link_Bps[d],
    link_lat_ns[d]."""
    p = mm_profile()
    p.G = G
    p.K = MM_MAX_K
    p.staged = int(staged)
    for d in range(G):
        for k, v in enumerate(fs_item[d]):
            p.fs_item[d][k] = int(v)
        if chunk_est_ns is not None:
            for k, v in enumerate(chunk_est_ns[d]):
                p.chunk_est_ns[d][k] = int(v)
        if link_Bps is not None:
            p.link_Bps[d] = int(link_Bps[d])
        if link_lat_ns is not None:
            p.link_lat_ns[d] = int(link_lat_ns[d])
    return p


def mm_split(app: int, prof: mm_profile, strategy: int) -> Tuple[List[List[Tuple[int, int]]], int]:
    K = mm_app_info(app)[0]
    G = prof.G
    out = (mm_range * (K * G))()
    used = C.c_int32()
    _call("mm_split", app, C.byref(prof), strategy, out, K * G, C.byref(used))
    return [[(out[k * G + d].begin, out[k * G + d].end) for d in range(G)] for k in range(K)], used.value


def plan_opts(strategy: int, chunks_per_dev: int = 8, staged: bool = False, grid_rows: int = 0,
              split=None, one_shot: bool = False, pipeline: int = 0, halo_split: bool = False) -> mm_plan_opts:
    o = mm_plan_opts()
    o.pipeline = pipeline
    o.halo_split = int(halo_split)
    o.strategy = strategy
    o.chunks_per_dev = chunks_per_dev
    o.staged = int(staged)
    o.grid_rows = grid_rows
    o.one_shot = int(one_shot)
    if split is not None:
        flat = [r for row in split for r in row]
        arr = (mm_range * len(flat))(*[mm_range(b, e) for b, e in flat])
        o._split_keep = arr
        o.split = C.cast(arr, C.POINTER(mm_range))
    return o


def mm_schedule(app: int, prof: mm_profile, opts: mm_plan_opts) -> List[mm_chunk]:
    n = C.c_int64()
    st = lib.mm_schedule(app, C.byref(prof), C.byref(opts), None, 0, C.byref(n))
    if st not in (MM_OK, MM_ERANGE):
        _check(st, "mm_schedule")
    out = (mm_chunk * max(1, n.value))()
    _call("mm_schedule", app, C.byref(prof), C.byref(opts), out, n.value, C.byref(n))
    return list(out[:n.value])


def mm_plan_build(app: int, prof: mm_profile, opts: mm_plan_opts) -> int:
    h = _P()
    _call("mm_plan_build", app, C.byref(prof), C.byref(opts), C.byref(h))
    return h.value


def mm_plan_destroy(plan: int):
    lib.mm_plan_destroy(plan)


def mm_plan_info(plan: int) -> mm_plan_info_t:
    i = mm_plan_info_t()
    _call("mm_plan_info", plan, C.byref(i))
    return i


def mm_plan_ranges(plan: int) -> List[Tuple[int, int]]:
    n = C.c_int32()
    lib.mm_plan_ranges(plan, None, 0, C.byref(n))
    out = (mm_range * max(1, n.value))()
    _call("mm_plan_ranges", plan, out, n.value, C.byref(n))
    return [(r.begin, r.end) for r in out[:n.value]]


def mm_plan_chunks(plan: int) -> List[mm_chunk]:
    n = C.c_int64()
    lib.mm_plan_chunks(plan, None, 0, C.byref(n))
    out = (mm_chunk * max(1, n.value))()
    _call("mm_plan_chunks", plan, out, n.value, C.byref(n))
    return list(out[:n.value])


def mm_plan_ops(plan: int) -> List[mm_op_rec]:
    n = C.c_int64()
    lib.mm_plan_ops(plan, None, 0, C.byref(n))
    out = (mm_op_rec * max(1, n.value))()
    _call("mm_plan_ops", plan, out, n.value, C.byref(n))
    return list(out[:n.value])


def mm_plan_owners(plan: int, slot: int) -> List[Tuple[int, int, int]]:
    """[(begin, end, owner_device)] covering the slot's elements."""
    n = C.c_int64()
    lib.mm_plan_owners(plan, slot, None, None, 0, C.byref(n))
    rr = (mm_range * max(1, n.value))()
    oo = (C.c_int32 * max(1, n.value))()
    _call("mm_plan_owners", plan, slot, rr, oo, n.value, C.byref(n))
    return [(rr[i].begin, rr[i].end, oo[i]) for i in range(n.value)]


def mm_rendezvous_id() -> bytes:
    """128 random bytes naming a multi-process context (IPC transport)."""
    buf = C.create_string_buffer(128)
    _call("mm_rendezvous_id", buf)
    return buf.raw


def mm_nccl_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    _call("mm_nccl_unique_id", buf)
    return buf.raw


def mm_ctx_create(devices: Sequence[Tuple[int, int, int]], my_rank: int = 0, world: int = 1,
                  nccl_id: Optional[bytes] = None) -> int:
    """devices = [(cuda_device, sm_budget, rank)] per logical device."""
    G = len(devices)
    specs = (mm_device_spec * G)(*[mm_device_spec(c, s, r, 0) for (c, s, r) in devices])
    h = _P()
    idb = C.create_string_buffer(nccl_id, 128) if nccl_id else None
    _call("mm_ctx_create", specs, G, my_rank, world, idb, C.byref(h))
    return h.value


def mm_ctx_destroy(ctx: int):
    lib.mm_ctx_destroy(ctx)


def mm_ctx_stream(ctx: int, d: int) -> int:
    s = _P()
    _call("mm_ctx_stream", ctx, d, C.byref(s))
    return s.value or 0


def mm_ctx_sm_count(ctx: int, d: int) -> int:
    s = C.c_int32()
    _call("mm_ctx_sm_count", ctx, d, C.byref(s))
    return s.value


def mm_ctx_set_stream(ctx: int, d: int, stream: int):
    """Order device d's runs with a caller stream (torch ``Stream.cuda_stream``); 0 clears it."""
    _call("mm_ctx_set_stream", ctx, d, stream or None)


def mm_buffer_register(ctx: int, elem_bytes: int, n_elems: int, dev_ptrs: Sequence[int]) -> int:
    """Register app buffer slot i (i-th call): one caller-owned device pointer per logical device."""
    b = C.c_int32()
    _call("mm_buffer_register", ctx, elem_bytes, n_elems, _ptr_array(dev_ptrs), C.byref(b))
    return b.value


def mm_app_finalize(app: int):
    _call("mm_app_finalize", app)


def mm_fill_uniform(ctx: int, d: int, ptr: int, n: int, seed: int, array_id: int, start: int,
                    lo: float, hi: float):
    _call("mm_fill_uniform", ctx, d, ptr, n, seed, array_id, start, lo, hi)


def mm_fill_integers(ctx: int, d: int, ptr: int, n: int, seed: int, array_id: int, start: int,
                     lo: int, hi: int):
    _call("mm_fill_integers", ctx, d, ptr, n, seed, array_id, start, lo, hi)


def mm_fill_spd_tiles(ctx: int, d: int, ptr: int, n: int, b: int, seed: int, array_id: int):
    _call("mm_fill_spd_tiles", ctx, d, ptr, n, b, seed, array_id)


def _ptr_array(ptrs: Sequence[int]):
    return (C.c_void_p * len(ptrs))(*[p or None for p in ptrs])


def mm_profile_run(ctx: int, app: int, buffers: Sequence[int], reps: int = 5, dp_warmup_chunks: int = 3,
                   chunks_per_dev: int = 8, probe_items: int = 0, link: str = "peer") -> mm_profile:
    """link = "peer" (resident exchanges) or "host" (staged: pinned PCIe copies; sets prof.staged)."""
    o = mm_profile_opts(probe_items, reps, dp_warmup_chunks, chunks_per_dev,
                        {"peer": MM_LINK_PEER, "host": MM_LINK_HOST}[link])
    p = mm_profile()
    _call("mm_profile_run", ctx, app, _ptr_array(buffers), C.byref(o), C.byref(p))
    return p


def mm_run(ctx: int, plan: int, buffers: Optional[Sequence[int]], use_graph: bool = False, time_kernels: bool = False,
           host: Optional[Sequence[int]] = None, adaptive: bool = False, max_inflight: int = 0,
           no_wait: bool = False, repeat: int = 1) -> mm_run_stats:
    o = mm_run_opts()
    o.repeat = int(repeat)
    o.use_graph = int(use_graph)
    o.no_wait = int(no_wait)
    o.time_kernels = int(time_kernels)
    o.adaptive = int(adaptive)
    o.max_inflight = int(max_inflight)
    if host is not None:
        harr = _ptr_array(host)
        o.host = C.cast(harr, C.POINTER(C.c_void_p))
    st = mm_run_stats()
    _call("mm_run", ctx, plan, None if buffers is None else _ptr_array(buffers), C.byref(o), C.byref(st))
    return st


def mm_tune_chunks(ctx: int, app: int, prof: mm_profile, opts: mm_plan_opts, candidates: Sequence[int],
                   buffers: Sequence[int], reps: int = 3):
    """-> (best chunks_per_dev, [median device ms per candidate])."""
    cand = (C.c_int32 * len(candidates))(*candidates)
    times = (C.c_double * len(candidates))()
    best = C.c_int32()
    _call("mm_tune_chunks", ctx, app, C.byref(prof), C.byref(opts), cand, len(candidates), _ptr_array(buffers),
          reps, C.byref(best), times)
    return best.value, list(times)


def mm_run_decisions(plan: int) -> List[mm_decision]:
    n = C.c_int64()
    lib.mm_run_decisions(plan, None, 0, C.byref(n))
    out = (mm_decision * max(1, n.value))()
    _call("mm_run_decisions", plan, out, n.value, C.byref(n))
    return list(out[:n.value])


def mm_collect(ctx: int, plan: int, buffers: Optional[Sequence[int]], slot: int, dst: int, dst_device: int = -1):
    _call("mm_collect", ctx, plan, None if buffers is None else _ptr_array(buffers), slot, dst, dst_device)


def mm_kernel_launch_count() -> int:
    return lib.mm_kernel_launch_count()


def mm_strategy_name(s: int) -> str:
    return lib.mm_strategy_name(s).decode()


def mm_class_name(c: int) -> str:
    return lib.mm_class_name(c).decode()
