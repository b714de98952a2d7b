"""ORACLE — ctypes front of ``oracle/numeric.c`` (plain single-threaded C).

TEST INFRASTRUCTURE ONLY (see the header of numeric.c).  Builds
``oracle/_numeric.so`` with gcc on first use (``build()`` in
``__graft_entry__`` also builds it).  Every wrapper takes/returns numpy arrays
and cites the same passages as the C function it calls.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "numeric.c")
_SO = os.path.join(_HERE, "_numeric.so")
_lib = None

# HotSpot coefficients (R15): Rodinia's values at its 1024^2 grid,
# derived from chip 0.016 m, t_chip 5e-4, K_SI 100, SPEC_HEAT_SI 1.75e6,
# FACTOR_CHIP 0.5, MAX_PD 3e6, PRECISION 1e-3 [ext]:
#   Rx = Ry = 1/(2 K t) = 10 -> rx1 = ry1 = 0.1; Rz = t/(K g^2) -> rz1 = 1/20480
#   step/Cap = (PRECISION/max_slope) / (FACTOR_CHIP*SPEC_HEAT*t*g^2) = 1.3653333
HOT_SDC = 1.3653333333333333
HOT_RX1 = 0.1
HOT_RY1 = 0.1
HOT_RZ1 = 1.0 / 20480.0
HOT_AMB = 80.0
BS_R, BS_V = 0.02, 0.30     # NVIDIA SDK riskfree / volatility [ext]
STREAM_SCALAR = 3.0         # STREAM's scalar [ext, McCalpin]


class HotCoef(C.Structure):
    _fields_ = [("sdc", C.c_float), ("rx1", C.c_float), ("ry1", C.c_float),
                ("rz1", C.c_float), ("amb", C.c_float)]


def hot_coef() -> HotCoef:
    return HotCoef(HOT_SDC, HOT_RX1, HOT_RY1, HOT_RZ1, HOT_AMB)


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math",
                               "-shared", "-fPIC", "-o", _SO, _SRC, "-lm"])
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_SO)
        f32p = np.ctypeslib.ndpointer(np.float32, flags="C_CONTIGUOUS")
        f64p = np.ctypeslib.ndpointer(np.float64, flags="C_CONTIGUOUS")
        i64 = C.c_int64
        L.or_stream_copy.argtypes = [f32p, f32p, i64, i64]
        L.or_stream_scale.argtypes = [f32p, f32p, C.c_float, i64, i64]
        L.or_stream_add.argtypes = [f32p, f32p, f32p, i64, i64]
        L.or_stream_triad.argtypes = [f32p, f32p, f32p, C.c_float, i64, i64]
        L.or_stream_run.argtypes = [f32p, f32p, f32p, i64, C.c_float, C.c_int32]
        L.or_hotspot_rows.argtypes = [f32p, f32p, f32p, i64, i64, i64, i64, C.POINTER(HotCoef)]
        L.or_hotspot_run.argtypes = [f32p, f32p, f32p, i64, i64, C.c_int32, C.POINTER(HotCoef)]
        L.or_hotspot_run.restype = C.c_int32
        L.or_row_residual.argtypes = [f32p, f32p, f64p, i64, i64, i64]
        L.or_cnd_public.argtypes = [C.c_double]
        L.or_cnd_public.restype = C.c_double
        L.or_blackscholes.argtypes = [f32p, f32p, f32p, f64p, f64p, i64, C.c_double, C.c_double]
        L.or_sgemm_rows.argtypes = [f32p, f32p, f32p, i64, i64, i64, i64, i64, f64p]
        L.or_cholesky.argtypes = [f64p, f64p, i64]
        L.or_cholesky.restype = C.c_int32
        _lib = L
    return _lib


# --- STREAM (P203, P473; McCalpin [22]) ------------------------------------
def stream_copy(a, c, lo=0, hi=None):
    lib().or_stream_copy(a, c, lo, len(a) if hi is None else hi)


def stream_scale(b, c, s=STREAM_SCALAR, lo=0, hi=None):
    lib().or_stream_scale(b, c, s, lo, len(b) if hi is None else hi)


def stream_add(a, b, c, lo=0, hi=None):
    lib().or_stream_add(a, b, c, lo, len(a) if hi is None else hi)


def stream_triad(a, b, c, s=STREAM_SCALAR, lo=0, hi=None):
    lib().or_stream_triad(a, b, c, s, lo, len(a) if hi is None else hi)


def stream_run(a, b, c, passes=1, s=STREAM_SCALAR):
    """In place on copies; returns (a, b, c)."""
    a, b, c = a.copy(), b.copy(), c.copy()
    lib().or_stream_run(a, b, c, len(a), s, passes)
    return a, b, c


# --- HotSpot (P319; Rodinia [2]) -------------------------------------------
def hotspot_rows(tin, pw, tout, r0=0, r1=None, coef=None):
    rows, cols = tin.shape
    k = hot_coef() if coef is None else coef
    lib().or_hotspot_rows(tin.reshape(-1), pw.reshape(-1), tout.reshape(-1), rows, cols,
                          r0, rows if r1 is None else r1, C.byref(k))


def hotspot_block_rows(tin, pw, tout, r0, r1, h, coef=None):
    """Temporal block of h iterations for rows [r0, r1) (SURVEY §8(f) f3,
    Rodinia's pyramid): only rows [r0-h, r1+h) of ``tin`` are read.  Written
    out as h single steps over shrinking row bands: step s (1..h) recomputes
    rows [r0-h+s, r1+h-s) (clipped to the grid) from step s-1, so step h holds
    rows [r0, r1) exactly as h full-grid iterations would (P319 + R16)."""
    rows, cols = tin.shape
    cur = np.array(tin, dtype=np.float32, copy=True)
    for s in range(1, h + 1):
        lo, hi = max(0, r0 - h + s), min(rows, r1 + h - s)
        nxt = cur.copy()
        hotspot_rows(cur, pw, nxt, lo, hi, coef)
        cur = nxt
    tout[r0:r1] = cur[r0:r1]


def hotspot_run(t0, pw, iters):
    rows, cols = t0.shape
    a = np.ascontiguousarray(t0, dtype=np.float32).copy()
    b = np.empty_like(a)
    k = hot_coef()
    which = lib().or_hotspot_run(a.reshape(-1), b.reshape(-1), np.ascontiguousarray(pw).reshape(-1),
                                 rows, cols, iters, C.byref(k))
    return a if which == 0 else b


def row_residual(t0, t1, r0=0, r1=None):
    rows, cols = t0.shape
    out = np.zeros(rows, dtype=np.float64)
    lib().or_row_residual(t0.reshape(-1), t1.reshape(-1), out, cols, r0,
                          rows if r1 is None else r1)
    return out


def stencil_reduction_run(t0, pw, steps):
    """MK-Loop app (BASELINE configs[3]): per step, kernel A = HotSpot update,
    kernel B = per-row residual; r_t = sum of row sums (math.fsum: correctly
    rounded, so independent of any summation order).  Returns (T, [r_t])."""
    import math
    cur = np.ascontiguousarray(t0, dtype=np.float32).copy()
    nxt = np.empty_like(cur)
    rs = []
    for _ in range(steps):
        hotspot_rows(cur, pw, nxt)
        rs.append(math.fsum(row_residual(cur, nxt)))
        cur, nxt = nxt, cur
    return cur, rs


# --- BlackScholes (P311; NVIDIA SDK) ---------------------------------------
def cnd(d: float) -> float:
    return lib().or_cnd_public(d)


def blackscholes(S, X, T, R=BS_R, V=BS_V):
    n = len(S)
    call = np.empty(n, np.float64)
    put = np.empty(n, np.float64)
    lib().or_blackscholes(S, X, T, call, put, n, R, V)
    return call, put


# --- MatrixMul (P311) -------------------------------------------------------
def sgemm(A, B, r0=0, r1=None):
    M, K = A.shape
    K2, N = B.shape
    assert K == K2
    Cm = np.zeros((M, N), np.float32)
    acc = np.zeros(N, np.float64)
    lib().or_sgemm_rows(np.ascontiguousarray(A).reshape(-1), np.ascontiguousarray(B).reshape(-1),
                        Cm.reshape(-1), M, N, K, r0, M if r1 is None else r1, acc)
    return Cm


# --- Cholesky (BASELINE configs[4]) ----------------------------------------
def cholesky(A):
    n = A.shape[0]
    L = np.zeros((n, n), np.float64)
    rc = lib().or_cholesky(np.ascontiguousarray(A, dtype=np.float64).reshape(-1), L.reshape(-1), n)
    if rc != 0:
        raise ValueError(f"not positive definite at row {-rc - 1}")
    return L


# --- Nbody (P223-227, P319; CUDA SDK integrator) ---------------------------
NBODY_DT, NBODY_EPS2 = 1e-3, 1e-2


def _nbody_lib():
    L = lib()
    if not hasattr(L, "_nbody_ready"):
        f32p = np.ctypeslib.ndpointer(np.float32, flags="C_CONTIGUOUS")
        L.or_nbody_step.argtypes = [f32p, f32p, f32p, f32p, C.c_int64, C.c_int64, C.c_int64,
                                    C.c_double, C.c_double]
        L._nbody_ready = True
    return L


def nbody_step_bodies(pos, vel, bodies, dt=NBODY_DT, eps2=NBODY_EPS2):
    """One step for the listed bodies only (each sums over ALL n bodies):
    returns (pos', vel') rows of shape (len(bodies), 4)."""
    L = _nbody_lib()
    n = pos.shape[0]
    p = np.ascontiguousarray(pos, dtype=np.float32)
    v = np.ascontiguousarray(vel, dtype=np.float32)
    p2, v2 = np.zeros_like(p), np.zeros_like(v)
    for i in bodies:
        L.or_nbody_step(p.reshape(-1), v.reshape(-1), p2.reshape(-1), v2.reshape(-1), n, int(i), int(i) + 1,
                        dt, eps2)
    idx = np.asarray(bodies)
    return p2[idx].copy(), v2[idx].copy()


def nbody_run(pos, vel, iters, dt=NBODY_DT, eps2=NBODY_EPS2):
    """pos, vel: (n, 4) float32.  Returns (pos, vel) after `iters` steps."""
    L = _nbody_lib()
    n = pos.shape[0]
    p = np.ascontiguousarray(pos, dtype=np.float32).copy()
    v = np.ascontiguousarray(vel, dtype=np.float32).copy()
    p2, v2 = np.empty_like(p), np.empty_like(v)
    for _ in range(iters):
        L.or_nbody_step(p.reshape(-1), v.reshape(-1), p2.reshape(-1), v2.reshape(-1), n, 0, n, dt, eps2)
        p, p2 = p2, p
        v, v2 = v2, v
    return p, v
