"""ORACLE — descriptors of the paper's applications for the control-plane oracle.

TEST INFRASTRUCTURE ONLY.  Kernel structure per Table II (P205-247) and the
workload text of §IV-B (P311, P319, P473, P533).  Buffer slots and access
patterns are the oracle's own statement of what each kernel reads/writes.
"""
from __future__ import annotations

from .control import (App, Access, Kernel, Task, TaskAccess, READ, WRITE, RW,
                      SYNC_BARRIER, SYNC_NONE)


def stream(n: int, passes: int = 1, sync: int = SYNC_NONE, granule: int = 32,
           min_items: int = 1) -> App:
    """STREAM (P235-245, P473): copy c=a; scale b=s c; add c=a+b; triad
    a=b+s c.  Buffers a=0, b=1, c=2 (4-byte elements).  STREAM-Seq: passes=1
    (MK-Seq); STREAM-Loop: passes>1 (MK-Loop, P533)."""
    ks = [
        Kernel("copy", n, granule, min_items, [Access(0, READ), Access(2, WRITE)]),
        Kernel("scale", n, granule, min_items, [Access(2, READ), Access(1, WRITE)]),
        Kernel("add", n, granule, min_items, [Access(0, READ), Access(1, READ), Access(2, WRITE)]),
        Kernel("triad", n, granule, min_items, [Access(1, READ), Access(2, READ), Access(0, WRITE)]),
    ]
    app = App(buffers=[(4, n)] * 3, kernels=ks)
    if passes > 1:
        app.loop = (0, 3, passes)
    if sync != SYNC_NONE:
        app.sync = {k: sync for k in range(4)}
    return app


def hotspot(rows: int, cols: int, iters: int, granule: int = 1, min_items: int = 1, tb: int = 1) -> App:
    """HotSpot (P229-233, P319): one stencil kernel iterated (SK-Loop), row-wise
    split; slots T_in=0, T_out=1 (ping-pong), P=2; halo one row.  With a
    temporal block tb > 1 one kernel invocation advances tb
    iterations, so it reads a halo of tb rows and the loop runs iters/tb times."""
    assert tb >= 1 and iters % tb == 0
    k = Kernel("hotspot", rows, granule, min_items,
               [Access(0, READ, cols, tb), Access(2, READ, cols, 0), Access(1, WRITE, cols, 0)])
    app = App(buffers=[(4, rows * cols)] * 3, kernels=[k], swaps=[(0, 1)])
    if iters // tb > 1:
        app.loop = (0, 0, iters // tb)
    return app


def stencil_reduction(rows: int, cols: int, steps: int, sync: int = SYNC_BARRIER,
                      granule: int = 1) -> App:
    """MK-Loop app of BASELINE configs[3]: kernel A = HotSpot update, kernel B =
    per-row residual (T_out - T_in)^2 in FP64 into rowsum (slot 3, 8 B/row)."""
    a = Kernel("stencil", rows, granule, 1,
               [Access(0, READ, cols, 1), Access(2, READ, cols, 0), Access(1, WRITE, cols, 0)])
    b = Kernel("residual", rows, granule, 1,
               [Access(0, READ, cols, 0), Access(1, READ, cols, 0), Access(3, WRITE, 1, 0)])
    app = App(buffers=[(4, rows * cols)] * 3 + [(8, rows)], kernels=[a, b], swaps=[(0, 1)],
              loop=(0, 1, steps))
    if sync != SYNC_NONE:
        app.sync = {1: sync}
    return app


def single(name: str, n: int, granule: int = 32, min_items: int = 1, iters: int = 1) -> App:
    """A generic single data-parallel kernel (MatrixMul rows, BlackScholes
    options): reads slot 0 (elems_per_item e), writes slot 1."""
    k = Kernel(name, n, granule, min_items, [Access(0, READ), Access(1, WRITE)])
    app = App(buffers=[(4, n), (4, n)], kernels=[k])
    if iters > 1:
        app.loop = (0, 0, iters)
    return app


def cholesky_tasks(T: int, b: int) -> App:
    """Right-looking tiled Cholesky (BASELINE configs[4]) as an explicit task
    DAG over a tile-major matrix (tile (i,j) = elements [(i T + j) b^2, +b^2)).
    Kernels: 0 POTRF, 1 TRSM, 2 SYRK, 3 GEMM.  Creation order is the loop nest
    with the next panel's updates first (lookahead, R34): k: POTRF(k);
    i>k: TRSM(i,k); SYRK(k+1,k); i>k+1: GEMM(i,k+1,k); i>k+1: SYRK(i,k);
    j>k+1, i>j: GEMM(i,j,k)."""
    bb = b * b

    def tile(i, j):
        return (i * T + j) * bb

    def acc(mode, i, j):
        lo = tile(i, j)
        return TaskAccess(0, mode, lo, lo + bb, lo, lo + bb)

    tasks = []
    for k in range(T):
        tasks.append(Task(0, k, tile(k, k), tile(k, k) + 1, [acc(RW, k, k)], ij=(k, k)))
        for i in range(k + 1, T):
            tasks.append(Task(1, k, tile(i, k), tile(i, k) + 1, [acc(READ, k, k), acc(RW, i, k)],
                              ij=(i, k)))
        def syrk(i):
            return Task(2, k, tile(i, i), tile(i, i) + 1, [acc(READ, i, k), acc(RW, i, i)],
                        ij=(i, i), lane=1 if i == k + 1 else 0)   # SYRK(k+1,k): lane 1

        def gemm(i, j):
            return Task(3, k, tile(i, j), tile(i, j) + 1,
                        [acc(READ, i, k), acc(READ, j, k), acc(RW, i, j)], ij=(i, j))

        if k + 1 < T:   # lookahead: the updates of column k+1
            tasks.append(syrk(k + 1))
            tasks.extend(gemm(i, k + 1) for i in range(k + 2, T))
        tasks.extend(syrk(i) for i in range(k + 2, T))
        for j in range(k + 2, T):
            tasks.extend(gemm(i, j) for i in range(j + 1, T))
    ks = [Kernel(nm, 1, 1, 1, []) for nm in ("potrf", "trsm", "syrk", "gemm")]
    edges = [(0, 1), (1, 2), (1, 3), (2, 0), (3, 1), (3, 2), (3, 3)]
    # the critical path on compute lane 1 (R31): POTRF, TRSM, and the update of
    # the next diagonal tile SYRK(k+1,k) (task lane 1)
    return App(buffers=[(4, T * T * bb)], kernels=ks, edges=edges, dag_tasks=tasks, lanes={0: 1, 1: 1})


def nbody(n: int, iters: int, granule: int = 256, min_items: int = 1) -> App:
    """Nbody (P223-227, P319): one all-pairs kernel iterated (SK-Loop); slots
    pos_in=0, pos_out=1, vel_in=2, vel_out=3 (float4 bodies = 4 elements per
    item); every body reads all positions (whole-buffer access, R18)."""
    k = Kernel("nbody", n, granule, min_items,
               [Access(0, READ, 0), Access(2, READ, 4), Access(1, WRITE, 4), Access(3, WRITE, 4)])
    app = App(buffers=[(4, 4 * n)] * 4, kernels=[k], swaps=[(0, 1), (2, 3)])
    if iters > 1:
        app.loop = (0, 0, iters)
    return app
