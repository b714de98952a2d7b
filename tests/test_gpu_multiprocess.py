"""Multi-process execution (world > 1, one logical device per process) on the
IPC transport, bit-exact against the oracle.  Two or three ranks share the one
GPU of this run: every exchange the op program holds — SP-Varied re-sync
(P119), HotSpot ghost rows (P391 -> P319), w-sync flushes, DP chunk inputs
and Cholesky panels — is a pull out of the peer process's buffer through its
CUDA IPC mapping, ordered by device-memory completion flags.  On an 8-GPU
node the same code pulls over NVLink."""
import os
import subprocess
import sys

import numpy as np
import pytest

import synthgen
from oracle import numeric as on

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
WORKER = os.path.join(ROOT, "tests", "ipc_worker.py")


def run_ranks(case, world, tmp_path, graph=False, runs=1):
    idhex = os.urandom(128).hex()
    outs = [str(tmp_path / f"{case}_{r}.npz") for r in range(world)]
    procs = [subprocess.Popen([sys.executable, WORKER, str(r), str(world), idhex, case, outs[r],
                               "graph" if graph else "eager", str(runs)],
                              cwd=ROOT, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)
             for r in range(world)]
    logs = []
    for p in procs:
        try:
            logs.append(p.communicate(timeout=300)[0])
        except subprocess.TimeoutExpired:
            for q in procs:
                q.kill()
            raise
    for p, lg in zip(procs, logs):
        assert p.returncode == 0, lg[-3000:]
    return [dict(np.load(o)) for o in outs]


def assemble(res, slot, n, dtype):
    out = np.full(n, np.nan, dtype=dtype)
    seen = np.zeros(n, bool)
    for r in res:
        pos = 0
        for b, e in r[f"r{slot}"]:
            out[b:e] = r[f"v{slot}"][pos:pos + e - b]
            assert not seen[b:e].any()
            seen[b:e] = True
            pos += e - b
    assert seen.all()
    return out


@pytest.mark.parametrize("case,world", [("stream_varied", 2), ("stream_varied", 3), ("stream_varied_flush", 2),
                                        ("stream_dp_perf", 2)])
@pytest.mark.parametrize("graph", [False, True])
def test_stream_multiprocess(tmp_path, case, world, graph):
    n, passes = {"stream_varied": (100003, 2), "stream_varied_flush": (65547, 1), "stream_dp_perf": (100003, 1)}[case]
    a0, b0, c0 = synthgen.stream_random(n)
    ref = on.stream_run(a0, b0, c0, passes)
    res = run_ranks(case, world, tmp_path, graph=graph, runs=2 if graph else 1)
    for slot in range(3):
        got = assemble(res, slot, n, np.float32)
        want = ref[slot] if not graph else on.stream_run(*on.stream_run(a0, b0, c0, passes), passes)[slot]
        assert np.array_equal(got, want), (case, world, slot)
    if case.startswith("stream_varied"):
        assert sum(int(r["xfer"][0]) for r in res) > 0   # the re-sync pulled across processes


@pytest.mark.parametrize("case,world", [("hotspot", 2), ("hotspot", 3), ("hotspot_tb4", 2), ("hotspot_dp_dep", 2),
                                        ("hotspot_split", 3)])
@pytest.mark.parametrize("graph", [False, True])
def test_hotspot_multiprocess(tmp_path, case, world, graph):
    rows, cols, iters, tb = {"hotspot": (257, 256, 7, 1), "hotspot_tb4": (300, 64, 24, 4),
                             "hotspot_dp_dep": (200, 128, 6, 1), "hotspot_split": (300, 64, 24, 4)}[case]
    slot = {"hotspot": 1, "hotspot_tb4": 0, "hotspot_dp_dep": 0, "hotspot_split": 0}[case]
    t0, p = synthgen.hotspot(rows, cols)
    res = run_ranks(case, world, tmp_path, graph=graph, runs=1)
    got = assemble(res, slot, rows * cols, np.float32).reshape(rows, cols)
    assert np.array_equal(got, on.hotspot_run(t0, p, iters)), (case, world)
    assert sum(int(r["xfer"][0]) for r in res) > 0   # ghost rows pulled from the peer


def test_stencil_reduction_multiprocess(tmp_path):
    rows, cols, steps = 200, 96, 5
    t0, p = synthgen.hotspot(rows, cols)
    res = run_ranks("stencil", 2, tmp_path)
    cur = t0.copy()
    nxt = np.empty_like(cur)
    for s in range(steps):
        on.hotspot_rows(cur, p, nxt)
        if s == steps - 1:
            rs = on.row_residual(cur, nxt)
        cur, nxt = nxt, cur
    assert np.array_equal(assemble(res, 1, rows * cols, np.float32).reshape(rows, cols), cur)
    got_rs = assemble(res, 3, rows, np.float64)
    assert np.max(np.abs(got_rs - rs) / np.maximum(np.abs(rs), 1e-300)) <= 1e-12


@pytest.mark.parametrize("case", ["chol", "chol_cyclic"])
@pytest.mark.parametrize("graph", [False, True])
def test_cholesky_multiprocess(tmp_path, case, graph):
    n, b = 1024, 256
    _, L0 = synthgen.cholesky_exact_factor(n)
    res = run_ranks(case, 2, tmp_path, graph=graph, runs=2 if graph else 1)
    got = assemble(res, 0, n * n, np.float32)
    T = n // b
    L = got.reshape(T, T, b, b).transpose(0, 2, 1, 3).reshape(n, n)
    assert np.array_equal(np.tril(L), L0)


def test_profile_multiprocess(tmp_path):
    """mm_profile_run across 3 ranks: per-rank probes, the exchange link as a
    pull out of the next rank's memory through its IPC mapping, rows
    exchanged so every rank returns the same profile (P49)."""
    res = run_ranks("profile", 3, tmp_path)
    for r in res[1:]:
        for key in ("fs", "link", "lat"):
            assert np.array_equal(r[key], res[0][key]), key
    assert (res[0]["fs"] > 0).all() and (res[0]["link"] > 10 ** 10).all() and (res[0]["lat"] > 0).all()


@pytest.mark.parametrize("case", ["stream_staged", "stream_staged_dp"])
@pytest.mark.parametrize("graph", [False, True])
def test_stream_staged_multiprocess(tmp_path, case, graph):
    """Staged mode across 2 ranks (P119's host-resident regime): each rank's
    inputs start in its pinned host memory, and the outputs each rank
    produced end there (FLUSH); DP-Perf with barriers also pulls chunk inputs
    across processes."""
    n = 100003
    a0, b0, c0 = synthgen.stream_random(n)
    ref = on.stream_run(a0, b0, c0, 1)
    res = run_ranks(case, 2, tmp_path, graph=graph)
    for slot in range(3):
        assert np.array_equal(assemble(res, slot, n, np.float32), ref[slot]), (case, slot)
    assert all(int(r["h2d"][0]) > 0 for r in res)
