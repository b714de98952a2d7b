"""B200-native matchmaking of applications and partitioning strategies
(Shen, Varbanescu, Martorell, Sips, ICPP'15).

The product is the C-ABI library ``libmm.so`` (include/mm.h): classification,
Table I ranking, Glinda-style split, DP-Perf / DP-Dep schedules, the op-program
executor and the sm_100a kernels.  ``mm`` is its same-name ctypes binding and
``runner.Session`` the torch plumbing (device memory, streams) around it.
Importing ``mm`` loads libmm.so and raises ImportError if it is missing (there
is no fallback); ``build`` compiles it.
"""
import importlib


def __getattr__(name):
    if name in ("mm", "runner", "build"):
        return importlib.import_module(f".{name}", __name__)
    raise AttributeError(name)
