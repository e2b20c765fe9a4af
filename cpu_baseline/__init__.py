"""CPU baselines timed by bench.py (not the product, not the test oracle):
std::nth_element on one core (the paper's reference check)
and __gnu_parallel::nth_element on all host cores (BASELINE.md CPU plan)."""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "nth.cpp")
_LIB = os.path.join(_HERE, "libcpu_nth.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O3", "-march=native", "-fopenmp", "-D_GLIBCXX_PARALLEL_NO_WARN",
                               "-fPIC", "-shared", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        lib.cpu_nth_element.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64,
                                        ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
        lib.cpu_nth_element.restype = ctypes.c_double
        lib.cpu_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def threads() -> int:
    return int(_load().cpu_threads())


def nth_element(x: np.ndarray, k: int, parallel: bool, reps: int = 1):
    """(best seconds over reps, element k) of (parallel) nth_element on a copy of x."""
    x = np.ascontiguousarray(x)
    if x.dtype not in (np.float32, np.float64):
        raise TypeError("float32 / float64 only")
    out = np.empty(1, x.dtype)
    t = _load().cpu_nth_element(0 if x.dtype == np.float32 else 1, x.ctypes.data, x.size, int(k),
                                int(bool(parallel)), int(reps), out.ctypes.data)
    return t, out[0]
