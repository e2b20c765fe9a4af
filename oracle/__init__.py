"""CPU test oracle for SampleSelect (Ribizel & Anzt, IPDPS-W 2019).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product path (``paper_conf_ipps_ribizela19_b200``) never imports
it, and this package imports nothing from the product.

The arithmetic lives in ``oracle/oracle.c`` (plain C, exact: selection only
compares).  This module compiles it with gcc on first use (or ``build()``) and
marshals numpy arrays through ctypes.  Every function cites the passage of
``/root/reference/PAPER.md`` it follows; see the header of ``oracle.c``.

:func:`quickselect` (the NEXT-3 baseline's method mirror) is pure Python on
top of :func:`select`, :func:`cmp` and :func:`sample_indices`.

Parity status: every function below is pinned in ``tests/test_oracle.py``
except the approximate *value* of :func:`approx_select`, which has no closed
form (it depends on the random sample); it is pinned statistically (mean rank
error ~ 1/(4b), L200-202 error bound) and its *rank* is pinned exactly.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

DTYPES = {np.dtype(np.float32): 0, np.dtype(np.float64): 1,
          np.dtype(np.int32): 2, np.dtype(np.int64): 3}


def build(force: bool = False) -> str:
    """Compile oracle.c into liboracle.so (gcc -O2).  Returns the path."""
    if force or not os.path.exists(_LIB_PATH) or \
            os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-std=gnu11",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            vp, i64, i32, u64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_uint64
            p64 = ctypes.POINTER(ctypes.c_int64)
            lib.oracle_cmp.argtypes = [i32, vp, vp]
            lib.oracle_select.argtypes = [i32, vp, i64, i64, vp]
            lib.oracle_select_bruteforce.argtypes = [i32, vp, i64, i64, vp]
            lib.oracle_count_less.argtypes = [i32, vp, i64, vp]
            lib.oracle_count_less.restype = i64
            lib.oracle_count_leq.argtypes = [i32, vp, i64, vp]
            lib.oracle_count_leq.restype = i64
            lib.oracle_splitmix64.argtypes = [u64]
            lib.oracle_splitmix64.restype = u64
            lib.oracle_sample_indices.argtypes = [u64, i32, i64, i64, i64, p64]
            lib.oracle_pick_splitters.argtypes = [i32, vp, i64, i32, vp]
            lib.oracle_equality_fixup.argtypes = [i32, vp, i32, vp]
            lib.oracle_heap_tree.argtypes = [i32, vp, i32, vp]
            lib.oracle_tree_bucket.argtypes = [i32, vp, i32, vp]
            lib.oracle_count_buckets.argtypes = [i32, vp, i64, vp, i32, p64, vp]
            lib.oracle_filter_bucket.argtypes = [i32, vp, i64, vp, i32, vp]
            lib.oracle_filter_bucket.restype = i64
            lib.oracle_approx_select.argtypes = [i32, vp, i64, i64, i32, i64, u64, vp, p64, p64]
            lib.oracle_select_upper.argtypes = [i32, vp, i64, i64, vp]
            lib.oracle_select_multi.argtypes = [i32, vp, i64, i32, p64, vp]
            lib.oracle_select_upper_bruteforce.argtypes = [i32, vp, i64, i64, vp]
            lib.oracle_select_upper_bruteforce.restype = i64
            lib.oracle_sampleselect.argtypes = [i32, vp, i64, i64, i32, i64, i64, u64, vp, p64, i32]
            _lib = lib
    return _lib


def _arr(x) -> np.ndarray:
    a = np.ascontiguousarray(x)
    if a.dtype not in DTYPES:
        raise TypeError(f"oracle: unsupported dtype {a.dtype}")
    return a


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _scalar(dtype, v) -> np.ndarray:
    return np.array([v], dtype=dtype) if not isinstance(v, np.ndarray) else np.ascontiguousarray(v.reshape(1).astype(dtype, copy=False))


def cmp(a, b, dtype) -> int:
    """totalOrder / numeric comparison (reading R3): -1, 0, 1."""
    dtype = np.dtype(dtype)
    x, y = _scalar(dtype, a), _scalar(dtype, b)
    return _load().oracle_cmp(DTYPES[dtype], _ptr(x), _ptr(y))


def select(data, k: int):
    """§II: element of rank k (0-based) of the sorted sequence.  Returns
    a 0-d numpy array with the exact bits."""
    a = _arr(data)
    out = np.empty(1, dtype=a.dtype)
    rc = _load().oracle_select(DTYPES[a.dtype], _ptr(a), a.size, int(k), _ptr(out))
    if rc:
        raise ValueError(f"oracle_select: invalid argument (n={a.size}, k={k})")
    return out[0]


def select_bruteforce(data, k: int):
    """O(n^2) count definition: unique v with #{x<v} <= k < #{x<=v}."""
    a = _arr(data)
    out = np.empty(1, dtype=a.dtype)
    rc = _load().oracle_select_bruteforce(DTYPES[a.dtype], _ptr(a), a.size, int(k), _ptr(out))
    if rc:
        raise ValueError("oracle_select_bruteforce: invalid argument")
    return out[0]


def select_upper(data, k: int) -> np.ndarray:
    """§IV.I L606-615 (top-k fusion): the kth-smallest element and all larger
    elements = positions k..n-1 of the sorted sequence (ascending)."""
    a = _arr(data)
    if not 0 <= k < a.size:
        raise ValueError(f"oracle_select_upper: invalid argument (n={a.size}, k={k})")
    out = np.empty(a.size - int(k), dtype=a.dtype)
    rc = _load().oracle_select_upper(DTYPES[a.dtype], _ptr(a), a.size, int(k), _ptr(out))
    if rc:
        raise ValueError(f"oracle_select_upper: rc={rc}")
    return out


def select_multi(data, ks) -> np.ndarray:
    """Reading R23: the elements of ranks ks (0-based, §II
    L82-88 per rank) -- one sort, m indexings."""
    a = _arr(data)
    k = np.ascontiguousarray(np.asarray(ks, dtype=np.int64).reshape(-1))
    out = np.empty(k.size, dtype=a.dtype)
    rc = _load().oracle_select_multi(DTYPES[a.dtype], _ptr(a), a.size, int(k.size),
                                     k.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)), _ptr(out))
    if rc:
        raise ValueError(f"oracle_select_multi: invalid argument (n={a.size}, ks={k.tolist()[:8]})")
    return out


def select_upper_bruteforce(data, k: int) -> np.ndarray:
    """O(n^2) count definition of :func:`select_upper` (unordered multiset)."""
    a = _arr(data)
    if not 0 <= k < a.size:
        raise ValueError("oracle_select_upper_bruteforce: invalid argument")
    out = np.empty(a.size - int(k), dtype=a.dtype)
    w = _load().oracle_select_upper_bruteforce(DTYPES[a.dtype], _ptr(a), a.size, int(k), _ptr(out))
    if w != a.size - int(k):
        raise ValueError(f"oracle_select_upper_bruteforce: wrote {w} of {a.size - int(k)}")
    return out


def count_less(data, v) -> int:
    """#{x_i < v}: the (smallest) rank of v (L86-88)."""
    a = _arr(data)
    s = _scalar(a.dtype, v)
    return int(_load().oracle_count_less(DTYPES[a.dtype], _ptr(a), a.size, _ptr(s)))


def count_leq(data, v) -> int:
    a = _arr(data)
    s = _scalar(a.dtype, v)
    return int(_load().oracle_count_leq(DTYPES[a.dtype], _ptr(a), a.size, _ptr(s)))


def splitmix64(x: int) -> int:
    return int(_load().oracle_splitmix64(ctypes.c_uint64(x & (2**64 - 1))))


def sample_indices(seed: int, level: int, n: int, j0: int, cnt: int) -> np.ndarray:
    """Reading R7: indices of sample slots [j0, j0+cnt) at `level`."""
    out = np.empty(cnt, dtype=np.int64)
    _load().oracle_sample_indices(ctypes.c_uint64(seed), level, n, j0, cnt,
                                  out.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)))
    return out


def pick_splitters(sample, b: int) -> np.ndarray:
    """§IV.B-a L254-259 / reading R8: s_i = sorted_sample[floor(i*s/b)], i=1..b-1."""
    a = _arr(sample)
    out = np.empty(b - 1, dtype=a.dtype)
    _load().oracle_pick_splitters(DTYPES[a.dtype], _ptr(a), a.size, b, _ptr(out))
    return out


def equality_fixup(splitters):
    """§IV.C L346-357 / reading R9.  Returns (modified splitters, eq flags[b])."""
    a = _arr(splitters).copy()
    b = a.size + 1
    eq = np.zeros(b, dtype=np.uint8)
    _load().oracle_equality_fixup(DTYPES[a.dtype], _ptr(a), b, _ptr(eq))
    return a, eq


def heap_tree(splitters) -> np.ndarray:
    """§IV.B-b, Fig. 3: heap-ordered implicit search tree."""
    a = _arr(splitters)
    out = np.empty_like(a)
    rc = _load().oracle_heap_tree(DTYPES[a.dtype], _ptr(a), a.size + 1, _ptr(out))
    if rc:
        raise ValueError("heap_tree: b must be a power of two")
    return out


def tree_bucket(tree, x) -> int:
    """Fig. 4 L331-338 walk."""
    t = _arr(tree)
    s = _scalar(t.dtype, x)
    return int(_load().oracle_tree_bucket(DTYPES[t.dtype], _ptr(t), t.size + 1, _ptr(s)))


def count_buckets(data, tree):
    """§II.A bucket sizes and the oracle bytes (Fig. 4 lines 7-8)."""
    a = _arr(data)
    t = _arr(tree).astype(a.dtype, copy=False)
    b = t.size + 1
    counts = np.zeros(b, dtype=np.int64)
    orc = np.zeros(a.size, dtype=np.uint8)
    _load().oracle_count_buckets(DTYPES[a.dtype], _ptr(a), a.size, _ptr(t), b,
                                 counts.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)), _ptr(orc))
    return counts, orc


def filter_bucket(data, oracles, bucket: int) -> np.ndarray:
    """§IV.B-c, stable (reading R15)."""
    a = _arr(data)
    o = np.ascontiguousarray(oracles, dtype=np.uint8)
    out = np.empty_like(a)
    m = _load().oracle_filter_bucket(DTYPES[a.dtype], _ptr(a), a.size, _ptr(o), int(bucket), _ptr(out))
    return out[:m].copy()


def approx_select(data, k: int, b: int, s: int, seed: int):
    """§II.C: returns (value, exact rank #{x<value}, splitter index i)."""
    a = _arr(data)
    out = np.empty(1, dtype=a.dtype)
    rank = ctypes.c_int64(0)
    idx = ctypes.c_int64(0)
    rc = _load().oracle_approx_select(DTYPES[a.dtype], _ptr(a), a.size, int(k), int(b), int(s),
                                      ctypes.c_uint64(seed), _ptr(out), ctypes.byref(rank),
                                      ctypes.byref(idx))
    if rc:
        raise ValueError("oracle_approx_select: invalid argument")
    return out[0], int(rank.value), int(idx.value)


def sampleselect(data, k: int, b: int, s: int, base_case: int, seed: int, max_levels: int = 64):
    """Fig. 1 L95-127 slow mirror of the whole method.  Returns (value, [n_l])."""
    a = _arr(data)
    out = np.empty(1, dtype=a.dtype)
    levels = np.zeros(max_levels, dtype=np.int64)
    lv = _load().oracle_sampleselect(DTYPES[a.dtype], _ptr(a), a.size, int(k), int(b), int(s),
                                     int(base_case), ctypes.c_uint64(seed), _ptr(out),
                                     levels.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                     max_levels)
    if lv < 0:
        raise ValueError("oracle_sampleselect: invalid argument")
    return out[0], levels[:min(lv, max_levels)].tolist()


QS_SAMPLE = 256


def quickselect(data, k: int, base_case: int, seed: int, max_levels: int = 128):
    """QuickSelect, the paper's comparison baseline (§IV.F), in the
    three-way reading R24 of Fig. 5's branchless bipartition (L375-389):
    per level, pivot = the median (sorted position QS_SAMPLE // 2 = 128) of
    the QS_SAMPLE = 256 keys at the R7 sample indices of the level; one pass over the level puts x < p at
    out[l++] and x > p at out[r--] and counts x == p; k < L recurses left,
    L <= k < L + E returns p, else recurses right with k - L - E.  Levels with
    n <= base_case are finished by sort-and-index (Fig. 1 lines 2-5).
    Pure Python loop over the elements: small inputs only.  Returns
    (value, [n_l for every level incl. the last]).  The level order of the
    GPU's partition is nondeterministic (atomics), so only the result and
    n_1 (level 0 draws its sample from the caller's array) are comparable."""
    cur = np.ascontiguousarray(_arr(data))
    dt = cur.dtype
    k = int(k)
    sizes = []
    for level in range(max_levels):
        n = cur.size
        sizes.append(n)
        if n <= base_case:
            return select(cur, k), sizes
        idx = sample_indices(seed, level, n, 0, QS_SAMPLE)
        p = select(cur[idx], QS_SAMPLE // 2)
        out = np.empty_like(cur)
        l, r, eq = 0, n - 1, 0
        for i in range(n):                   # Fig. 5, three-way (R24)
            c = cmp(cur[i], p, dt)
            if c < 0:
                out[l] = cur[i]
                l += 1
            elif c > 0:
                out[r] = cur[i]
                r -= 1
            else:
                eq += 1
        L, G = l, n - 1 - r
        if k < L:
            cur = out[:L].copy()
        elif k < L + eq:
            return _scalar(dt, p)[0], sizes
        else:
            cur = out[n - G:].copy()
            k -= L + eq
    raise RuntimeError("oracle quickselect: level limit")


def sample_size(b: int) -> int:
    """Reading R7: s = clamp(16 b, 4096, 16384) (a tuning knob, L557-561)."""
    return max(4096, min(16 * b, 16384))
