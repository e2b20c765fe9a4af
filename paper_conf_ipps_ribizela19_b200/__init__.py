"""B200-native SampleSelect (Ribizel & Anzt, "Approximate and Exact Selection
on GPUs", IPDPS-W 2019).

Thin Python binding over the C ABI in ``include/sampleselect.h`` (argument
marshalling only; every step runs in the sm_100a kernels of
``libsampleselect.so``; there is no CPU fallback).

    import torch, paper_conf_ipps_ribizela19_b200 as ss
    x = torch.rand(1 << 24, device="cuda")
    v = ss.select(x, k)                  # element of rank k (§II)
    v, r = ss.approx_select(x, k, 1024)  # approximate value + exact rank (§II.C)

Inputs: 1-D contiguous torch tensors on a CUDA device (float32/float64/
int32/int64), or numpy arrays in host memory (copied to the device inside the
call -- the end-to-end path).  Results are numpy scalars with the exact bits.
"""
from __future__ import annotations

import ctypes
import threading

import numpy as np

from . import _abi
from ._abi import SSConfig, SSError, SSStats

__all__ = ["Context", "LocalGroup", "select", "approx_select", "default_context", "nccl_unique_id", "SSError"]

_NP_DT = {np.dtype(np.float32): _abi.SS_FLOAT32, np.dtype(np.float64): _abi.SS_FLOAT64,
          np.dtype(np.int32): _abi.SS_INT32, np.dtype(np.int64): _abi.SS_INT64}
_NP_OF = {v: k for k, v in _NP_DT.items()}


_TORCH_DT = None


def _torch_dt(t):
    global _TORCH_DT
    if _TORCH_DT is None:
        import torch
        _TORCH_DT = {torch.float32: _abi.SS_FLOAT32, torch.float64: _abi.SS_FLOAT64,
                     torch.int32: _abi.SS_INT32, torch.int64: _abi.SS_INT64}
    code = _TORCH_DT.get(t.dtype)
    if code is None:
        raise TypeError(f"unsupported dtype {t.dtype}; use float32/float64/int32/int64")
    return code


def _current_stream(device: int) -> int:
    """The raw cudaStream_t torch considers current on `device`."""
    import torch
    raw = getattr(torch._C, "_cuda_getCurrentRawStream", None)
    if raw is not None:
        return raw(device)
    return torch.cuda.current_stream(device).cuda_stream


def _is_tensor(x) -> bool:
    try:
        import torch
        return isinstance(x, torch.Tensor)
    except ImportError:  # pragma: no cover
        return False


class Context:
    """One ss_context: a device, its workspace and its tuning knobs."""

    def __init__(self, device: int = 0, **config):
        self._lib = _abi.lib()
        self._h = ctypes.c_void_p()
        rc = self._lib.ss_create(int(device), ctypes.byref(self._h))
        if rc:
            raise SSError(rc, f"ss_create(device={device}) failed (is a CUDA device visible?)")
        self.device = int(device)
        self._out = {code: np.empty(1, dtype=npdt) for npdt, code in _NP_DT.items()}
        if config:
            self.configure(**config)

    # ---------------------------------------------------------- plumbing --
    def close(self):
        if self._h:
            self._lib.ss_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):  # pragma: no cover
        try:
            self.close()
        except Exception:
            pass

    def _check(self, rc: int):
        if rc:
            raise SSError(rc, self._lib.ss_last_error(self._h).decode())

    def _stream(self, stream):
        if stream is not None:
            return stream if isinstance(stream, int) else stream.cuda_stream
        return _current_stream(self.device)

    @property
    def config(self) -> dict:
        c = SSConfig()
        self._check(self._lib.ss_get_config(self._h, ctypes.byref(c)))
        return {f: getattr(c, f) for f, _ in SSConfig._fields_}

    def configure(self, **kw):
        c = SSConfig(**{**self.config, **kw})
        self._check(self._lib.ss_set_config(self._h, ctypes.byref(c)))

    def stats(self) -> dict:
        s = SSStats()
        self._check(self._lib.ss_last_stats(self._h, ctypes.byref(s)))
        L = s.levels
        return {"levels": L, "equality_exit": bool(s.equality_exit),
                "n_level": list(s.n_level[:L + 1]), "bucket": list(s.bucket[:L]),
                "bytes_algorithmic": s.bytes_algorithmic, "launches": s.launches,
                "h2d_bytes": s.h2d_bytes, "d2h_bytes": s.d2h_bytes,
                "ms_kernel": [list(s.ms_kernel[l]) for l in range(L + 1)],
                "tl_us": [[list(s.tl_us[l][q]) for q in range(3)] for l in range(L + 1)],
                "spec_levels": s.spec_levels, "fused_levels": s.fused_levels,
                "lut_ctas": s.lut_ctas, "upper_greater": s.upper_greater,
                "ms_upper_gather": s.ms_upper_gather, "ms_quick": s.ms_quick,
                "incomplete_rounds": s.incomplete_rounds, "shard_levels": s.shard_levels,
                "shard_ranks": s.shard_ranks, "workspace_bytes": s.workspace_bytes,
                "upper_onepass": s.upper_onepass}

    def raw_tl(self):
        """profile=3: the full 32x3 timeline (us after init; -1 = not stamped)."""
        s = SSStats()
        self._check(self._lib.ss_last_stats(self._h, ctypes.byref(s)))
        return [[list(s.tl_us[l][q]) for q in range(3)] for l in range(_abi.SS_MAX_LEVELS)]

    def profile_totals(self, reset: bool = False) -> dict:
        """Per-(level, kernel) device ms summed over calls made with
        profile=1, launch and call counts since the last reset."""
        L = _abi.SS_MAX_LEVELS
        ms = (ctypes.c_double * (3 * L))()
        cnt = (ctypes.c_int64 * (3 * L))()
        launches, calls = ctypes.c_int64(), ctypes.c_int64()
        self._check(self._lib.ss_profile_totals(self._h, ms, cnt, ctypes.byref(launches),
                                                ctypes.byref(calls), int(reset)))
        return {"ms_sum": [[ms[l * 3 + q] for q in range(3)] for l in range(L)],
                "count": [[cnt[l * 3 + q] for q in range(3)] for l in range(L)],
                "launches": launches.value, "calls": calls.value}

    def _args(self, x):
        """-> (dtype code, pointer, n, numpy dtype, on_device)"""
        if _is_tensor(x):
            if not x.is_cuda:
                raise ValueError("torch tensor must live on a CUDA device (use numpy for host data)")
            if x.dim() != 1 or not x.is_contiguous():
                raise ValueError("input must be a 1-D contiguous tensor")
            if x.device.index != self.device:
                raise ValueError(f"tensor on cuda:{x.device.index}, context on cuda:{self.device}")
            dt = _torch_dt(x)
            return dt, x.data_ptr(), x.numel(), _NP_OF[dt], True
        a = np.asarray(x)
        if a.ndim != 1 or not a.flags.c_contiguous:
            raise ValueError("input must be a 1-D contiguous array")
        if a.dtype not in _NP_DT:
            raise TypeError(f"unsupported dtype {a.dtype}")
        return _NP_DT[a.dtype], ctypes.c_void_p(a.ctypes.data), a.size, a.dtype, False

    # ------------------------------------------------------------- API ----
    def select(self, x, k: int, stream=None):
        """Element of rank k (0-based; ties take the smallest rank, §II)."""
        dt, p, n, npdt, dev = self._args(x)
        out = self._out[dt]                     # (a per-context result slot: the call is synchronous)
        fn = self._lib.ss_select if dev else self._lib.ss_select_host
        rc = fn(self._h, dt, p, n, int(k), out.ctypes.data, self._stream(stream))
        if rc:
            self._check(rc)
        return out[0]

    def approx_select(self, x, k: int, b: int = 1024, stream=None):
        """Approximate element of rank ~k with b buckets and its exact rank
        #{x < value} (§II.C)."""
        dt, p, n, npdt, dev = self._args(x)
        out = np.empty(1, dtype=npdt)
        rank = ctypes.c_int64(0)
        fn = self._lib.ss_approx_select if dev else self._lib.ss_approx_select_host
        self._check(fn(self._h, dt, p, n, int(k), int(b), ctypes.c_void_p(out.ctypes.data),
                       ctypes.byref(rank), self._stream(stream)))
        return out[0], int(rank.value)

    def select_upper(self, x, k: int, out=None, stream=None):
        """Top-k fusion (§IV.I): the element of rank k and the n-k
        elements of ranks k..n-1 (a multiset, order unspecified).  x must be a
        CUDA tensor; returns (value, out) with out a tensor of n-k elements."""
        if not _is_tensor(x):
            raise TypeError("select_upper takes a CUDA tensor (the output is a device buffer)")
        dt, p, n, npdt, dev = self._args(x)
        if out is None:
            import torch
            out = torch.empty(max(n - int(k), 0), dtype=x.dtype, device=x.device)
        elif out.dtype != x.dtype or out.device != x.device or not out.is_contiguous() or \
                out.numel() < n - int(k):
            raise ValueError("out must be a contiguous tensor of x's dtype/device with >= n-k elements")
        val = np.empty(1, dtype=npdt)
        self._check(self._lib.ss_select_upper(self._h, dt, p, n, int(k), ctypes.c_void_p(out.data_ptr()),
                                              ctypes.c_void_p(val.ctypes.data), self._stream(stream)))
        return val[0], out

    def quickselect(self, x, k: int, stream=None, with_levels: bool = False):
        """QuickSelect baseline: the same
        element as select(x, k), by one pivot per level.  x must be a CUDA
        tensor.  with_levels=True also returns the list of n_l per level."""
        if not _is_tensor(x):
            raise TypeError("quickselect takes a CUDA tensor")
        dt, p, n, npdt, _ = self._args(x)
        val = np.empty(1, dtype=npdt)
        cap = 128
        nl = (ctypes.c_int64 * cap)()
        lv = ctypes.c_int32(0)
        self._check(self._lib.ss_quickselect(self._h, dt, p, n, int(k), ctypes.c_void_p(val.ctypes.data),
                                             nl, cap, ctypes.byref(lv), self._stream(stream)))
        if with_levels:
            return val[0], [int(nl[i]) for i in range(lv.value + 1)]
        return val[0]

    def select_multi(self, x, ks, stream=None):
        """Multi-rank selection: the elements of ranks ks
        (0-based) of the CUDA tensor x, as a numpy array; one shared count pass."""
        if not _is_tensor(x):
            raise TypeError("select_multi takes a CUDA tensor")
        dt, p, n, npdt, _ = self._args(x)
        ka = np.ascontiguousarray(np.asarray(ks, dtype=np.int64).reshape(-1))
        out = np.empty(ka.size, dtype=npdt)
        self._check(self._lib.ss_select_multi(self._h, dt, p, n, int(ka.size),
                                              ka.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                              ctypes.c_void_p(out.ctypes.data), self._stream(stream)))
        return out

    # ------------------------------------------------ sharded (§8e) -------
    def comm_init(self, unique_id: bytes, nranks: int, rank: int):
        """Bind a NCCL communicator (collective over all ranks; unique_id from
        nccl_unique_id() on one rank, broadcast by the caller)."""
        if len(unique_id) != 128:
            raise ValueError("unique_id must be 128 bytes")
        self._check(self._lib.ss_comm_init(self._h, ctypes.c_char_p(bytes(unique_id)), int(nranks), int(rank)))

    def comm_init_local(self, group: "LocalGroup", rank: int):
        """Bind rank `rank` of an in-process group (virtual ranks, one host
        thread per rank)."""
        self._check(self._lib.ss_comm_init_local(self._h, group._h, int(rank)))

    def select_sharded(self, x, k: int, stream=None):
        """Element of rank k (0-based) of the union of every rank's shard x
        (a 1-D CUDA tensor, may be empty); collective: every rank calls it
        with the same k and gets the same result."""
        if not _is_tensor(x):
            raise TypeError("select_sharded takes a CUDA tensor")
        if x.numel() == 0:
            if not x.is_cuda or x.dim() != 1:
                raise ValueError("input must be a 1-D CUDA tensor")
            dt, p, n, npdt = _torch_dt(x), ctypes.c_void_p(0), 0, _NP_OF[_torch_dt(x)]
        else:
            dt, p, n, npdt, _ = self._args(x)
        out = np.empty(1, dtype=npdt)
        self._check(self._lib.ss_select_sharded(self._h, dt, p, n, int(k), ctypes.c_void_p(out.ctypes.data),
                                                self._stream(stream)))
        return out[0]

    # -------------------------------------------- single steps (tensors) --
    def step_sample(self, x, level: int, slot_begin: int, count: int, out_keys, stream=None):
        dt, p, n, _, _ = self._args(x)
        self._check(self._lib.ss_step_sample(self._h, dt, p, n, int(level), int(slot_begin), int(count),
                                             ctypes.c_void_p(out_keys.data_ptr()), self._stream(stream)))

    def step_tree(self, dt_code: int, sample_keys, b: int, fixup: bool, tree, splitters, eq, stream=None):
        self._check(self._lib.ss_step_tree(self._h, dt_code, ctypes.c_void_p(sample_keys.data_ptr()),
                                           sample_keys.numel(), int(b), int(bool(fixup)),
                                           ctypes.c_void_p(tree.data_ptr()),
                                           ctypes.c_void_p(splitters.data_ptr()),
                                           ctypes.c_void_p(eq.data_ptr()), self._stream(stream)))

    def step_count(self, x, tree, b: int, totals, oracles=None, stream=None):
        dt, p, n, _, _ = self._args(x)
        self._check(self._lib.ss_step_count(self._h, dt, p, n, ctypes.c_void_p(tree.data_ptr()), int(b),
                                            ctypes.c_void_p(totals.data_ptr()),
                                            ctypes.c_void_p(oracles.data_ptr() if oracles is not None else 0),
                                            self._stream(stream)))

    def step_count_ablation(self, x, tree, b: int, mode, totals, stream=None):
        """Atomics ablation: bucket totals from the plain
        Fig. 4 count kernel with the increment strategy `mode` (a name from
        _abi.ABLATION_MODES or its code)."""
        dt, p, n, _, _ = self._args(x)
        m = _abi.ABLATION_MODES[mode] if isinstance(mode, str) else int(mode)
        self._check(self._lib.ss_step_count_ablation(self._h, dt, p, n, ctypes.c_void_p(tree.data_ptr()), int(b), m,
                                                     ctypes.c_void_p(totals.data_ptr()), self._stream(stream)))

    def step_filter(self, x, oracles, bucket: int, out, count, stream=None):
        dt, p, n, _, _ = self._args(x)
        self._check(self._lib.ss_step_filter(self._h, dt, p, n, ctypes.c_void_p(oracles.data_ptr()),
                                             int(bucket), ctypes.c_void_p(out.data_ptr()),
                                             ctypes.c_void_p(count.data_ptr()), self._stream(stream)))

    def step_search(self, totals, b: int, k: int, eq, out, stream=None):
        self._check(self._lib.ss_step_search(self._h, ctypes.c_void_p(totals.data_ptr()), int(b), int(k),
                                             ctypes.c_void_p(eq.data_ptr() if eq is not None else 0),
                                             ctypes.c_void_p(out.data_ptr()), self._stream(stream)))

    def oracle_offset(self, x) -> int:
        """Offset of element 0's oracle byte in an oracle buffer for x
        (ss_oracle_offset: byte i lives at offset + i)."""
        dt, p, n, _, _ = self._args(x)
        return int(self._lib.ss_oracle_offset(dt, p, n))

    def step_keys_to_values(self, dt_code: int, keys, values, stream=None):
        self._check(self._lib.ss_step_keys_to_values(self._h, dt_code, ctypes.c_void_p(keys.data_ptr()),
                                                     keys.numel(), ctypes.c_void_p(values.data_ptr()),
                                                     self._stream(stream)))


class LocalGroup:
    """An in-process rank group (ss_local_group): contexts in different host
    threads exchange through device memory -- virtual ranks on one GPU."""

    def __init__(self, nranks: int):
        self._lib = _abi.lib()
        self._h = ctypes.c_void_p()
        rc = self._lib.ss_local_group_create(int(nranks), ctypes.byref(self._h))
        if rc:
            raise SSError(rc, f"ss_local_group_create({nranks})")
        self.nranks = int(nranks)

    def close(self):
        if self._h:
            self._lib.ss_local_group_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):  # pragma: no cover
        try:
            self.close()
        except Exception:
            pass


def nccl_unique_id() -> bytes:
    """A NCCL unique id (128 bytes) for Context.comm_init."""
    buf = ctypes.create_string_buffer(128)
    lib = _abi.lib()
    rc = lib.ss_nccl_unique_id(buf)
    if rc:
        raise SSError(rc, "ss_nccl_unique_id: NCCL unavailable")
    return buf.raw


_tls = threading.local()


def default_context(device: int | None = None) -> Context:
    """Thread-local context per device (mirrors north_star's select(data, n, k))."""
    if device is None:
        import torch
        device = torch.cuda.current_device()
    cache = getattr(_tls, "ctx", None)
    if cache is None:
        cache = _tls.ctx = {}
    if device not in cache:
        cache[device] = Context(device)
    return cache[device]


def _device_of(x):
    if _is_tensor(x) and x.is_cuda:
        return x.device.index
    return None


def select(x, k: int):
    """Element of rank k of x (exact; bit-identical to sort-and-index)."""
    return default_context(_device_of(x)).select(x, k)


def approx_select(x, k: int, b: int = 1024):
    """(approximate value, its exact rank) with b buckets, one level."""
    return default_context(_device_of(x)).approx_select(x, k, b)


def select_upper(x, k: int, out=None):
    """(element of rank k, tensor of the n-k elements of rank >= k) -- top-k, §IV.I."""
    return default_context(_device_of(x)).select_upper(x, k, out)


def select_multi(x, ks):
    """Elements of ranks ks of x (one shared sample + count pass)."""
    return default_context(_device_of(x)).select_multi(x, ks)
