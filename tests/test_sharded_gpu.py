"""ss_select_sharded on one GPU against the CPU oracle.

* Virtual ranks: P = 2, 4, 8 host threads, each with its own context and
  stream on cuda:0, bound to one in-process group (ss_comm_init_local) --
  the same device-side level loop, kernels and exchange pattern as over NCCL
  (NCCL refuses two ranks on one device).  Every rank must return the
  oracle's element of the union, for iid, non-iid, empty, duplicate-heavy and
  integer shards, at sizes that run several sharded levels, misses and the
  gather.
* NCCL at world size 1: the real communicator (ss_nccl_unique_id +
  ss_comm_init) through the same call, equal to ss_select.
"""
import threading

import numpy as np
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu


def _bits(v):
    v = np.asarray(v)
    u = np.uint32 if v.dtype.itemsize == 4 else np.uint64
    return int(v.reshape(1).view(u)[0])


def _run(shards, ks, P, **cfg):
    import torch
    import paper_conf_ipps_ribizela19_b200 as ss
    group = ss.LocalGroup(P)
    out = [None] * P
    stats = [None] * P
    errs = []

    def worker(r):
        try:
            torch.cuda.set_device(0)
            st = torch.cuda.Stream()
            with torch.cuda.stream(st):
                ctx = ss.Context(0, **cfg)
                ctx.comm_init_local(group, r)
                x = torch.from_numpy(np.ascontiguousarray(shards[r])).to("cuda:0")
                res, sts = [], []
                for k in ks:
                    res.append(_bits(ctx.select_sharded(x, k)))
                    sts.append(ctx.stats())
                out[r], stats[r] = res, sts
                torch.cuda.synchronize()
                ctx.close()
        except Exception as e:  # pragma: no cover
            errs.append(repr(e))

    ts = [threading.Thread(target=worker, args=(r,)) for r in range(P)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(timeout=600)
    group.close()
    assert not errs, errs
    return out, stats


def _shards(case, P, n, dtype, seed):
    if case == "iid":
        return [datagen.make("uniform" if np.dtype(dtype).kind == "f" else "int", n, dtype, seed + r)
                for r in range(P)]
    if case == "noniid":       # rank r holds [r, r + 1): the sample must follow the shard sizes
        return [datagen.uniform(n // (r + 1), dtype, seed + r) + dtype(r) for r in range(P)]
    if case == "empty":        # odd ranks hold nothing
        return [datagen.normal(n, dtype, seed + r) if r % 2 == 0 else np.zeros(0, dtype) for r in range(P)]
    if case == "distinct16":
        return [datagen.distinct(n, 16, dtype, seed + r) for r in range(P)]
    if case == "equal":
        return [datagen.all_equal(n, 42, dtype) for _ in range(P)]
    if case == "specials":
        return [datagen.specials(n, dtype, seed + r) for r in range(P)]
    raise ValueError(case)


@pytest.mark.parametrize("P", [2, 4, 8])
@pytest.mark.parametrize("case", ["iid", "noniid", "empty", "distinct16", "equal"])
def test_virtual_ranks(P, case, cuda_device):
    dtype = np.float32
    n = (1 << 20) // P + 17
    shards = _shards(case, P, n, dtype, seed=100 + P)
    full = np.concatenate(shards)
    N = full.size
    ks = sorted({0, N // 2, N - 1, datagen.rank(N, P)})
    out, stats = _run(shards, ks, P, shard_gather_log2=14)
    for r in range(P):
        assert out[r] == out[0], "every rank returns the same element"
    for i, k in enumerate(ks):
        assert out[0][i] == _bits(oracle.select(full, k)), (case, P, k)
        st = stats[0][i]
        assert st["shard_ranks"] == P
        if case in ("iid", "noniid"):
            assert st["shard_levels"] >= 1 and st["n_level"][0] == N


@pytest.mark.parametrize("dtype", [np.float32, np.float64, np.int32, np.int64])
def test_virtual_ranks_dtypes(dtype, cuda_device):
    P = 4
    n = (1 << 19) + 3
    kind = "specials" if np.dtype(dtype).kind == "f" else "iid"
    shards = _shards(kind, P, n, dtype, seed=7)
    full = np.concatenate(shards)
    N = full.size
    ks = [0, 1, N // 3, N // 2, N - 1]
    out, _ = _run(shards, ks, P, shard_gather_log2=15)
    for i, k in enumerate(ks):
        assert all(out[r][i] == out[0][i] for r in range(P))
        assert out[0][i] == _bits(oracle.select(full, k)), (dtype, k)


def test_virtual_ranks_gather_overflow_adds_levels(cuda_device):
    """A gather buffer far below the planned survivors forces the host to
    add sharded levels after the hand-off (dist_halt); still exact."""
    P = 2
    n = 1 << 20
    shards = _shards("iid", P, n, np.float32, seed=3)
    full = np.concatenate(shards)
    ks = [full.size // 2, 12345]
    out, stats = _run(shards, ks, P, shard_gather_log2=12, spec_z=1.0)
    for i, k in enumerate(ks):
        assert out[0][i] == out[1][i] == _bits(oracle.select(full, k))


def test_virtual_ranks_poisoned_sample_miss(cuda_device):
    """Rank 0's share of the level-0 sample lands on its smallest values, so
    the window misses k: the directed level must recover (exact answer)."""
    P = 2
    n = 1 << 20
    shards = _shards("iid", P, n, np.float32, seed=5)
    seed = 0x5A17
    # rank 0 draws slots [0, s/2) of level 0 from its own shard (R7)
    idx = oracle.sample_indices(seed, 0, n, 0, 2048)
    shards[0][idx] = -1000.0 - np.arange(idx.size, dtype=np.float32)
    full = np.concatenate(shards)
    ks = [full.size // 2, full.size - 5]
    out, stats = _run(shards, ks, P)
    for i, k in enumerate(ks):
        assert out[0][i] == out[1][i] == _bits(oracle.select(full, k)), k


def test_nccl_world1(cuda_device):
    """The real NCCL communicator at world size 1 (one GPU in this harness)."""
    import torch
    import paper_conf_ipps_ribizela19_b200 as ss
    ctx = ss.Context(0)
    ctx.comm_init(ss.nccl_unique_id(), 1, 0)
    for dtype, n in [(np.float32, (1 << 22) + 5), (np.float64, 300001), (np.int32, 1 << 16)]:
        kind = "uniform" if np.dtype(dtype).kind == "f" else "int"
        x = datagen.make(kind, n, dtype, seed=9)
        xd = torch.from_numpy(x).to("cuda:0")
        for k in (0, n // 2, n - 1, datagen.rank(n, 1)):
            v = ctx.select_sharded(xd, k)
            assert _bits(v) == _bits(oracle.select(x, k)) == _bits(ctx.select(xd, k)), (dtype, k)
    with pytest.raises(ss.SSError):
        ctx.select_sharded(xd, n)                   # k outside the union
    ctx.close()


def test_sharded_without_comm_fails(cuda_device):
    import torch
    import paper_conf_ipps_ribizela19_b200 as ss
    ctx = ss.Context(0)
    with pytest.raises(ss.SSError):
        ctx.select_sharded(torch.zeros(10, device="cuda:0"), 3)
    ctx.close()


def test_convenience_calls(cuda_device):
    """ss_select_f32/_f64/_i32/_i64 and ss_approx_select_f32 (north_star's
    select(data, n, k)) on the thread's default context."""
    import ctypes
    import torch
    from paper_conf_ipps_ribizela19_b200 import _abi
    L = _abi.lib()
    n = 100003
    for name, dtype in [("ss_select_f32", np.float32), ("ss_select_f64", np.float64),
                        ("ss_select_i32", np.int32), ("ss_select_i64", np.int64)]:
        kind = "normal" if np.dtype(dtype).kind == "f" else "int"
        x = datagen.make(kind, n, dtype, seed=2)
        xd = torch.from_numpy(x).to("cuda:0")
        out = np.empty(1, dtype)
        for k in (0, n // 2, n - 1):
            rc = getattr(L, name)(ctypes.c_void_p(xd.data_ptr()), n, k, ctypes.c_void_p(out.ctypes.data))
            assert rc == 0 and _bits(out[0]) == _bits(oracle.select(x, k))
    x = datagen.uniform(n, np.float32, seed=4)
    xd = torch.from_numpy(x).to("cuda:0")
    out = np.empty(1, np.float32)
    rank = ctypes.c_int64()
    assert L.ss_approx_select_f32(ctypes.c_void_p(xd.data_ptr()), n, n // 2, 256,
                                  ctypes.c_void_p(out.ctypes.data), ctypes.byref(rank)) == 0
    assert rank.value == oracle.count_less(x, out[0])
