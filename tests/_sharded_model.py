"""CPU model of the sharded selection protocol (test infrastructure only).

The product runs this protocol on the GPU (ss_select_sharded: csrc/sharded.cuh,
csrc/dist_kernels.cuh).  This model replays the same host-visible protocol --
the same exchanges in the same order, the same proportional sample slots
(dist_slot_range), the same window rule (reading R21), the same hit / equality
exit / directed-miss decision, the gather once the level is small -- over real
multi-process collectives (gloo), with plain numpy per-rank steps and the CPU
oracle for the final selection.  It checks the protocol itself (every rank
takes the same decisions; non-iid, empty and duplicate shards give the exact
answer); the GPU parity of the product is tests/test_sharded_gpu.py.

Values are compared with numpy's `<`, so the model's inputs avoid NaNs and
signed zeros (the product orders those by totalOrder, reading R3).
"""
from __future__ import annotations

import math
from typing import List

import numpy as np

import oracle


def slot_range(sizes: List[int], rank: int, s: int):
    """Sample slots of `rank`: [floor(s P_r / N), floor(s P_{r+1} / N))."""
    N = sum(sizes)
    if N == 0:
        return 0, 0
    lo = sum(sizes[:rank])
    return (s * lo) // N, (s * (lo + sizes[rank])) // N


class TorchDistExchange:
    """The one collective of the protocol: a sum-allreduce of an int64 buffer
    in which every rank fills disjoint slots (torch.distributed, gloo)."""

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist, self.group = dist, group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)

    def allreduce(self, a: np.ndarray) -> np.ndarray:
        import torch
        t = torch.from_numpy(np.ascontiguousarray(a.astype(np.int64)))
        self.dist.all_reduce(t, op=self.dist.ReduceOp.SUM, group=self.group)
        return t.numpy()


class ShardedModel:
    def __init__(self, comm, s: int = 256, z: float = 3.0, gather: int = 1 << 10, seed: int = 0x5A17):
        self.comm, self.s, self.z, self.G, self.seed = comm, s, z, gather, seed
        self.levels: List[int] = []     # global level sizes of the sharded levels
        self.hits: List[int] = []       # 1 hit, 0 miss, per sharded level

    def _window(self, sorted_sample, N, k):
        """Reading R21 (spec_window): the window of sample ranks s p -/+ (z sigma + 2)."""
        s = sorted_sample.size
        p = k / N
        mu = p * s
        half = self.z * math.sqrt(s * p * (1 - p)) + 2.0
        qlo, qhi = math.floor(mu - half), math.ceil(mu + half)
        lo_inf, hi_inf = qlo <= 0, qhi >= s - 1
        vlo = sorted_sample[0 if lo_inf else qlo]
        vhi = sorted_sample[s - 1 if hi_inf else qhi]
        if vlo == vhi:
            return ("eq", vlo, None)
        return ("range", None if lo_inf else vlo, None if hi_inf else vhi)

    def select(self, x: np.ndarray, k: int):
        comm, P, r = self.comm, self.comm.world, self.comm.rank
        # exchange 0: the sizes
        a = np.zeros(P, np.int64)
        a[r] = x.size
        sizes = [int(v) for v in comm.allreduce(a)]
        N = sum(sizes)
        if not 0 <= k < N:
            raise ValueError("k outside the union")
        cur, lev, directed = x, 0, None
        self.levels, self.hits = [], []
        while N > self.G:
            self.levels.append(N)
            # exchange 1: the sample (each rank fills its proportional slots)
            lo, hi = slot_range(sizes, r, self.s)
            table = np.zeros(self.s, np.int64)
            if hi > lo:
                idx = oracle.sample_indices(self.seed, lev, cur.size, lo, hi - lo)
                table[lo:hi] = _to_bits(cur[idx])
            sample = np.sort(_from_bits(comm.allreduce(table), x.dtype))
            if directed is None:
                kind, klo, khi = self._window(sample, N, k)
            else:
                kind, klo, khi = directed
            # per rank: below, window count, the window's elements
            if kind == "eq":
                inw = cur == klo
                below = int(np.sum(cur < klo))
            else:
                inw = np.ones(cur.size, bool)
                below = 0
                if klo is not None:
                    inw &= cur >= klo
                    below = int(np.sum(cur < klo))
                if khi is not None:
                    inw &= cur < khi
            rows = np.zeros((P, 3), np.int64)
            rows[r] = [below, int(inw.sum()), cur.size]
            rows = comm.allreduce(rows.reshape(-1)).reshape(P, 3)           # exchange 2
            B, W = int(rows[:, 0].sum()), int(rows[:, 1].sum())
            if B <= k < B + W:
                self.hits.append(1)
                if kind == "eq":
                    return klo
                cur = cur[inw]
                k -= B
                directed = None
                sizes = [int(v) for v in rows[:, 1]]
            else:
                self.hits.append(0)
                lo_v = klo
                hi_v = klo if kind == "eq" else khi
                if k < B:
                    directed = ("range", None, lo_v)
                else:
                    directed = ("range", _succ(hi_v) if kind == "eq" else hi_v, None)
                sizes = [int(v) for v in rows[:, 2]]
            N = sum(sizes)
            lev += 1
        # exchange 3: gather into one buffer (rank r at offset sum of sizes < r)
        off = sum(sizes[:r])
        buf = np.zeros(N, np.int64)
        buf[off:off + cur.size] = _to_bits(cur)
        allx = _from_bits(comm.allreduce(buf), x.dtype)
        return oracle.select(allx, k)


def _to_bits(v: np.ndarray) -> np.ndarray:
    """Raw bits as int64 (the exchange sums integers, as the product does)."""
    v = np.ascontiguousarray(v)
    if v.dtype.itemsize == 4:
        return v.view(np.int32).astype(np.int64)
    return v.view(np.int64).copy()


def _from_bits(a: np.ndarray, dtype) -> np.ndarray:
    dtype = np.dtype(dtype)
    if dtype.itemsize == 4:
        return a.astype(np.int32).view(dtype)
    return a.astype(np.int64).view(dtype)


def _succ(v):
    """The next value up (the key successor of reading R9)."""
    if np.issubdtype(np.asarray(v).dtype, np.integer):
        return v + 1
    return np.nextafter(v, np.inf)
