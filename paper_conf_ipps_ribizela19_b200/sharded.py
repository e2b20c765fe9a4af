"""Sharded (multi-GPU) exact SampleSelect.

One process (or, for tests, one thread) per shard.  Every rank owns a
contiguous shard of the input; the global rank k is the same on all ranks.
Per level (Fig. 1 L95-127 distributed over the shards):

  1. sample (C1): global sample slot j of level l is owned by the rank whose
     prefix of shard sizes covers floor(j * N / s) -- each rank draws its
     share, proportional to its shard size, with the counter-based RNG of
     reading R7 (`ss_step_sample`), and the keys are all-gathered in slot
     order, so every rank holds the identical sample;
  2. every rank sorts the identical sample and builds the identical splitter
     tree (`ss_step_tree`, K1b) -- no broadcast needed;
  3. each rank classifies and counts its own shard (`ss_step_count`, K2);
  4. the b bucket totals are all-reduced (C2, uint64 sums);
  5. every rank runs the identical bucket search (`ss_step_search`, K3/K4):
     an equality bucket ends the selection (§IV.C); otherwise
  6. each rank filters its shard (`ss_step_filter`, K5).

When the global survivor count is at most `gather_threshold`, the survivors
are all-gathered (C3) and every rank finishes with the single-GPU path
(`ss_select`); the answer is then identical on every rank (C4 implicit).

The host logic here talks to the collectives through a `Comm` and to the
kernels through a `Steps` object: `TorchDistComm` + `CudaSteps` are the
product (NCCL over NVLink/NVSwitch, sm_100a kernels through the C ABI);
tests substitute gloo, threads on one GPU, or CPU reference steps.
"""
from __future__ import annotations

import threading
from typing import List

import numpy as np

from . import _abi


# ------------------------------------------------------------------ comms --
class Comm:
    world: int
    rank: int

    def allgather_int(self, x: int) -> List[int]:
        raise NotImplementedError

    def allgather_var(self, t, counts: List[int]):
        """Concatenate every rank's first counts[r] entries of `t`, rank order."""
        raise NotImplementedError

    def allreduce_sum_(self, t):
        raise NotImplementedError


class TorchDistComm(Comm):
    """torch.distributed collectives (NCCL for CUDA tensors, gloo for CPU)."""

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist, self.group = dist, group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)

    def _dev(self):
        import torch
        if self.dist.get_backend(self.group) == "nccl":
            return torch.device("cuda", torch.cuda.current_device())
        return torch.device("cpu")

    def allgather_int(self, x: int) -> List[int]:
        import torch
        t = torch.tensor([int(x)], dtype=torch.int64, device=self._dev())
        out = [torch.empty_like(t) for _ in range(self.world)]
        self.dist.all_gather(out, t, group=self.group)
        return [int(o.item()) for o in out]

    def allgather_var(self, t, counts: List[int]):
        import torch
        m = max(counts)
        if m == 0:
            return t[:0]
        pad = torch.empty(m, dtype=t.dtype, device=t.device)
        c = counts[self.rank]
        if c:
            pad[:c].copy_(t[:c])
        if self.dist.get_backend(self.group) == "nccl":
            out = torch.empty(m * self.world, dtype=t.dtype, device=t.device)
            self.dist.all_gather_into_tensor(out, pad, group=self.group)
            parts = [out[r * m: r * m + counts[r]] for r in range(self.world)]
        else:
            outs = [torch.empty_like(pad) for _ in range(self.world)]
            self.dist.all_gather(outs, pad, group=self.group)
            parts = [outs[r][:counts[r]] for r in range(self.world)]
        return torch.cat(parts)

    def allreduce_sum_(self, t):
        self.dist.all_reduce(t, op=self.dist.ReduceOp.SUM, group=self.group)
        return t


class ThreadComm(Comm):
    """Collectives between threads of one process (virtual shards on one GPU,
    SURVEY §4 (a)).  Create one shared `ThreadComm.Hub(world)` and one
    `ThreadComm(hub, rank)` per thread."""

    class Hub:
        def __init__(self, world: int):
            self.world = world
            self.barrier = threading.Barrier(world)
            self.slots = [None] * world

    def __init__(self, hub: "ThreadComm.Hub", rank: int):
        self.hub, self.world, self.rank = hub, hub.world, rank

    def _exchange(self, obj):
        h = self.hub
        h.barrier.wait()
        h.slots[self.rank] = obj
        h.barrier.wait()
        out = list(h.slots)
        h.barrier.wait()
        return out

    def allgather_int(self, x: int) -> List[int]:
        return [int(v) for v in self._exchange(int(x))]

    def allgather_var(self, t, counts: List[int]):
        import torch
        if t.is_cuda:
            torch.cuda.current_stream().synchronize()
        parts = self._exchange(t[:counts[self.rank]])
        return torch.cat([p.to(t.device) for p in parts])

    def allreduce_sum_(self, t):
        import torch
        if t.is_cuda:
            torch.cuda.current_stream().synchronize()
        parts = self._exchange(t.clone())
        acc = parts[0].to(t.device).clone()
        for p in parts[1:]:
            acc += p.to(t.device)
        t.copy_(acc)
        return t


# ------------------------------------------------------------------ steps --
class CudaSteps:
    """The product steps: sm_100a kernels through the C ABI on this rank's GPU."""

    _DT = {"float32": _abi.SS_FLOAT32, "float64": _abi.SS_FLOAT64,
           "int32": _abi.SS_INT32, "int64": _abi.SS_INT64}

    def __init__(self, ctx):
        import torch
        self.ctx = ctx
        self.torch = torch
        self.device = torch.device("cuda", ctx.device)

    def _code(self, x):
        return self._DT[str(x.dtype).replace("torch.", "")]

    def key_dtype(self, x):
        return self.torch.int32 if x.element_size() == 4 else self.torch.int64

    def sample(self, x, level: int, slot_begin: int, count: int):
        keys = self.torch.empty(count, dtype=self.key_dtype(x), device=self.device)
        if count and x.numel():
            self.ctx.step_sample(x, level, slot_begin, count, keys)
        return keys

    def tree(self, x_like, keys, b: int):
        t = self.torch
        tree = t.empty(b - 1, dtype=keys.dtype, device=self.device)
        spl = t.empty(b - 1, dtype=keys.dtype, device=self.device)
        eq = t.empty(b, dtype=t.uint8, device=self.device)
        self.ctx.step_tree(self._code(x_like), keys, b, True, tree, spl, eq)
        return tree, spl, eq

    def count(self, x, tree, b: int):
        t = self.torch
        totals = t.zeros(b, dtype=t.int64, device=self.device)
        orc = t.empty(x.numel() + 64, dtype=t.uint8, device=self.device)
        if x.numel():
            self.ctx.step_count(x, tree, b, totals, orc)
        return totals, orc

    def search(self, totals, b: int, k: int, eq):
        out = self.torch.empty(4, dtype=self.torch.int64, device=self.device)
        self.ctx.step_search(totals, b, k, eq, out)
        j, kk, nj, is_eq = (int(v) for v in out.cpu().tolist())
        return j, kk, nj, bool(is_eq)

    def filter(self, x, orc, j: int, expected: int):
        t = self.torch
        out = t.empty(max(expected, 1), dtype=x.dtype, device=self.device)
        cnt = t.zeros(1, dtype=t.int64, device=self.device)
        if x.numel() and expected:
            self.ctx.step_filter(x, orc, j, out, cnt)
        return out[:expected]

    def splitter_value(self, x_like, spl, j: int):
        t = self.torch
        vals = t.empty(1, dtype=x_like.dtype, device=self.device)
        key = spl[j - 1: j].contiguous()
        self.ctx.step_keys_to_values(self._code(x_like), key, vals.view(key.dtype))
        return vals.cpu().numpy()[0]

    def select(self, x, k: int):
        return self.ctx.select(x, k)


# ----------------------------------------------------------------- driver --
class ShardedSelect:
    """Exact selection of global rank k over the union of all ranks' shards."""

    def __init__(self, steps, comm: Comm | None = None, b: int = 256, s: int = 4096,
                 gather_threshold: int = 1 << 24, max_levels: int = 24):
        if comm is None:
            comm = TorchDistComm()
        if b < 4 or b > 256 or b & (b - 1):
            raise ValueError("b must be a power of two in [4, 256]")
        if s < b or s > 16384 or s & (s - 1):
            raise ValueError("s must be a power of two in [b, 16384]")
        self.steps, self.comm, self.b, self.s = steps, comm, b, s
        self.gather_threshold = int(gather_threshold)
        self.max_levels = max_levels
        self.last_levels: List[int] = []   # global n_l of the distributed levels

    @staticmethod
    def slot_range(sizes: List[int], rank: int, s: int):
        """Sample slots owned by `rank`: [floor(s*P_r/N), floor(s*P_{r+1}/N))."""
        N = sum(sizes)
        lo = sum(sizes[:rank])
        hi = lo + sizes[rank]
        return (s * lo) // N, (s * hi) // N

    def select(self, x, k: int):
        comm, steps, b, s = self.comm, self.steps, self.b, self.s
        sizes = comm.allgather_int(x.numel())
        N = sum(sizes)
        if not 0 <= k < N:
            raise ValueError(f"k={k} not in [0, {N})")
        cur, level = x, 0
        self.last_levels = []
        while True:
            N = sum(sizes)
            if N <= self.gather_threshold or level >= self.max_levels:
                allx = comm.allgather_var(cur, sizes)        # C3
                return steps.select(allx, k)                 # C4 implicit
            self.last_levels.append(N)
            s0, s1 = self.slot_range(sizes, comm.rank, s)
            local_keys = steps.sample(cur, level, s0, s1 - s0)
            counts = [self.slot_range(sizes, r, s)[1] - self.slot_range(sizes, r, s)[0]
                      for r in range(comm.world)]
            keys = comm.allgather_var(local_keys, counts)    # C1
            tree, spl, eq = steps.tree(cur, keys, b)
            local, orc = steps.count(cur, tree, b)
            totals = local.clone()
            comm.allreduce_sum_(totals)                      # C2
            j, kk, nj, is_eq = steps.search(totals, b, k, eq)
            if is_eq:                                        # §IV.C early exit
                return steps.splitter_value(cur, spl, j)
            mine = int(local[j].item())                      # this rank's share of bucket j
            cur = steps.filter(cur, orc, j, mine)
            sizes = comm.allgather_int(cur.numel())
            assert sum(sizes) == nj, (sizes, nj)
            k, level = kk, level + 1
