"""Multi-process (world_size 2, gloo, CPU) tests of the sharded driver's host
protocol: proportional sample slots, sample all-gather, count all-reduce,
global bucket search, equality exit, survivor gather.  The per-rank steps are
the CPU oracle's (tests/_oracle_steps.py)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import datagen
import oracle
from paper_conf_ipps_ribizela19_b200.sharded import ShardedSelect, TorchDistComm

WORLD = 2


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _shards(case):
    if case == "iid":
        return [datagen.uniform(3000, np.float32, seed=1 + r) for r in range(WORLD)]
    if case == "noniid":   # rank r holds values in [r, r+1)
        return [datagen.uniform(2000 + 500 * r, np.float32, seed=5 + r) + np.float32(r) for r in range(WORLD)]
    if case == "empty":
        return [datagen.normal(4000, np.float64, seed=3), np.zeros(0, np.float64)]
    if case == "equal":
        return [datagen.all_equal(2500, 7.0, np.float32) for _ in range(WORLD)]
    if case == "distinct":
        return [datagen.distinct(3000, 16, np.float32, seed=9 + r) for r in range(WORLD)]
    if case == "int":
        return [datagen.int_uniform(2049 + 7 * r, np.int64, seed=11 + r) for r in range(WORLD)]
    raise ValueError(case)


def _worker(rank, port, case, ks, thresholds, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    try:
        from _oracle_steps import OracleSteps
        shard = torch.from_numpy(_shards(case)[rank])
        res = []
        for thr in thresholds:
            sel = ShardedSelect(OracleSteps(), TorchDistComm(), b=16, s=256, gather_threshold=thr)
            for k in ks:
                v = sel.select(shard, k)
                res.append((thr, k, np.asarray(v).tobytes(), list(sel.last_levels)))
        q.put((rank, res))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("case", ["iid", "noniid", "empty", "equal", "distinct", "int"])
def test_sharded_protocol_gloo(case):
    full = np.concatenate(_shards(case))
    N = full.size
    ks = sorted({0, 1, N // 2, N - 1, datagen.rank(N, 4)})
    thresholds = [0, 64, 1 << 30]           # all levels distributed / mixed / gather at once
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, case, ks, thresholds, q)) for r in range(WORLD)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert out[0] == out[1]                 # every rank returns the identical answer
    for thr, k, bits, levels in out[0]:
        assert bits == np.asarray(oracle.select(full, k)).tobytes(), (case, thr, k)
        assert all(a > b for a, b in zip(levels, levels[1:]))
        if thr == 0 and case not in ("equal", "distinct"):
            assert len(levels) >= 1


def test_slot_ranges_partition_the_sample():
    sizes = [5, 0, 17, 3, 1000]
    s = 4096
    ranges = [ShardedSelect.slot_range(sizes, r, s) for r in range(len(sizes))]
    assert ranges[0][0] == 0 and ranges[-1][1] == s
    for (a0, a1), (b0, b1) in zip(ranges, ranges[1:]):
        assert a1 == b0
    assert ranges[1][0] == ranges[1][1]       # empty shard draws nothing
    # proportional to shard size (within one slot)
    for r, (a, b) in enumerate(ranges):
        assert abs((b - a) - s * sizes[r] / sum(sizes)) <= 1
