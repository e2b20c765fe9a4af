"""The sharded driver with the real sm_100a steps at P > 1 on one GPU:
P virtual shards, one thread + context + stream each, collectives through
ThreadComm (NCCL refuses two ranks on one device)."""
import threading

import numpy as np
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu


def _run(shards, ks, P, b=256, thr=1 << 12):
    import torch
    import paper_conf_ipps_ribizela19_b200 as ss
    from paper_conf_ipps_ribizela19_b200.sharded import CudaSteps, ShardedSelect, ThreadComm
    hub = ThreadComm.Hub(P)
    out = [None] * P
    errs = []

    def worker(r):
        try:
            torch.cuda.set_device(0)
            st = torch.cuda.Stream()
            with torch.cuda.stream(st):
                ctx = ss.Context(0)
                x = torch.from_numpy(shards[r]).to("cuda:0")
                sel = ShardedSelect(CudaSteps(ctx), ThreadComm(hub, r), b=b, gather_threshold=thr)
                out[r] = [(np.asarray(sel.select(x, k)).tobytes(), list(sel.last_levels)) for k in ks]
                torch.cuda.synchronize()
                ctx.close()
        except Exception as e:  # pragma: no cover
            errs.append(e)
            hub.barrier.abort()

    ts = [threading.Thread(target=worker, args=(r,)) for r in range(P)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    if errs:
        raise errs[0]
    return out


@pytest.mark.parametrize("P", [2, 4])
@pytest.mark.parametrize("kind", ["uniform", "normal", "distinct16"])
def test_sharded_virtual_ranks(P, kind):
    n = (1 << 20) + 11
    shards = [datagen.make(kind, n + 1000 * r, np.float32, seed=datagen.dataset_seed(5, 0) + 7919 * r)
              for r in range(P)]
    full = np.concatenate(shards)
    N = full.size
    ks = [0, N // 2, N - 1, datagen.rank(N, 8)]
    out = _run(shards, ks, P)
    for r in range(1, P):
        assert out[r] == out[0]
    for (bits, levels), k in zip(out[0], ks):
        assert bits == np.asarray(oracle.select(full, k)).tobytes(), (kind, k)
    if kind != "distinct16":
        assert out[0][1][1], "expected at least one distributed level"


def test_sharded_noniid_and_empty():
    P = 3
    shards = [datagen.uniform(300000, np.float64, seed=1) + 10.0,
              np.zeros(0, np.float64),
              datagen.uniform(700000, np.float64, seed=2) - 10.0]
    full = np.concatenate(shards)
    ks = [0, 12345, full.size // 2, full.size - 1]
    out = _run(shards, ks, P, thr=1000)
    for (bits, _), k in zip(out[0], ks):
        assert bits == np.asarray(oracle.select(full, k)).tobytes()


def test_sharded_nccl_world1():
    """The NCCL code path of TorchDistComm (world size 1 on the test box)."""
    import os
    import socket
    import torch
    import torch.distributed as dist
    import paper_conf_ipps_ribizela19_b200 as ss
    from paper_conf_ipps_ribizela19_b200.sharded import CudaSteps, ShardedSelect, TorchDistComm
    with socket.socket() as s_:
        s_.bind(("127.0.0.1", 0))
        port = s_.getsockname()[1]
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda:0"))
    try:
        x_np = datagen.normal((1 << 20) + 3, np.float32, seed=4)
        x = torch.from_numpy(x_np).to("cuda:0")
        ctx = ss.Context(0)
        sel = ShardedSelect(CudaSteps(ctx), TorchDistComm(), gather_threshold=1000)
        for k in [0, 777, x_np.size // 2, x_np.size - 1]:
            assert np.asarray(sel.select(x, k)).tobytes() == np.asarray(oracle.select(x_np, k)).tobytes()
        assert sel.last_levels
        ctx.close()
    finally:
        dist.destroy_process_group()
