"""The cached CUDA graph of an exact call is keyed on (dtype, plan), not on
the input pointer or n: the size n, the rank k and the input pointer are
patched into the graph's init node, and level 0's kernels read the input from
LevelCtl::src (every kernel reads its level's size from its LevelCtl).
Calls that rotate over distinct buffers -- including misaligned views, whose
peeled heads differ -- must each return the oracle's element."""
import numpy as np
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu


def _bits(v):
    v = np.asarray(v)
    u = np.uint32 if v.dtype.itemsize == 4 else np.uint64
    return int(v.reshape(1).view(u)[0])


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("fused", [1, 0])
def test_rotating_buffers_share_one_graph(dtype, fused, cuda_device):
    import torch
    import paper_conf_ipps_ribizela19_b200 as ss
    ctx = ss.Context(0, fused_filter=fused)
    n = (1 << 22) + 3
    xs, xds = [], []
    for i in range(6):
        x = datagen.make(["uniform", "normal", "exponential"][i % 3], n + 3, dtype, seed=40 + i)
        base = torch.from_numpy(x).to("cuda:0")
        off = i % 4 if i < 4 else 0          # offsets 0..3 elements: different 16-byte heads
        xs.append(x[off:off + n])
        xds.append(base[off:off + n])
    ks = [n // 2, 7, n - 9]
    for rep in range(2):
        for i, (x, xd) in enumerate(zip(xs, xds)):
            k = ks[(i + rep) % len(ks)]
            assert _bits(ctx.select(xd, k)) == _bits(oracle.select(x, k)), (i, k, rep)
    ctx.close()


@pytest.mark.parametrize("dtype", [np.float32, np.int64])
def test_varying_sizes_share_graphs(dtype, cuda_device):
    """Sizes with the same level plan reuse one graph with n patched; sizes
    with other plans get their own.  Every call is exact, in any order."""
    import torch
    import paper_conf_ipps_ribizela19_b200 as ss
    ctx = ss.Context(0)
    kind = "normal" if np.dtype(dtype).kind == "f" else "int"
    sizes = [(1 << 22) + 3, (1 << 22) + 1001, (1 << 22) - 77777, (1 << 20) + 5, 70000, 5000, (1 << 22) + 5]
    data = {}
    for i, n in enumerate(sizes):
        x = datagen.make(kind, n, dtype, seed=60 + i)
        data[n] = (x, torch.from_numpy(x).to("cuda:0"))
    for rep in range(2):
        for i, n in enumerate(sizes if rep == 0 else sizes[::-1]):
            x, xd = data[n]
            for k in (n // 2, datagen.rank(n, i + 3 * rep)):
                assert _bits(ctx.select(xd, k)) == _bits(oracle.select(x, k)), (n, k, rep)
    ctx.close()
