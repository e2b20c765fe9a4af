"""GPU parity of the atomics ablation count kernel (§V.E
L854-865, Fig. 6, Fig. 8 right): every increment strategy -- shared
or global atomics, with or without warp aggregation, and Fig. 6's per-bit
ballot mask (reading R13) -- must give exactly the oracle's bucket sizes
(§II.A) for the same tree."""
import numpy as np
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu

MODES = ["shared", "shared_wa", "shared_fig6", "global", "global_wa"]


@pytest.fixture(scope="module")
def ctx(cuda_device):
    import paper_conf_ipps_ribizela19_b200 as ss
    return ss.Context(0)


def _gen(kind, n, dtype, seed):
    if np.dtype(dtype).kind == "i" and kind in ("normal", "uniform"):
        kind = "int"
    return datagen.make(kind, n, dtype, seed)


def _tree(ctx, x, xd, b, dtype):
    import torch
    s = 4096
    kd = torch.int32 if np.dtype(dtype).itemsize == 4 else torch.int64
    keys = torch.empty(s, dtype=kd, device="cuda:0")
    ctx.step_sample(xd, 0, 0, s, keys)
    idx = oracle.sample_indices(ctx.config["seed"], 0, x.size, 0, s)
    fixed, _ = oracle.equality_fixup(oracle.pick_splitters(x[idx], b))
    tree_o = oracle.heap_tree(fixed)
    tree = torch.empty(b - 1, dtype=kd, device="cuda:0")
    spl = torch.empty(b - 1, dtype=kd, device="cuda:0")
    eq = torch.empty(b, dtype=torch.uint8, device="cuda:0")
    dtc = {4: 0, 8: 1}[np.dtype(dtype).itemsize] if np.dtype(dtype).kind == "f" else \
        {4: 2, 8: 3}[np.dtype(dtype).itemsize]
    ctx.step_tree(dtc, keys, b, True, tree, spl, eq)
    return tree, tree_o


@pytest.mark.parametrize("dtype", [np.float32, np.float64, np.int32])
@pytest.mark.parametrize("kind", ["normal", "distinct16", "equal", "perm"])
@pytest.mark.parametrize("b", [16, 256])
def test_ablation_modes_match_oracle_counts(ctx, dtype, kind, b):
    import torch
    n = (1 << 20) + 9
    x = _gen(kind, n, dtype, seed=41)
    xd = torch.from_numpy(x).to("cuda:0")
    tree, tree_o = _tree(ctx, x, xd, b, dtype)
    counts_o, _ = oracle.count_buckets(x, tree_o)
    for mode in MODES:
        totals = torch.full((b,), -1, dtype=torch.int64, device="cuda:0")
        ctx.step_count_ablation(xd, tree, b, mode, totals)
        assert np.array_equal(totals.cpu().numpy(), counts_o), (mode, kind)


@pytest.mark.parametrize("offset", [1, 3])
def test_ablation_misaligned_and_tiny(ctx, offset):
    import torch
    for n in (1, 5, 37, 4097 + offset):
        base = _gen("normal", n + offset, np.float32, seed=n)
        bd = torch.from_numpy(base).to("cuda:0")
        x, xd = base[offset:], bd[offset:]
        big = _gen("normal", 1 << 14, np.float32, seed=3)
        tree, tree_o = _tree(ctx, big, torch.from_numpy(big).to("cuda:0"), 16, np.float32)
        counts_o, _ = oracle.count_buckets(x, tree_o)
        for mode in MODES:
            totals = torch.zeros(16, dtype=torch.int64, device="cuda:0")
            ctx.step_count_ablation(xd, tree, 16, mode, totals)
            assert np.array_equal(totals.cpu().numpy(), counts_o), (mode, n)
