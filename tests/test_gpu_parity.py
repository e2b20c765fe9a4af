"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs.  Exact selection must be bit-exact; the approximate
variant must match the oracle's algorithm mirror bit-exactly (same seed) and
report the exact rank."""
import numpy as np
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu

DTYPES = [np.float32, np.float64, np.int32, np.int64]


def _bits(v):
    v = np.asarray(v)
    u = np.uint32 if v.dtype.itemsize == 4 else np.uint64
    return int(v.reshape(1).view(u)[0])


@pytest.fixture(scope="module")
def ctx(cuda_device):
    import paper_conf_ipps_ribizela19_b200 as ss
    return ss.Context(0)


def _dev(x):
    import torch
    return torch.from_numpy(np.ascontiguousarray(x)).to("cuda:0")


def _gen(kind, n, dtype, seed):
    if kind in ("uniform", "normal", "exponential", "specials") and np.dtype(dtype).kind == "i":
        kind = "int"
    if kind == "int" and np.dtype(dtype).kind == "f":
        kind = "uniform"
    return datagen.make(kind, n, dtype, seed)


def _ranks(n, seed):
    ks = {0, n - 1, n // 2, min(1, n - 1), datagen.rank(n, seed)}
    return sorted(ks)


# ----------------------------------------------------------- exact -------
@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("n", [1, 2, 3, 17, 1000, 16384, 16385, 65536 + 13, (1 << 20) + 7])
def test_exact_sizes(ctx, dtype, n):
    """Tiny (base case only), exactly B, B+1 (one level), ragged tails."""
    x = _gen("normal", n, dtype, seed=n)
    xd = _dev(x)
    for k in _ranks(n, n):
        assert _bits(ctx.select(xd, k)) == _bits(oracle.select(x, k)), (n, k)


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("n", [16385, 40001, 65535, 65536, 65537])
@pytest.mark.parametrize("kind", ["normal", "distinct16", "specials"])
def test_small_level_sizes(ctx, dtype, n, kind):
    """Just above the base case B = 16384 up to the smallest fused level
    (spec_min_n = 2^16): one paper or fused level, then the cluster base case."""
    x = _gen(kind, n, dtype, seed=n + 3)
    xd = _dev(x)
    for k in _ranks(n, n + 1) + [n // 3, n - 2]:
        assert _bits(ctx.select(xd, k)) == _bits(oracle.select(x, k)), (n, k, kind)


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("kind", ["uniform", "normal", "exponential", "distinct16", "distinct128",
                                  "distinct1024", "equal", "perm", "specials"])
def test_exact_distributions(ctx, dtype, kind):
    n = (1 << 18) + 5
    x = _gen(kind, n, dtype, seed=7)
    xd = _dev(x)
    for k in _ranks(n, 11):
        assert _bits(ctx.select(xd, k)) == _bits(oracle.select(x, k)), (kind, k)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("offset", [1, 2, 3])
def test_exact_misaligned_views(ctx, dtype, offset):
    """Device pointers that are not 16-byte aligned (head peeling)."""
    n = 100003
    x = _gen("uniform", n + offset, dtype, seed=offset)
    xd = _dev(x)[offset:]
    ref = x[offset:]
    for k in _ranks(n, offset):
        assert _bits(ctx.select(xd, k)) == _bits(oracle.select(ref, k))


def test_exact_host_input_path(ctx):
    x = _gen("normal", 300001, np.float32, seed=5)
    for k in _ranks(x.size, 5):
        assert _bits(ctx.select(x, k)) == _bits(oracle.select(x, k))


@pytest.mark.parametrize("b", [4, 16, 64, 128, 256])
def test_exact_bucket_counts(ctx, b):
    import paper_conf_ipps_ribizela19_b200 as ss
    c = ss.Context(0, b_exact=b, base_case=1024)
    x = _gen("normal", 200000, np.float64, seed=b)
    xd = _dev(x)
    for k in _ranks(x.size, b):
        assert _bits(c.select(xd, k)) == _bits(oracle.select(x, k))
    c.close()


def test_equality_exit_all_equal(ctx):
    x = datagen.all_equal(1 << 20, 42.0, np.float32)
    v = ctx.select(_dev(x), 12345)
    assert v == np.float32(42.0)
    st = ctx.stats()
    assert st["equality_exit"] and st["levels"] == 1


def test_signed_zeros_and_nans(ctx):
    """Reading R3: totalOrder places -0 before +0 and NaNs at the ends."""
    n = 50000
    x = np.zeros(n, np.float32)
    x[: n // 2] = -0.0
    x[:100] = np.array([0xFFC00000], np.uint32).view(np.float32)[0]   # -NaN
    x[-100:] = np.array([0x7FC00000], np.uint32).view(np.float32)[0]  # +NaN
    xd = _dev(x)
    for k in [0, 99, 100, n // 2 - 1, n // 2, n - 101, n - 100, n - 1]:
        assert _bits(ctx.select(xd, k)) == _bits(oracle.select(x, k)), k


def test_exact_level_statistics(ctx):
    """§II.B L169-171 depth bound and strictly shrinking levels."""
    n = 1 << 22
    x = _gen("uniform", n, np.float32, seed=1)
    ctx.select(_dev(x), n // 3)
    st = ctx.stats()
    nl = st["n_level"]
    assert nl[0] == n and all(a > b for a, b in zip(nl, nl[1:]))
    assert st["levels"] <= 3
    assert st["bytes_algorithmic"] >= 4 * n


# ------------------------------------------------------- approximate -----
@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("b", [64, 256, 1024])
def test_approx_matches_mirror(ctx, dtype, b):
    """§II.C: same seed, same sample -> identical value and exact rank."""
    n = (1 << 18) + 3
    x = _gen("normal", n, dtype, seed=b)
    xd = _dev(x)
    s = oracle.sample_size(b)
    seed = ctx.config["seed"]
    for k in _ranks(n, b):
        v, r = ctx.approx_select(xd, k, b)
        vo, ro, _ = oracle.approx_select(x, k, b, s, seed)
        assert _bits(v) == _bits(vo) and r == ro, (k, v, vo, r, ro)
        assert r == oracle.count_less(x, v)


def test_approx_duplicates(ctx):
    x = datagen.distinct(1 << 18, 16, np.float32, seed=2)
    xd = _dev(x)
    for k in [0, 1000, 1 << 17, (1 << 18) - 1]:
        v, r = ctx.approx_select(xd, k, 256)
        vo, ro, _ = oracle.approx_select(x, k, 256, oracle.sample_size(256), ctx.config["seed"])
        assert _bits(v) == _bits(vo) and r == ro


# ------------------------------------------------------- single steps -----
def test_step_tree_and_count_and_filter(ctx):
    import torch
    n, b, s = (1 << 20) + 9, 256, 4096
    x = _gen("normal", n, np.float32, seed=3)
    xd = _dev(x)
    keys = torch.empty(s, dtype=torch.int32, device="cuda:0")
    ctx.step_sample(xd, 0, 0, s, keys)
    idx = oracle.sample_indices(ctx.config["seed"], 0, n, 0, s)
    # keys are order-preserving images; compare the tree against the oracle
    # tree built from the same sampled values
    spl = oracle.pick_splitters(x[idx], b)
    fixed, eq_o = oracle.equality_fixup(spl)
    tree_o = oracle.heap_tree(fixed)
    tree = torch.empty(b - 1, dtype=torch.int32, device="cuda:0")
    splt = torch.empty(b - 1, dtype=torch.int32, device="cuda:0")
    eq = torch.empty(b, dtype=torch.uint8, device="cuda:0")
    ctx.step_tree(0, keys, b, True, tree, splt, eq)
    vals = torch.empty(b - 1, dtype=torch.float32, device="cuda:0")
    ctx.step_keys_to_values(0, tree, vals)
    assert np.array_equal(vals.cpu().numpy().view(np.uint32), tree_o.view(np.uint32))
    assert np.array_equal(eq.cpu().numpy(), eq_o)
    totals = torch.zeros(b, dtype=torch.int64, device="cuda:0")
    orc = torch.empty(n + 64, dtype=torch.uint8, device="cuda:0")
    ctx.step_count(xd, tree, b, totals, orc)
    counts_o, orc_o = oracle.count_buckets(x, tree_o)
    assert np.array_equal(totals.cpu().numpy(), counts_o)
    assert np.array_equal(orc[:n].cpu().numpy(), orc_o)   # 16B-aligned tensor: pad 0
    j = int(np.argmax(counts_o))
    out = torch.empty(n, dtype=torch.float32, device="cuda:0")
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda:0")
    ctx.step_filter(xd, orc, j, out, cnt)
    m = int(cnt.item())
    assert m == counts_o[j]
    # the filter is not stable (R15, like the paper's shared counter): compare the multisets
    assert np.array_equal(np.sort(out[:m].cpu().numpy().view(np.uint32)),
                          np.sort(oracle.filter_bucket(x, orc_o, j).view(np.uint32)))
    sr = torch.empty(4, dtype=torch.int64, device="cuda:0")
    k = n // 2
    ctx.step_search(totals, b, k, eq, sr)
    C = np.concatenate([[0], np.cumsum(counts_o)])
    jj = int(np.searchsorted(C, k, side="right") - 1)
    assert sr.cpu().tolist() == [jj, k - C[jj], counts_o[jj], int(eq_o[jj])]


# ------------------------------------------------------- full sizes ------
def _invariant(x, k, v):
    """#{x<v} <= k < #{x<=v}: holds for exactly one bit pattern v."""
    return oracle.count_less(x, v) <= k < oracle.count_leq(x, v)


@pytest.mark.parametrize("dtype,kind", [(np.float32, "uniform"), (np.float32, "normal"),
                                        (np.float64, "uniform"), (np.float64, "normal")])
def test_config2_n2p24(ctx, dtype, kind):
    """BASELINE config 2: n=2^24, k in {1, n/2, n-1}."""
    n = 1 << 24
    x = _gen(kind, n, dtype, seed=datagen.dataset_seed(2, 0))
    xd = _dev(x)
    for k in [1, n // 2, n - 1]:
        assert _invariant(x, k, ctx.select(xd, k)), k


@pytest.mark.parametrize("kind", ["distinct16", "equal"])
def test_config3_adversarial_n2p26(ctx, kind):
    n = 1 << 26
    x = _gen(kind, n, np.float32, seed=datagen.dataset_seed(3, 0))
    xd = _dev(x)
    for k in [0, n // 2, n - 1, datagen.rank(n, 3)]:
        assert _invariant(x, k, ctx.select(xd, k)), k
        assert ctx.stats()["equality_exit"]


def test_bench_workload_n2p28(ctx):
    """The bench's configuration: n=2^28 uniform fp32, k=n/2 and random k."""
    n = 1 << 28
    x = datagen.uniform(n, np.float32, seed=datagen.dataset_seed(5, 0))
    xd = _dev(x)
    for k in [n // 2, datagen.rank(n, 5)]:
        assert _invariant(x, k, ctx.select(xd, k)), k
    v, r = ctx.approx_select(xd, n // 2, 1024)
    assert r == oracle.count_less(x, v)
    assert abs(r - n // 2) <= 4 * n // 1024
