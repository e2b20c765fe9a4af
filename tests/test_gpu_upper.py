"""GPU parity of the top-k fusion (§IV.I, reading R22):
ss_select_upper returns the element of rank k and the n-k elements of ranks
k..n-1.  The output is a multiset (order unspecified), so it is compared with
the oracle's sorted slice as sorted raw bits; the value is bit-exact."""
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


def _sorted_bits(a):
    a = np.ascontiguousarray(a)
    u = np.uint32 if a.dtype.itemsize == 4 else np.uint64
    return np.sort(a.view(u))


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
    return datagen.make(kind, n, dtype, seed)


def _check(ctx, x, xd, k):
    v, out = ctx.select_upper(xd, k)
    ref = oracle.select_upper(x, k)
    assert _bits(v) == _bits(ref[0]) == _bits(oracle.select(x, k)), k
    got = out.cpu().numpy()
    assert got.size == x.size - k
    assert np.array_equal(_sorted_bits(got), _sorted_bits(ref)), k
    st = ctx.stats()
    assert st["upper_greater"] == x.size - oracle.count_leq(x, v), k


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("n", [1, 2, 3, 17, 1000, 4097, 16385, 65536 + 13, (1 << 20) + 7])
def test_upper_sizes(ctx, dtype, n):
    """Base case only, one level, several gather tiles with a ragged tail."""
    x = _gen("normal", n, dtype, seed=n + 5)
    xd = _dev(x)
    for k in sorted({0, n // 2, n - 1, min(1, n - 1), datagen.rank(n, n)}):
        _check(ctx, x, xd, k)


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("kind", ["uniform", "exponential", "distinct16", "equal", "perm", "specials"])
def test_upper_distributions(ctx, dtype, kind):
    """Duplicate-heavy and all-equal inputs (equality exits: the output is
    mostly copies of the result), the permutation, +-0 / NaN / inf."""
    n = (1 << 18) + 5
    x = _gen(kind, n, dtype, seed=21)
    xd = _dev(x)
    for k in sorted({0, 3, n // 2, n - 2, datagen.rank(n, 23)}):
        _check(ctx, x, xd, k)


@pytest.mark.parametrize("dtype", [np.float32, np.float64, np.int32])
@pytest.mark.parametrize("offset", [1, 2, 3])
def test_upper_misaligned_views(ctx, dtype, offset):
    """Unaligned heads (scalar edge path of the gather kernel)."""
    n = (1 << 17) + 11
    base = _gen("uniform", n + offset, dtype, seed=offset)
    bd = _dev(base)
    x, xd = base[offset:], bd[offset:]
    for k in (0, n // 3, n - 1):
        _check(ctx, x, xd, k)


def test_upper_paper_filter_path_same(cuda_device):
    """The fused-filter select and the paper's oracle-byte path give the same
    upper set (the gather depends only on the result)."""
    import paper_conf_ipps_ribizela19_b200 as ss
    n = (1 << 22) + 3
    x = _gen("normal", n, np.float32, seed=31)
    xd = _dev(x)
    a, b = ss.Context(0), ss.Context(0, fused_filter=0)
    for k in (n // 2, n - 4096):
        va, oa = a.select_upper(xd, k)
        vb, ob = b.select_upper(xd, k)
        assert _bits(va) == _bits(vb) == _bits(oracle.select(x, k))
        assert np.array_equal(_sorted_bits(oa.cpu().numpy()), _sorted_bits(ob.cpu().numpy()))
        assert np.array_equal(_sorted_bits(oa.cpu().numpy()), _sorted_bits(oracle.select_upper(x, k)))
    a.close()
    b.close()


def test_upper_rejects_bad_arguments(ctx):
    import torch
    from paper_conf_ipps_ribizela19_b200 import SSError
    xd = torch.arange(100, dtype=torch.float32, device="cuda:0")
    with pytest.raises(SSError):
        ctx.select_upper(xd, 100)
    with pytest.raises(SSError):          # output overlapping the input
        ctx.select_upper(xd, 50, out=xd[10:60])
    with pytest.raises(ValueError):       # too small
        ctx.select_upper(xd, 50, out=torch.empty(10, dtype=torch.float32, device="cuda:0"))


@pytest.mark.parametrize("k_frac", [0.5, 1.0 - 2.0 ** -18])
def test_upper_full_size_properties(ctx, k_frac):
    """BASELINE size (n = 2^28 fp32 uniform, the bench's launch config): the
    CPU oracle cannot sort 2^28 in seconds, so the multiset is checked against
    torch.sort on the device (a library sort; uniform [0,1) has no NaN / -0,
    where torch's order is totalOrder) and the value against the count
    invariant #{x < v} <= k < #{x <= v}."""
    import torch
    n = 1 << 28
    g = torch.Generator(device="cuda:0").manual_seed(1234)
    xd = torch.rand(n, device="cuda:0", generator=g, dtype=torch.float32)
    k = int(n * k_frac)
    v, out = ctx.select_upper(xd, k)
    vt = torch.tensor(float(v), device="cuda:0", dtype=torch.float32)
    assert int((xd < vt).sum()) <= k < int((xd <= vt).sum())
    assert ctx.stats()["upper_greater"] == int((xd > vt).sum())
    srt = torch.sort(xd).values[k:]
    assert torch.equal(torch.sort(out).values, srt)


# ---------------------------------------------- one-pass top-k (§IV.I) ----
# The paper's top-k fusion copies "not only elements from the target bucket,
# but also from all buckets containing larger elements" in the same filter
# pass (L606-615): a fused level 0 streams the keys above its window to the
# output while it copies the window; the tail adds the window's keys > result
# and the copies of result.  Same multiset as the two-pass path and the oracle.

@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("kind", ["normal", "distinct16", "equal", "specials"])
def test_upper_onepass_vs_oracle(ctx, dtype, kind):
    n = (1 << 20) + 7                     # a fused level 0 (>= spec_min_n), a ragged tail
    x = _gen(kind, n, dtype, seed=41)
    xd = _dev(x)
    for k in sorted({0, 1, n // 2, n - (1 << 14), n - 2, n - 1, datagen.rank(n, 42)}):
        _check(ctx, x, xd, k)
        st = ctx.stats()
        # level 0 is a fused hit (or an equality exit) on these inputs; with
        # 16 distinct values a window can collapse onto one value next to
        # rank k's run and miss (then the two-pass path ran; still exact);
        # outputs above n / 4 elements take the two-pass path by design
        # (specials: the +-0 / NaN runs likewise)
        if kind in ("normal", "equal") and n - k <= n // 4:
            assert st["upper_onepass"] == 1, (kind, k, st["spec_levels"], st["fused_levels"])


def test_upper_onepass_off_is_two_pass(cuda_device):
    import paper_conf_ipps_ribizela19_b200 as ss
    n = (1 << 21) + 5
    x = _gen("uniform", n, np.float32, seed=43)
    xd = _dev(x)
    a, b = ss.Context(0), ss.Context(0, upper_onepass=0)
    try:
        for k in (n - n // 10, n - 1000):
            va, oa = a.select_upper(xd, k)
            assert a.stats()["upper_onepass"] == 1
            vb, ob = b.select_upper(xd, k)
            assert b.stats()["upper_onepass"] == 0
            assert _bits(va) == _bits(vb) == _bits(oracle.select(x, k))
            assert np.array_equal(_sorted_bits(oa.cpu().numpy()), _sorted_bits(ob.cpu().numpy()))
    finally:
        a.close()
        b.close()


def _poisoned(n, dtype, seed, sample_seed, s):
    """Level 0's R7 sample draws land on the s smallest values (as in
    test_gpu_gaps.py): the fused window of level 0 misses rank k."""
    x = datagen.make("uniform" if np.dtype(dtype).kind == "f" else "int", n, dtype, seed)
    idx = oracle.sample_indices(sample_seed, 0, n, 0, s)
    if np.dtype(dtype).kind == "f":
        x[idx] = (np.min(x) - 1 - np.arange(idx.size)).astype(dtype)
    else:
        x[idx] = (np.iinfo(dtype).min + np.arange(idx.size)).astype(dtype)
    return x


@pytest.mark.parametrize("dtype", [np.float32, np.int64])
def test_upper_onepass_level0_miss_falls_back(ctx, dtype):
    """A level-0 window that misses rank k: the keys already streamed are
    discarded and the two-pass path writes the output; exact either way."""
    n = (1 << 22) + 1
    x = _poisoned(n, dtype, 6, ctx.config["seed"], 16384)
    xd = _dev(x)
    for k in (n // 2, n // 3):
        _check(ctx, x, xd, k)
        st = ctx.stats()
        assert st["upper_onepass"] == 0 and not st["fused_levels"] & 1, st


@pytest.mark.parametrize("dtype", [np.float32, np.int64])
def test_upper_onepass_overflowing_window(ctx, dtype):
    """40 % of the input is one value inside level 0's window: the window does
    not fit the level buffers, the level halts, the host grows them and
    re-runs; the output is still the exact multiset."""
    n = 1 << 22
    rng = np.random.default_rng(17)
    if np.dtype(dtype).kind == "f":
        x = datagen.uniform(n, dtype, seed=18)
        v = dtype(0.5)
    else:
        x = datagen.int_uniform(n, dtype, seed=18)
        v = dtype(0)
    x[rng.random(n) < 0.4] = v
    xd = _dev(x)
    below = int(np.sum(x < v))
    for k in (below + int(0.4 * n) - 1000, below - 5, n // 2, below + int(0.4 * n) + 50):
        _check(ctx, x, xd, k)


def test_upper_onepass_rotating_outputs(ctx):
    """The output pointer is patched into the cached graph: distinct output
    buffers on successive calls each get their own exact result."""
    import torch
    n = (1 << 20) + 3
    x = _gen("normal", n, np.float32, seed=47)
    xd = _dev(x)
    k = n - 5000
    ref = _sorted_bits(oracle.select_upper(x, k))
    outs = [torch.empty(n - k, dtype=torch.float32, device="cuda:0") for _ in range(3)]
    for o in outs:
        o.fill_(float("nan"))
    for o in outs:
        ctx.select_upper(xd, k, out=o)
        assert ctx.stats()["upper_onepass"] == 1
    for o in outs:
        assert np.array_equal(_sorted_bits(o.cpu().numpy()), ref)
