"""GPU parity of multi-rank selection (reading R23): every
rank's element bit-exact against the oracle (one sort, m indexings) on the
same seeded inputs, through the shared-count path (n >= 2^20) and the
per-rank path (smaller n)."""
import numpy as np
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu

DTYPES = [np.float32, np.float64, np.int32, np.int64]


def _bits_arr(a):
    a = np.ascontiguousarray(a)
    return a.view(np.uint32 if a.dtype.itemsize == 4 else np.uint64)


@pytest.fixture(scope="module")
def ctx(cuda_device):
    import paper_conf_ipps_ribizela19_b200 as ss
    return ss.Context(0)


def _gen(kind, n, dtype, seed):
    if kind in ("normal", "uniform", "exponential", "specials") and np.dtype(dtype).kind == "i":
        kind = "int"
    return datagen.make(kind, n, dtype, seed)


def _ranks(n, seed, m):
    rng = np.random.default_rng(seed)
    return [0, n - 1, n // 2, n // 2, 1] + rng.integers(0, n, m).tolist()


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("n", [1, 1000, 16385, (1 << 20) + 7, (1 << 22) + 3])
def test_multi_sizes(ctx, dtype, n):
    import torch
    x = _gen("normal", n, dtype, seed=n + 1)
    ks = [k for k in _ranks(n, n, 12) if k < n]
    got = ctx.select_multi(torch.from_numpy(x).to("cuda:0"), ks)
    assert np.array_equal(_bits_arr(got), _bits_arr(oracle.select_multi(x, ks)))


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("kind", ["uniform", "exponential", "distinct16", "distinct1024", "equal", "perm",
                                  "specials"])
def test_multi_distributions(ctx, dtype, kind):
    """Equality buckets (distinct16, equal: answered by their splitter),
    many ranks in one bucket, ranks spread over many buckets."""
    import torch
    n = (1 << 20) + 5
    x = _gen(kind, n, dtype, seed=51)
    ks = _ranks(n, 53, 40) + [n // 2 + i for i in range(5)]
    got = ctx.select_multi(torch.from_numpy(x).to("cuda:0"), ks)
    assert np.array_equal(_bits_arr(got), _bits_arr(oracle.select_multi(x, ks)))


def test_multi_equals_single_selects(ctx):
    """Same answers as m independent ss_select calls, paper path included."""
    import torch
    import paper_conf_ipps_ribizela19_b200 as ss
    n = (1 << 22) + 1
    x = _gen("normal", n, np.float32, seed=61)
    xd = torch.from_numpy(x).to("cuda:0")
    ks = _ranks(n, 62, 20)
    got = ctx.select_multi(xd, ks)
    single = np.array([ctx.select(xd, k) for k in ks], dtype=np.float32)
    assert np.array_equal(_bits_arr(got), _bits_arr(single))
    for m in (1, 2, 3):   # below MULTI_MIN_M: the per-rank path
        assert np.array_equal(_bits_arr(ctx.select_multi(xd, ks[:m])), _bits_arr(single[:m]))
    p = ss.Context(0, fused_filter=0)
    assert np.array_equal(_bits_arr(p.select_multi(xd, ks)), _bits_arr(got))
    p.close()


def test_multi_rejects_bad_arguments(ctx):
    import torch
    from paper_conf_ipps_ribizela19_b200 import SSError
    xd = torch.arange(100, dtype=torch.float32, device="cuda:0")
    with pytest.raises(SSError):
        ctx.select_multi(xd, [100])
    with pytest.raises(SSError):
        ctx.select_multi(xd, [-1])
    with pytest.raises(SSError):
        ctx.select_multi(xd, [])


@pytest.mark.parametrize("m", [2 * 4, 200])
def test_multi_one_pass_and_per_bucket_extraction(ctx, m):
    """<= 64 distinct buckets: one multi-bucket extraction pass; more: one
    filter pass per bucket.  Both bit-exact."""
    import torch
    n = (1 << 21) + 3
    x = _gen("normal", n, np.float32, seed=71 + m)
    ks = np.random.default_rng(m).integers(0, n, m).tolist()
    got = ctx.select_multi(torch.from_numpy(x).to("cuda:0"), ks)
    assert np.array_equal(_bits_arr(got), _bits_arr(oracle.select_multi(x, ks)))


# ------------------------------------------------ per-rank tails --------
# The per-rank selects run as exact calls on child contexts (their own
# streams), with graphs keyed on the plan and n patched per call.

def _check(ctx, x, xd, ks):
    got = ctx.select_multi(xd, ks)
    assert np.array_equal(_bits_arr(got), _bits_arr(oracle.select_multi(x, ks))), ks
    return ctx.stats()


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("kind", ["normal", "distinct16", "equal", "specials"])
def test_multi_few_ranks(ctx, dtype, kind):
    """4 .. 16 ranks (the bench's regime): shared count, one extraction pass,
    the per-rank tails concurrently on the child contexts."""
    import torch
    n = (1 << 22) + 9
    x = _gen(kind, n, dtype, seed=71)
    xd = torch.from_numpy(x).to("cuda:0")
    rng = np.random.default_rng(72)
    for ks in ([0, 1, n // 2, n - 1], [n // 3, n // 3 + 1, n // 3 + 2, n // 3 + 50000, 2 * n // 3],
               rng.integers(0, n, 8).tolist(), rng.integers(0, n, 16).tolist()):
        _check(ctx, x, xd, ks)


def test_multi_sorted_input(ctx):
    """A sorted input: each extracted bucket comes from one or two CTAs."""
    import torch
    n = (1 << 22) + 1
    x = np.sort(_gen("normal", n, np.float32, seed=74))
    xd = torch.from_numpy(x).to("cuda:0")
    _check(ctx, x, xd, [5, n // 4, n // 2, n - 7, 3 * n // 4])


def test_multi_rotating_sizes(ctx):
    """Bucket sizes change from call to call: the per-rank selects reuse their
    graphs with n patched (graphs keyed on the plan)."""
    import torch
    for i, n in enumerate([(1 << 22) + 1, (1 << 22) + 777, (1 << 21) + 5]):
        x = _gen("normal", n, np.float32, seed=80 + i)
        xd = torch.from_numpy(x).to("cuda:0")
        rng = np.random.default_rng(90 + i)
        _check(ctx, x, xd, rng.integers(0, n, 6).tolist())
