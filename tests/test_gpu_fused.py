"""GPU parity of the fused speculative filter ("fused filter"):
the count kernel copies the sample-predicted bucket window to the next level
instead of writing oracle bytes; a miss falls back to a re-classifying filter.
The answer must be the same element as the oracle's on every input, hit or
miss, for every dtype -- the window only changes which superset of bucket j the
next level sees (reading R6: r_wlo <= k < r_{whi+1})."""
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


def _dev(x):
    import torch
    return torch.from_numpy(np.ascontiguousarray(x)).to("cuda:0")


def _gen(kind, n, dtype, seed):
    if np.dtype(dtype).kind == "i" and kind in ("uniform", "normal", "exponential"):
        kind = "int"
    return datagen.make(kind, n, dtype, seed)


@pytest.fixture(scope="module")
def fctx(cuda_device):
    """Fused filter on every level that samples wide (spec_min_n = 1)."""
    import paper_conf_ipps_ribizela19_b200 as ss
    c = ss.Context(0, spec_min_n=1)
    yield c
    c.close()


@pytest.fixture(scope="module")
def missctx(cuda_device):
    """z = 0: a window of +-2 sample ranks, so most calls miss and take the
    re-classifying fallback filter."""
    import paper_conf_ipps_ribizela19_b200 as ss
    c = ss.Context(0, spec_min_n=1, spec_z=0.0)
    yield c
    c.close()


def _ranks(n, seed):
    return sorted({0, 1, n // 3, n // 2, n - 2, n - 1, datagen.rank(n, seed), datagen.rank(n, seed + 1)})


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("kind", ["uniform", "normal", "exponential", "distinct1024", "perm", "specials"])
def test_fused_exact(fctx, dtype, kind):
    if kind == "specials" and np.dtype(dtype).kind == "i":
        pytest.skip("float specials")
    n = (1 << 20) + 13
    x = _gen(kind, n, dtype, seed=21)
    xd = _dev(x)
    hits = 0
    for k in _ranks(n, 5):
        assert _bits(fctx.select(xd, k)) == _bits(oracle.select(x, k)), (kind, k)
        st = fctx.stats()
        hits += st["fused_levels"] & 1
        if st["spec_levels"] & 1 and st["fused_levels"] & 1 and not st["equality_exit"]:
            assert st["n_level"][1] < n
    if kind in ("uniform", "normal", "exponential", "perm"):
        assert hits >= 6, hits      # the window holds k's bucket with probability ~1 - 6e-5


@pytest.mark.parametrize("dtype", DTYPES)
def test_fused_miss_fallback(missctx, dtype):
    n = (1 << 20) + 7
    x = _gen("normal", n, dtype, seed=33)
    xd = _dev(x)
    misses = 0
    for k in _ranks(n, 9) + [datagen.rank(n, s) for s in range(20, 30)]:
        assert _bits(missctx.select(xd, k)) == _bits(oracle.select(x, k)), k
        st = missctx.stats()
        misses += (st["spec_levels"] & 1) and not (st["fused_levels"] & 1)
    assert misses >= 3, misses


def test_fused_vs_paper_filter_same_answer(cuda_device):
    import paper_conf_ipps_ribizela19_b200 as ss
    a = ss.Context(0, spec_min_n=1)
    b = ss.Context(0, fused_filter=0)
    n = (1 << 21) + 3
    x = _gen("exponential", n, np.float32, seed=4)
    xd = _dev(x)
    for k in _ranks(n, 77):
        assert _bits(a.select(xd, k)) == _bits(b.select(xd, k)) == _bits(oracle.select(x, k))
        assert b.stats()["spec_levels"] == 0
    a.close()
    b.close()


@pytest.mark.parametrize("offset", [1, 3])
def test_fused_misaligned(fctx, offset):
    n = 300007
    x = _gen("uniform", n + offset, np.float32, seed=offset)
    xd = _dev(x)[offset:]
    ref = x[offset:]
    for k in _ranks(n, offset):
        assert _bits(fctx.select(xd, k)) == _bits(oracle.select(ref, k))


@pytest.mark.parametrize("kind", ["distinct16", "equal", "distinct128"])
def test_fused_duplicates(fctx, kind):
    n = (1 << 20) + 1
    x = _gen(kind, n, np.float32, seed=8)
    xd = _dev(x)
    for k in _ranks(n, 3):
        assert _bits(fctx.select(xd, k)) == _bits(oracle.select(x, k)), k


def test_fused_default_large(cuda_device):
    """Default configuration at n = 2^25 (fused on level 0): invariant-checked,
    the level-0 window hit, and fewer algorithmic bytes than the paper's filter."""
    import paper_conf_ipps_ribizela19_b200 as ss
    c = ss.Context(0)
    n = 1 << 25
    x = datagen.uniform(n, np.float32, seed=datagen.dataset_seed(2, 1))
    xd = _dev(x)
    for k in [n // 2, 7, n - 3, datagen.rank(n, 2)]:
        v = c.select(xd, k)
        assert oracle.count_less(x, v) <= k < oracle.count_leq(x, v), k
        st = c.stats()
        assert st["spec_levels"] & 1 and st["fused_levels"] & 1, st
        assert st["bytes_algorithmic"] < 5.0 * n
    c.close()


# ------------------------------------------------- approximate variant -----
@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("b", [64, 256, 1024])
@pytest.mark.parametrize("z", [3.0, 0.0])
def test_fused_approx_matches_mirror(cuda_device, dtype, b, z):
    """§II.C through the one-pass splitter window (approx_window): the same
    splitter and the exact rank as the oracle's mirror with the same seed,
    whether the window decides (z = 3) or mostly falls back (z = 0)."""
    import paper_conf_ipps_ribizela19_b200 as ss
    c = ss.Context(0, spec_min_n=1, spec_z=z)
    n = (1 << 20) + 5
    x = _gen("normal", n, dtype, seed=b + 1)
    xd = _dev(x)
    s = oracle.sample_size(b)
    seed = c.config["seed"]
    decided = 0
    for k in _ranks(n, b):
        v, r = c.approx_select(xd, k, b)
        vo, ro, _ = oracle.approx_select(x, k, b, s, seed)
        assert _bits(v) == _bits(vo) and r == ro, (k, v, vo, r, ro)
        decided += c.stats()["fused_levels"] & 1
    if z == 3.0:
        assert decided >= 5, decided
    c.close()


def test_fused_approx_duplicates(cuda_device):
    import paper_conf_ipps_ribizela19_b200 as ss
    c = ss.Context(0, spec_min_n=1)
    for kind in ("distinct16", "distinct1024", "equal"):
        n = (1 << 20) + 1
        x = _gen(kind, n, np.float32, seed=4)
        xd = _dev(x)
        for k in _ranks(n, 2):
            for b in (64, 1024):
                v, r = c.approx_select(xd, k, b)
                vo, ro, _ = oracle.approx_select(x, k, b, oracle.sample_size(b), c.config["seed"])
                assert _bits(v) == _bits(vo) and r == ro, (kind, k, b)
    c.close()
