"""GPU parity of the histogram-directed levels (reading R28): a fused
level counts the keys it copies in 1024 equal key bins and the bin holding the
rank becomes the next level's window (no sample, no K1w, cannot miss).  The
answer must be the oracle's element on every input and rank, with the directed
levels on (default) and off, and the directed levels must actually run and hit
(no host re-run) on inputs without heavy duplicates."""
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


def _ranks(n, seed):
    return sorted({0, 1, 2, n // 3, n // 2, n - 3, n - 2, n - 1, datagen.rank(n, seed), datagen.rank(n, seed + 1)})


@pytest.fixture(scope="module")
def ctxs(cuda_device):
    import paper_conf_ipps_ribizela19_b200 as ss
    on, off = ss.Context(0), ss.Context(0, directed=0)
    assert on.config["directed"] == 1
    yield on, off
    on.close()
    off.close()


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("kind", ["uniform", "normal", "exponential", "perm", "distinct1024", "specials"])
def test_directed_exact(ctxs, dtype, kind):
    if kind == "specials" and np.dtype(dtype).kind == "i":
        pytest.skip("float specials")
    on, off = ctxs
    n = (1 << 22) + 11                       # plan: fused level 0, directed level 1, base case
    x = _gen(kind, n, dtype, seed=29)
    xd = _dev(x)
    for k in _ranks(n, 7):
        ref = _bits(oracle.select(x, k))
        assert _bits(on.select(xd, k)) == ref, (kind, k, "directed")
        st = on.stats()
        if kind in ("uniform", "normal", "exponential", "perm"):
            # level 1 is the directed level and it hit; no host round trip
            assert st["incomplete_rounds"] == 0, (k, st)
            if not st["equality_exit"]:
                assert st["spec_levels"] & 2 and st["fused_levels"] & 3 == 3, (k, st)
                assert st["n_level"][0] > st["n_level"][1] > st["n_level"][2], (k, st)
        assert _bits(off.select(xd, k)) == ref, (kind, k, "sampled")


@pytest.mark.parametrize("dtype", [np.float32, np.int64])
def test_directed_chain(cuda_device, dtype):
    """spec_min_n = 1 and the smallest base case: several directed levels in a row."""
    import paper_conf_ipps_ribizela19_b200 as ss
    c = ss.Context(0, spec_min_n=1, base_case=256)
    try:
        n = (1 << 21) + 5
        x = _gen("uniform", n, dtype, seed=3)
        xd = _dev(x)
        for k in _ranks(n, 11):
            assert _bits(c.select(xd, k)) == _bits(oracle.select(x, k)), k
            st = c.stats()
            assert st["incomplete_rounds"] == 0, st
            assert st["levels"] >= 3 or st["equality_exit"], st
    finally:
        c.close()


@pytest.mark.parametrize("dtype", DTYPES)
@pytest.mark.parametrize("case", ["top_run", "bottom_run", "narrow"])
def test_directed_duplicates(ctxs, dtype, case):
    """Runs at the largest / smallest key (padding below / above the window)
    and a narrow key range (one key bin holds a whole level)."""
    on, _ = ctxs
    n = (1 << 22) + 3
    rng = np.random.default_rng(5)
    x = _gen("uniform", n, dtype, seed=5)
    info = np.finfo(dtype) if np.dtype(dtype).kind == "f" else np.iinfo(dtype)
    if case == "top_run":
        x[rng.random(n) < 0.3] = info.max
    elif case == "bottom_run":
        x[rng.random(n) < 0.3] = info.min
    else:                                    # 1000 distinct values around one point
        base = np.asarray(1000, dtype)
        x = (base + rng.integers(0, 1000, n)).astype(dtype) if np.dtype(dtype).kind == "i" else \
            (np.asarray(1.0, dtype) + rng.integers(0, 1000, n).astype(dtype) * np.finfo(dtype).eps).astype(dtype)
    xd = _dev(x)
    for k in _ranks(n, 13):
        assert _bits(on.select(xd, k)) == _bits(oracle.select(x, k)), (case, k)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_top_window_histogram_spans_the_sample(dtype, cuda_device):
    """A level-0 window that runs to the top of the key range ([klo, 2^bits))
    is binned up to its sample's largest key plus one bin above it (which
    holds the ~n/s keys above the sample): the directed level after it leaves
    at most the base case B = 16384 keys, where bins over all of
    [klo, 2^bits) -- of which uniform [0, 1) keys occupy a sliver -- left
    21920 keys and needed one more level.  The answer stays exact."""
    import torch
    import paper_conf_ipps_ribizela19_b200 as ss
    c = ss.Context(0)
    try:
        n = (1 << 24) + 3
        x = datagen.uniform(n, dtype, seed=17)
        xd = torch.from_numpy(x).to("cuda:0")
        for k in (n - 1, n - 2, n - 100):
            assert _bits(c.select(xd, k)) == _bits(oracle.select(x, k)), k
            nl = c.stats()["n_level"]
            assert len(nl) == 3 and nl[2] <= 16384, nl
    finally:
        c.close()
