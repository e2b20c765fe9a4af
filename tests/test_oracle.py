"""Pins for the CPU oracle (``oracle/``) against things other than itself:
hand-worked examples from the paper (tests/golden/), closed forms, library
special cases (numpy.partition / min / max / searchsorted), brute force on
tiny inputs, a published RNG test vector and invariants.  CPU only."""
import json
import os

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import datagen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def _bits_array(bits, dtype):
    u = np.uint32 if np.dtype(dtype).itemsize == 4 else np.uint64
    return np.array([int(b, 16) for b in bits], dtype=u).view(dtype)


def _bits(v):
    v = np.asarray(v)
    u = np.uint32 if v.dtype.itemsize == 4 else np.uint64
    return int(v.reshape(1).view(u)[0])


# ---------------------------------------------------------------- golden -----
@pytest.mark.parametrize("case", _load("select_examples.json")["cases"],
                         ids=lambda c: c["cite"][:40])
def test_golden_select(case):
    dt = np.dtype(case["dtype"])
    if "bits" in case:
        x = _bits_array(case["bits"], dt)
        exp = int(case["expect"], 16)
        assert _bits(oracle.select(x, case["k"])) == exp
        assert _bits(oracle.select_bruteforce(x, case["k"])) == exp
    else:
        x = np.array(case["values"], dtype=dt)
        assert int(oracle.select(x, case["k"])) == case["expect"]
        assert int(oracle.select_bruteforce(x, case["k"])) == case["expect"]
    if "rank" in case:
        assert oracle.count_less(x, oracle.select(x, case["k"])) == case["rank"]


def test_golden_tree_walk():
    g = _load("tree_examples.json")["heap"]
    spl = np.array(g["splitters"], dtype=np.int32)
    tree = oracle.heap_tree(spl)
    assert tree.tolist() == g["tree"]
    for w in g["walks"]:
        assert oracle.tree_bucket(tree, w["x"]) == w["bucket"], w["path"]


@pytest.mark.parametrize("case", _load("tree_examples.json")["fixup"], ids=lambda c: c["cite"][:40])
def test_golden_equality_fixup(case):
    dt = np.dtype(case["dtype"])
    if "splitters" in case:
        fixed, eq = oracle.equality_fixup(np.array(case["splitters"], dtype=dt))
        assert fixed.tolist() == case["fixed"]
    else:
        fixed, eq = oracle.equality_fixup(_bits_array(case["splitter_bits"], dt))
        assert [hex(_bits(v)) for v in fixed] == [hex(int(b, 16)) for b in case["fixed_bits"]]
    assert eq.tolist() == case["eq"]


def test_splitmix64_published_vector():
    g = _load("tree_examples.json")["splitmix64"]
    state, outs = 0, []
    for _ in range(3):
        outs.append(oracle.splitmix64(state))
        state = (state + 0x9E3779B97F4A7C15) % 2**64
    assert outs == [int(h, 16) for h in g["outputs_from_state_0"]]


# ----------------------------------------------------------- ordering --------
F32_ORDER = ["0xffffffff", "0xffc00000", "0xff800001", "0xff800000", "0xff7fffff", "0xbf800000",
             "0x80000001", "0x80000000", "0x00000000", "0x00000001", "0x3f800000", "0x7f7fffff",
             "0x7f800000", "0x7f800001", "0x7fc00000", "0x7fffffff"]


def test_total_order_table_f32():
    """Hand-listed IEEE totalOrder chain (reading R3): -NaN(max payload) <
    -qNaN < -sNaN < -inf < -max < -1 < -denorm < -0 < +0 < ... < +qNaN < +NaN(max)."""
    vals = _bits_array(F32_ORDER, np.float32)
    for i in range(len(vals)):
        for j in range(len(vals)):
            assert oracle.cmp(vals[i], vals[j], np.float32) == (i > j) - (i < j), (i, j)


def test_total_order_table_f64():
    order = ["0xffffffffffffffff", "0xfff8000000000000", "0xfff0000000000000", "0xbff0000000000000",
             "0x8000000000000001", "0x8000000000000000", "0x0000000000000000", "0x0000000000000001",
             "0x3ff0000000000000", "0x7ff0000000000000", "0x7ff0000000000001", "0x7fffffffffffffff"]
    vals = _bits_array(order, np.float64)
    for i in range(len(vals)):
        for j in range(len(vals)):
            assert oracle.cmp(vals[i], vals[j], np.float64) == (i > j) - (i < j)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_order_matches_ieee_less_on_ordinary_values(dtype):
    x = datagen.normal(500, dtype, seed=3)
    x = x[x != 0]
    for a, b in zip(x[:-1], x[1:]):
        assert oracle.cmp(a, b, dtype) == int(a > b) - int(a < b)


# ------------------------------------------------------ exact selection ------
@pytest.mark.parametrize("dtype", [np.float32, np.float64, np.int32, np.int64])
@pytest.mark.parametrize("kind", ["uniform", "normal", "distinct16", "equal", "int"])
def test_select_matches_numpy_partition(dtype, kind):
    """L601-603: the paper checks against std::nth_element; numpy.partition is
    the same library special case (NaN-free, no mixed +-0)."""
    if kind == "int" and np.dtype(dtype).kind == "f":
        kind = "exponential"
    if kind in ("uniform", "normal", "exponential") and np.dtype(dtype).kind == "i":
        kind = "int"
    x = datagen.make(kind, 3001, dtype, seed=11)
    for k in [0, 1, 1500, 2999, 3000, datagen.rank(3001, 5)]:
        ref = np.partition(x, k)[k]
        assert _bits(oracle.select(x, k)) == _bits(ref)


@pytest.mark.parametrize("dtype", [np.float32, np.float64, np.int32, np.int64])
def test_select_min_max(dtype):
    x = datagen.make("int" if np.dtype(dtype).kind == "i" else "normal", 777, dtype, seed=2)
    assert _bits(oracle.select(x, 0)) == _bits(x.min())
    assert _bits(oracle.select(x, x.size - 1)) == _bits(x.max())


@pytest.mark.parametrize("dtype", [np.float32, np.float64, np.int32, np.int64])
def test_select_permutation_closed_form(dtype):
    """permutation input -> the rank-k element is base + k."""
    n = 4099
    x = datagen.permutation(n, dtype, seed=9)
    base = {4: 0x00800000, 8: 0x0010000000000000}[np.dtype(dtype).itemsize] \
        if np.dtype(dtype).kind == "f" else 0
    for k in [0, 1, 2048, n - 1]:
        v = oracle.select(x, k)
        if np.dtype(dtype).kind == "f":
            assert _bits(v) == base + k
        else:
            assert int(v) == k


def test_select_d_distinct_closed_form():
    """d distinct values v_j with counts c_j: the answer is v_j with
    C_j <= k < C_{j+1} (C = cumulative counts, computed with bincount)."""
    n, d = 10000, 16
    x = datagen.distinct(n, d, np.float32, seed=4)
    c = np.bincount(x.astype(np.int64), minlength=d)
    C = np.concatenate([[0], np.cumsum(c)])
    for k in range(0, n, 97):
        j = int(np.searchsorted(C, k, side="right") - 1)
        assert oracle.select(x, k) == np.float32(j)


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_count_invariant_with_specials(dtype):
    """§II L82-88 as an invariant: #{x < v} <= k < #{x <= v}."""
    x = datagen.specials(2000, dtype, seed=7)
    for k in [0, 1, 500, 1000, 1999]:
        v = oracle.select(x, k)
        assert oracle.count_less(x, v) <= k < oracle.count_leq(x, v)


_f32_special = st.sampled_from([int(b, 16) for b in F32_ORDER] + [0x3f800000, 0x40000000, 0xc0000000])


@settings(max_examples=150, deadline=None)
@given(st.lists(_f32_special, min_size=1, max_size=40), st.data())
def test_select_bruteforce_tiny_special_f32(bits, data):
    x = np.array(bits, dtype=np.uint32).view(np.float32)
    k = data.draw(st.integers(0, len(bits) - 1))
    v = oracle.select(x, k)
    assert _bits(v) == _bits(oracle.select_bruteforce(x, k))
    # independent check: sorting the hand-ordered index table
    pos = {int(b, 16): i for i, b in enumerate(F32_ORDER)}
    if all(b in pos for b in bits):
        assert _bits(v) == sorted(bits, key=lambda b: pos[b])[k]


@settings(max_examples=150, deadline=None)
@given(st.lists(st.integers(-3, 3), min_size=1, max_size=50), st.data())
def test_select_bruteforce_tiny_duplicates_int64(vals, data):
    x = np.array(vals, dtype=np.int64)
    k = data.draw(st.integers(0, len(vals) - 1))
    assert int(oracle.select(x, k)) == sorted(vals)[k] == int(oracle.select_bruteforce(x, k))


def test_select_rejects_bad_rank():
    with pytest.raises(ValueError):
        oracle.select(np.zeros(3, np.float32), 3)
    with pytest.raises(ValueError):
        oracle.select(np.zeros(3, np.float32), -1)


# --------------------------------------------------------- method steps ------
def test_sample_indices_range_determinism_and_sharding():
    idx = oracle.sample_indices(0x5A17, 0, 1000, 0, 4096)
    assert idx.min() >= 0 and idx.max() < 1000
    assert np.array_equal(idx, oracle.sample_indices(0x5A17, 0, 1000, 0, 4096))
    assert np.array_equal(idx[100:300], oracle.sample_indices(0x5A17, 0, 1000, 100, 200))
    assert not np.array_equal(idx, oracle.sample_indices(0x5A17, 1, 1000, 0, 4096))
    # uniformity (§II.B L182-184 assumes uniform, independent draws): chi-square
    big = oracle.sample_indices(1, 0, 64, 0, 64000)
    c = np.bincount(big, minlength=64)
    chi2 = ((c - 1000.0) ** 2 / 1000.0).sum()
    assert chi2 < 120  # 63 dof; p ~ 1e-5 threshold


def test_pick_splitters_closed_form():
    """Sample = a permutation of 0..s-1: the i/b percentile is floor(i*s/b)."""
    s, b = 4096, 256
    sample = datagen.permutation(s, np.int32, seed=1)
    spl = oracle.pick_splitters(sample, b)
    assert spl.tolist() == [(i * s) // b for i in range(1, b)]


@pytest.mark.parametrize("b", [2, 4, 8, 64, 256, 1024])
def test_heap_tree_inorder_is_sorted(b):
    spl = np.sort(datagen.int_uniform(b - 1, np.int32, seed=b))
    tree = oracle.heap_tree(spl)

    def inorder(i):
        if i >= b - 1:
            return []
        return inorder(2 * i + 1) + [int(tree[i])] + inorder(2 * i + 2)
    assert inorder(0) == spl.tolist()


@pytest.mark.parametrize("b", [4, 16, 256])
def test_tree_bucket_counts_splitters_leq(b):
    """Fig. 4 walk == #{splitters <= x} (incl. duplicate splitters)."""
    g = datagen.rng(b)
    for trial in range(20):
        spl = np.sort(g.integers(-5, 6, size=b - 1).astype(np.int64))
        tree = oracle.heap_tree(spl)
        for x in range(-7, 8):
            assert oracle.tree_bucket(tree, x) == int((spl <= x).sum())


def test_count_buckets_matches_searchsorted():
    x = datagen.uniform(20000, np.float32, seed=8)
    spl = np.sort(x[:255].copy())
    counts, orc = oracle.count_buckets(x, oracle.heap_tree(spl))
    ref = np.searchsorted(spl, x, side="right")
    assert np.array_equal(orc, ref.astype(np.uint8))
    assert np.array_equal(counts, np.bincount(ref, minlength=256))
    j = int(orc[123])
    assert np.array_equal(oracle.filter_bucket(x, orc, j), x[orc == j])


@pytest.mark.parametrize("kind", ["distinct16", "equal", "distinct1024"])
def test_equality_buckets_hold_only_copies(kind):
    """§IV.C: after the fix-up every flagged bucket contains copies of one value."""
    x = datagen.make(kind, 1 << 15, np.float32, seed=3)
    idx = oracle.sample_indices(0x5A17, 0, x.size, 0, 4096)
    spl = oracle.pick_splitters(x[idx], 256)
    fixed, eq = oracle.equality_fixup(spl)
    counts, orc = oracle.count_buckets(x, oracle.heap_tree(fixed))
    for j in np.nonzero(eq)[0]:
        vals = np.unique(x[orc == j])
        assert vals.size <= 1
    if kind != "distinct1024":
        # d <= 16 values, all sampled: every non-empty bucket is an equality bucket
        assert all(eq[j] for j in np.nonzero(counts)[0])


# ------------------------------------------------------- method mirror -------
@pytest.mark.parametrize("kind,dtype", [("uniform", np.float32), ("normal", np.float64),
                                        ("distinct16", np.float32), ("equal", np.float32),
                                        ("perm", np.int32), ("specials", np.float32),
                                        ("int", np.int64), ("distinct128", np.float64)])
def test_sampleselect_mirror_matches_definition(kind, dtype):
    """Fig. 1 recursion reaches exactly the sort-and-index answer."""
    n = 1 << 16
    x = datagen.make(kind, n, dtype, seed=21)
    for k in [0, 1, n // 2, n - 1, datagen.rank(n, 3)]:
        v, levels = oracle.sampleselect(x, k, b=256, s=4096, base_case=1024, seed=0x5A17)
        assert _bits(v) == _bits(oracle.select(x, k))
        assert all(a > b for a, b in zip(levels, levels[1:]))  # strict progress
        if kind == "equal":
            assert len(levels) == 1  # one count pass, then the equality exit


def test_sampleselect_depth_bound():
    """§II.B: at most log_b(n/B) + 1 levels on continuous data (+1
    slack for sample imbalance)."""
    n, b, B = 1 << 18, 64, 256
    x = datagen.uniform(n, np.float32, seed=5)
    _, levels = oracle.sampleselect(x, n // 3, b=b, s=4096, base_case=B, seed=1)
    assert len(levels) <= int(np.ceil(np.log(n / B) / np.log(b))) + 2


# ------------------------------------------------------ approximate ----------
def test_approx_rank_exact_and_error_bound():
    """§II.C: rank r_i of the returned splitter is exact, and the
    rank error is at most half the size of the bucket holding k (interior)
    or the bucket size (edge buckets)."""
    n, b, s = 1 << 16, 64, 4096
    x = datagen.normal(n, np.float32, seed=12)
    idx = oracle.sample_indices(77, 0, n, 0, s)
    spl = oracle.pick_splitters(x[idx], b)
    ranks = np.searchsorted(np.sort(x), spl, side="left")
    sizes = np.diff(np.concatenate([[0], ranks, [n]]))
    for k in [0, 5, n // 2, n - 1, 12345]:
        v, r, i = oracle.approx_select(x, k, b, s, 77)
        assert r == int((x < v).sum())                  # exact rank, brute force
        assert v == spl[i - 1]                          # a splitter
        j = int(np.searchsorted(ranks, k, side="right"))
        bound = sizes[j] if j in (0, b - 1) else (sizes[j] + 1) // 2
        assert abs(r - k) <= bound


@pytest.mark.parametrize("b", [64, 256])
def test_approx_error_statistics(b):
    """§V.G L897-908 / reading R12: mean relative rank error ~ 1/(4b), max <= 4/b."""
    n, s = 1 << 18, oracle.sample_size(b)
    x = datagen.uniform(n, np.float32, seed=13)
    errs = []
    for t in range(60):
        k = datagen.rank(n, 100 + t)
        _, r, _ = oracle.approx_select(x, k, b, s, 1000 + t)
        errs.append(abs(r - k) / n)
    errs = np.array(errs)
    assert 0.4 / (4 * b) <= errs.mean() <= 2.5 / (4 * b)
    assert errs.max() <= 4.0 / b


# ------------------------------------------- top-k fusion (§IV.I) ------------
def _sorted_bits(a):
    a = np.asarray(a)
    u = np.uint32 if a.dtype.itemsize == 4 else np.uint64
    return sorted(int(v) for v in a.view(u))


@pytest.mark.parametrize("case", _load("upper_examples.json")["cases"], ids=lambda c: c["cite"][:40])
def test_golden_select_upper(case):
    dt = np.dtype(case["dtype"])
    if "bits" in case:
        x = _bits_array(case["bits"], dt)
        exp = [int(b, 16) for b in case["expect_bits"]]
        got = oracle.select_upper(x, case["k"])
        assert [_bits(v) for v in got] == exp
        assert _sorted_bits(oracle.select_upper_bruteforce(x, case["k"])) == sorted(exp)
    else:
        x = np.array(case["values"], dtype=dt)
        assert oracle.select_upper(x, case["k"]).tolist() == case["expect"]
        assert sorted(oracle.select_upper_bruteforce(x, case["k"]).tolist()) == case["expect"]


@settings(max_examples=150, deadline=None)
@given(st.lists(_f32_special, min_size=1, max_size=40), st.data())
def test_select_upper_bruteforce_tiny_special_f32(bits, data):
    x = np.array(bits, dtype=np.uint32).view(np.float32)
    k = data.draw(st.integers(0, len(bits) - 1))
    up = oracle.select_upper(x, k)
    assert up.size == len(bits) - k
    assert _sorted_bits(up) == _sorted_bits(oracle.select_upper_bruteforce(x, k))
    pos = {int(b, 16): i for i, b in enumerate(F32_ORDER)}
    if all(b in pos for b in bits):   # independent: the hand-ordered totalOrder table
        assert [_bits(v) for v in up] == sorted(bits, key=lambda b: pos[b])[k:]


@settings(max_examples=150, deadline=None)
@given(st.lists(st.integers(-3, 3), min_size=1, max_size=50), st.data())
def test_select_upper_bruteforce_tiny_duplicates_int64(vals, data):
    x = np.array(vals, dtype=np.int64)
    k = data.draw(st.integers(0, len(vals) - 1))
    assert oracle.select_upper(x, k).tolist() == sorted(vals)[k:]
    assert sorted(oracle.select_upper_bruteforce(x, k).tolist()) == sorted(vals)[k:]


@pytest.mark.parametrize("dtype", [np.float32, np.float64, np.int32, np.int64])
def test_select_upper_special_cases_and_numpy(dtype):
    """k = 0 -> the input as a multiset; k = n-1 -> [max]; NaN-free data with
    no mixed +-0 -> numpy.sort(x)[k:] (library special case); the first output
    is select(x, k) (the definition of §IV.I)."""
    x = datagen.make("normal" if np.dtype(dtype).kind == "f" else "int", 3001, dtype, seed=11)
    x = x[x != 0] if np.dtype(dtype).kind == "f" else x
    assert _sorted_bits(oracle.select_upper(x, 0)) == _sorted_bits(x)
    assert oracle.select_upper(x, x.size - 1).tolist() == [np.max(x)]
    for k in (1, x.size // 3, x.size - 2):
        up = oracle.select_upper(x, k)
        assert np.array_equal(up, np.sort(x)[k:])
        assert _bits(up[0]) == _bits(oracle.select(x, k))


# ------------------------------------- multi-rank selection (NEXT-2) ---------
@settings(max_examples=100, deadline=None)
@given(st.lists(st.integers(-3, 3), min_size=1, max_size=40), st.data())
def test_select_multi_bruteforce_tiny(vals, data):
    """Each rank against the O(n^2) count definition and Python's sort."""
    x = np.array(vals, dtype=np.int64)
    ks = data.draw(st.lists(st.integers(0, len(vals) - 1), min_size=1, max_size=8))
    got = oracle.select_multi(x, ks)
    assert got.tolist() == [sorted(vals)[k] for k in ks]
    assert got.tolist() == [int(oracle.select_bruteforce(x, k)) for k in ks]


@pytest.mark.parametrize("dtype", [np.float32, np.float64, np.int32, np.int64])
def test_select_multi_monotone_and_numpy(dtype):
    """Ranks in increasing order give non-decreasing results (totalOrder);
    NaN-free data without mixed +-0 equals numpy.sort indexing; repeats and
    the extremes are allowed."""
    x = datagen.make("normal" if np.dtype(dtype).kind == "f" else "int", 5003, dtype, seed=17)
    x = x[x != 0] if np.dtype(dtype).kind == "f" else x
    ks = [0, 1, 7, 7, x.size // 2, x.size - 1]
    got = oracle.select_multi(x, ks)
    assert np.array_equal(got, np.sort(x)[ks])
    for a, b in zip(got[:-1], got[1:]):
        assert oracle.cmp(a, b, dtype) <= 0
    with pytest.raises(ValueError):
        oracle.select_multi(x, [x.size])


# ---- QuickSelect mirror (reading R24) -------
@settings(max_examples=120, deadline=None)
@given(st.lists(st.integers(-3, 3), min_size=1, max_size=60), st.data())
def test_quickselect_mirror_tiny_duplicates(vals, data):
    """base_case = 0 forces the three-way partition at every level down to a
    single pivot answer: duplicates exercise the == pivot exit."""
    x = np.array(vals, dtype=np.int64)
    k = data.draw(st.integers(0, len(vals) - 1))
    v, sizes = oracle.quickselect(x, k, base_case=0, seed=3)
    assert int(v) == sorted(vals)[k] == int(oracle.select_bruteforce(x, k))
    assert all(a > b for a, b in zip(sizes, sizes[1:]))


@settings(max_examples=80, deadline=None)
@given(st.lists(_f32_special, min_size=1, max_size=30), st.data())
def test_quickselect_mirror_tiny_special_f32(bits, data):
    """-0/+0, NaNs, infinities: the partition uses totalOrder (R3)."""
    x = np.array(bits, dtype=np.uint32).view(np.float32)
    k = data.draw(st.integers(0, len(bits) - 1))
    v, _ = oracle.quickselect(x, k, base_case=0, seed=9)
    assert _bits(v) == _bits(oracle.select_bruteforce(x, k))


@pytest.mark.parametrize("kind,dtype", [("uniform", np.float32), ("distinct16", np.float64),
                                        ("equal", np.int32), ("perm", np.int64)])
def test_quickselect_mirror_level0_counts(kind, dtype):
    """Level 0 keeps exactly #{x < p} (left) or #{x > p} (right) elements
    for the median-of-sample pivot p, and the result is sorted[k]; the
    median-of-sample pivot roughly halves continuous data."""
    n = 3000
    x = datagen.make(kind, n, dtype, seed=4)
    idx = oracle.sample_indices(11, 0, n, 0, oracle.QS_SAMPLE)
    p = oracle.select(x[idx], oracle.QS_SAMPLE // 2)
    L, Le = oracle.count_less(x, p), oracle.count_leq(x, p)
    for k in [0, n // 2, n - 1]:
        v, sizes = oracle.quickselect(x, k, base_case=64, seed=11)
        assert _bits(v) == _bits(oracle.select(x, k))
        assert sizes[0] == n
        if k < L:
            assert sizes[1] == L
        elif k >= Le:
            assert sizes[1] == n - Le
        else:
            assert len(sizes) == 1
    if kind in ("uniform", "perm"):
        assert abs(L - n / 2) < 0.1 * n
