/*
 * oracle.c -- CPU TEST ORACLE for SampleSelect (Ribizel & Anzt, "Approximate
 * and Exact Selection on GPUs", IPDPS-W 2019; /root/reference/PAPER.md).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  It
 * shares no code, header, table or constant generator with the CUDA path in
 * paper_conf_ipps_ribizela19_b200/csrc/, and includes nothing from it.
 *
 * Precision: selection is comparison-only (§III: "purely
 * comparison-based"), so there is no rounding anywhere; every function below is
 * exact.  Floating-point values are ordered by IEEE-754 totalOrder (DESIGN.md
 * reading R3: -NaN < -inf < ... < -0 < +0 < ... < +inf < +NaN), integers
 * numerically.
 *
 * Functions and the passage each follows:
 *   oracle_cmp                  totalOrder / numeric order         (R3; L82-85)
 *   oracle_select               sort-and-index: the plain definition of
 *                               "the element at position k in the sorted
 *                               sequence" (§II)
 *   oracle_select_bruteforce    O(n^2): the unique v with
 *                               #{x < v} <= k < #{x <= v}          (§II)
 *   oracle_count_less / _leq    #{x_i < v}, #{x_i <= v}: "smallest rank" (L86-88)
 *   oracle_splitmix64, oracle_sample_indices
 *                               counter-based sampling with replacement
 *                               (§II.B, reading R7)
 *   oracle_pick_splitters       sort sample, take the i/b percentiles
 *                               (§IV.B-a, reading R8)
 *   oracle_equality_fixup       equality buckets (§IV.C, reading R9)
 *   oracle_heap_tree            implicit complete BST, heap indexing
 *                               (§IV.B-b, Fig. 3)
 *   oracle_tree_bucket          Fig. 4 walk i = 2i + (x < tree[i] ? 1 : 2)
 *                               (Fig. 4)
 *   oracle_count_buckets        bucket sizes n_i                    (§II.A)
 *   oracle_filter_bucket        extract one bucket, input order     (§IV.B-c)
 *   oracle_approx_select        approximate selection: splitter whose rank
 *                               r_i is closest to k (§II.C, §V.G)
 *   oracle_select_upper         top-k fusion: the kth-smallest element and
 *                               "all larger elements" = positions k..n-1 of
 *                               the sorted sequence (§IV.I, reading R22)
 *   oracle_select_multi         m ranks: the elements at positions k_1..k_m of
 *                               the sorted sequence (reading R23)
 *   oracle_select_upper_bruteforce
 *                               O(n^2): value v appears #{x<=v} - max(#{x<v}, k)
 *                               times among ranks >= k (§IV.I, §II)
 *
 * Parity pins (tests/test_oracle.py, -m "not gpu"): hand-worked examples
 * (tests/golden/), min/max special cases, numpy.partition on NaN-free data,
 * the permutation closed form, d-distinct closed form, the count invariant,
 * O(n^2) brute force, the SplitMix64 published test vector, the Fig. 4 worked
 * tree example and #{splitters <= x}.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

enum { OR_F32 = 0, OR_F64 = 1, OR_I32 = 2, OR_I64 = 3 };
enum { OR_OK = 0, OR_EINVAL = 1, OR_ENOMEM = 3 };

static size_t elem_size(int dt) {
    switch (dt) {
    case OR_F32: case OR_I32: return 4;
    case OR_F64: case OR_I64: return 8;
    default: return 0;
    }
}

/* ---------------------------------------------------------------------------
 * Ordering (reading R3).  Written from the IEEE-754 totalOrder definition:
 * sign first (negative before positive), then magnitude, larger magnitude
 * first among negatives.  NaNs sort by sign and payload like any other bit
 * pattern.  Deliberately sign/magnitude logic, not an integer key transform.
 * ------------------------------------------------------------------------- */
static int cmp_f32_bits(uint32_t a, uint32_t b) {
    unsigned sa = a >> 31, sb = b >> 31;
    uint32_t ma = a & 0x7FFFFFFFu, mb = b & 0x7FFFFFFFu;
    if (sa != sb) return sa ? -1 : 1;          /* negative < positive */
    if (ma == mb) return 0;
    if (sa == 0) return ma < mb ? -1 : 1;      /* both positive */
    return ma > mb ? -1 : 1;                   /* both negative */
}
static int cmp_f64_bits(uint64_t a, uint64_t b) {
    unsigned sa = (unsigned)(a >> 63), sb = (unsigned)(b >> 63);
    uint64_t ma = a & 0x7FFFFFFFFFFFFFFFull, mb = b & 0x7FFFFFFFFFFFFFFFull;
    if (sa != sb) return sa ? -1 : 1;
    if (ma == mb) return 0;
    if (sa == 0) return ma < mb ? -1 : 1;
    return ma > mb ? -1 : 1;
}

int oracle_cmp(int dt, const void* a, const void* b) {
    switch (dt) {
    case OR_F32: { uint32_t x, y; memcpy(&x, a, 4); memcpy(&y, b, 4); return cmp_f32_bits(x, y); }
    case OR_F64: { uint64_t x, y; memcpy(&x, a, 8); memcpy(&y, b, 8); return cmp_f64_bits(x, y); }
    case OR_I32: { int32_t x, y; memcpy(&x, a, 4); memcpy(&y, b, 4); return (x > y) - (x < y); }
    case OR_I64: { int64_t x, y; memcpy(&x, a, 8); memcpy(&y, b, 8); return (x > y) - (x < y); }
    default: return 0;
    }
}

static int q_f32(const void* a, const void* b) { return oracle_cmp(OR_F32, a, b); }
static int q_f64(const void* a, const void* b) { return oracle_cmp(OR_F64, a, b); }
static int q_i32(const void* a, const void* b) { return oracle_cmp(OR_I32, a, b); }
static int q_i64(const void* a, const void* b) { return oracle_cmp(OR_I64, a, b); }

static void sort_copy(int dt, void* buf, int64_t n) {
    int (*f)(const void*, const void*) =
        dt == OR_F32 ? q_f32 : dt == OR_F64 ? q_f64 : dt == OR_I32 ? q_i32 : q_i64;
    qsort(buf, (size_t)n, elem_size(dt), f);
}

/* §II: the element at position k (0-based) of the sorted sequence. */
int oracle_select(int dt, const void* data, int64_t n, int64_t k, void* out) {
    size_t S = elem_size(dt);
    if (!S || !data || !out || n < 1 || k < 0 || k >= n) return OR_EINVAL;
    char* buf = (char*)malloc((size_t)n * S);
    if (!buf) return OR_ENOMEM;
    memcpy(buf, data, (size_t)n * S);
    sort_copy(dt, buf, n);
    memcpy(out, buf + (size_t)k * S, S);
    free(buf);
    return OR_OK;
}

/* #{x_i < v} and #{x_i <= v} under the order above (L86-88 "smallest rank"). */
int64_t oracle_count_less(int dt, const void* data, int64_t n, const void* v) {
    size_t S = elem_size(dt);
    const char* p = (const char*)data;
    int64_t c = 0;
    for (int64_t i = 0; i < n; ++i) c += oracle_cmp(dt, p + (size_t)i * S, v) < 0;
    return c;
}
int64_t oracle_count_leq(int dt, const void* data, int64_t n, const void* v) {
    size_t S = elem_size(dt);
    const char* p = (const char*)data;
    int64_t c = 0;
    for (int64_t i = 0; i < n; ++i) c += oracle_cmp(dt, p + (size_t)i * S, v) <= 0;
    return c;
}

/* §II L82-88 written as a count: the unique v (bitwise) among the inputs with
 * #{x < v} <= k < #{x <= v}.  O(n^2); for tiny inputs only. */
int oracle_select_bruteforce(int dt, const void* data, int64_t n, int64_t k, void* out) {
    size_t S = elem_size(dt);
    if (!S || !data || !out || n < 1 || k < 0 || k >= n) return OR_EINVAL;
    const char* p = (const char*)data;
    for (int64_t i = 0; i < n; ++i) {
        const void* v = p + (size_t)i * S;
        int64_t lt = oracle_count_less(dt, data, n, v);
        int64_t le = oracle_count_leq(dt, data, n, v);
        if (lt <= k && k < le) { memcpy(out, v, S); return OR_OK; }
    }
    return OR_EINVAL; /* unreachable for a valid k */
}

/* §IV.I: "not only the kth-smallest element is required, but also
 * all larger elements" -- positions k..n-1 of the sorted sequence, written to
 * out[0..n-k) in ascending order. */
int oracle_select_upper(int dt, const void* data, int64_t n, int64_t k, void* out) {
    size_t S = elem_size(dt);
    if (!S || !data || !out || n < 1 || k < 0 || k >= n) return OR_EINVAL;
    char* buf = (char*)malloc((size_t)n * S);
    if (!buf) return OR_ENOMEM;
    memcpy(buf, data, (size_t)n * S);
    sort_copy(dt, buf, n);
    memcpy(out, buf + (size_t)k * S, (size_t)(n - k) * S);
    free(buf);
    return OR_OK;
}

/* Reading R23 (§VI): m ranks -- the definition of
 * §II L82-88 applied to each k_i; one sort, m indexings. */
int oracle_select_multi(int dt, const void* data, int64_t n, int32_t m, const int64_t* ks, void* out) {
    size_t S = elem_size(dt);
    if (!S || !data || !out || !ks || n < 1 || m < 1) return OR_EINVAL;
    for (int32_t i = 0; i < m; ++i)
        if (ks[i] < 0 || ks[i] >= n) return OR_EINVAL;
    char* buf = (char*)malloc((size_t)n * S);
    if (!buf) return OR_ENOMEM;
    memcpy(buf, data, (size_t)n * S);
    sort_copy(dt, buf, n);
    for (int32_t i = 0; i < m; ++i) memcpy((char*)out + (size_t)i * S, buf + (size_t)ks[i] * S, S);
    free(buf);
    return OR_OK;
}

/* The same multiset by counting, O(n^2): the copies of a value v occupy the
 * ranks #{x<v} .. #{x<=v}-1 (L86-88), so #{x<=v} - max(#{x<v}, k) of them (if
 * positive) have rank >= k.  Each distinct value (first occurrence) is emitted
 * that many times, in input order of first occurrence.  Returns the count. */
int64_t oracle_select_upper_bruteforce(int dt, const void* data, int64_t n, int64_t k, void* out) {
    size_t S = elem_size(dt);
    if (!S || !data || !out || n < 1 || k < 0 || k >= n) return -1;
    const char* p = (const char*)data;
    char* o = (char*)out;
    int64_t w = 0;
    for (int64_t i = 0; i < n; ++i) {
        const void* v = p + (size_t)i * S;
        int seen = 0;
        for (int64_t j = 0; j < i && !seen; ++j) seen = oracle_cmp(dt, p + (size_t)j * S, v) == 0;
        if (seen) continue;
        int64_t lt = oracle_count_less(dt, data, n, v);
        int64_t le = oracle_count_leq(dt, data, n, v);
        int64_t m = le - (lt > k ? lt : k);
        for (int64_t c = 0; c < m; ++c) memcpy(o + (size_t)(w++) * S, v, S);
    }
    return w;
}

/* ---------------------------------------------------------------------------
 * Sampling (§II.B, reading R7).  Sampling with replacement, uniform
 * indices.  Counter-based: every draw is a pure function of (seed, level,
 * global slot j), so the sample is reproducible and shardable.
 *   base_l = splitmix64(seed + level * 0xD1B54A32D192ED03)
 *   u_j    = splitmix64(base_l + j)
 *   idx_j  = floor(u_j * n / 2^64)              (128-bit multiply-high)
 * SplitMix64 (Steele, Lea, Flood 2014) is the published finaliser; pinned by
 * its published test vector in tests/test_oracle.py.
 * ------------------------------------------------------------------------- */
uint64_t oracle_splitmix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/* Indices for sample slots [j0, j0 + cnt) at `level` from a set of n elements. */
void oracle_sample_indices(uint64_t seed, int level, int64_t n, int64_t j0, int64_t cnt,
                           int64_t* idx_out) {
    uint64_t base = oracle_splitmix64(seed + (uint64_t)level * 0xD1B54A32D192ED03ull);
    for (int64_t j = 0; j < cnt; ++j) {
        uint64_t u = oracle_splitmix64(base + (uint64_t)(j0 + j));
        idx_out[j] = (int64_t)(((unsigned __int128)u * (uint64_t)n) >> 64);
    }
}

/* §IV.B-a: sort the sample, pick the i/b percentiles, i = 1..b-1.
 * Reading R8: splitter_i = sorted_sample[floor(i * s / b)].
 * splitters_out has b-1 entries; splitters_out[i-1] = s_i. */
int oracle_pick_splitters(int dt, const void* sample, int64_t s, int b, void* splitters_out) {
    size_t S = elem_size(dt);
    if (!S || s < 1 || b < 2) return OR_EINVAL;
    char* buf = (char*)malloc((size_t)s * S);
    if (!buf) return OR_ENOMEM;
    memcpy(buf, sample, (size_t)s * S);
    sort_copy(dt, buf, s);
    for (int i = 1; i < b; ++i) {
        int64_t pos = (int64_t)(((__int128)i * s) / b);
        memcpy((char*)splitters_out + (size_t)(i - 1) * S, buf + (size_t)pos * S, S);
    }
    free(buf);
    return OR_OK;
}

/* totalOrder successor of a value (the "+ epsilon" of §IV.C, reading
 * R9).  Returns 0 if v is the largest value of its type (no successor). */
static int successor(int dt, const void* v, void* out) {
    switch (dt) {
    case OR_F32: {
        uint32_t x; memcpy(&x, v, 4);
        if (x == 0x7FFFFFFFu) return 0;               /* +NaN, max payload: the maximum */
        if (x >> 31) { x = (x == 0x80000000u) ? 0x00000000u : x - 1; } /* negative: toward -0, then +0 */
        else x = x + 1;                               /* positive: next bit pattern */
        memcpy(out, &x, 4); return 1;
    }
    case OR_F64: {
        uint64_t x; memcpy(&x, v, 8);
        if (x == 0x7FFFFFFFFFFFFFFFull) return 0;
        if (x >> 63) { x = (x == 0x8000000000000000ull) ? 0ull : x - 1; }
        else x = x + 1;
        memcpy(out, &x, 8); return 1;
    }
    case OR_I32: { int32_t x; memcpy(&x, v, 4); if (x == INT32_MAX) return 0; ++x; memcpy(out, &x, 4); return 1; }
    case OR_I64: { int64_t x; memcpy(&x, v, 8); if (x == INT64_MAX) return 0; ++x; memcpy(out, &x, 8); return 1; }
    default: return 0;
    }
}

/* §IV.C L346-357 (reading R9): for each maximal run of equal splitters
 * s_a = ... = s_e = v with a < e, replace s_e by succ(v); bucket e-1 = [v, succ v)
 * then holds exactly the copies of v and is flagged as an equality bucket.
 * If v has no successor, bucket b-1 = [v, inf) is flagged instead.
 * splitters[i-1] = s_i (i = 1..b-1), modified in place; eq_out has b bytes. */
int oracle_equality_fixup(int dt, void* splitters, int b, uint8_t* eq_out) {
    size_t S = elem_size(dt);
    if (!S || b < 2) return OR_EINVAL;
    char* sp = (char*)splitters;
    memset(eq_out, 0, (size_t)b);
    int i = 1;
    while (i < b) {
        int e = i;  /* run [a=i, e] of equal original values */
        while (e + 1 < b && oracle_cmp(dt, sp + (size_t)e * S, sp + (size_t)(i - 1) * S) == 0) ++e;
        if (e > i) {
            void* se = sp + (size_t)(e - 1) * S;
            unsigned char tmp[8];
            if (successor(dt, se, tmp)) { memcpy(se, tmp, S); eq_out[e - 1] = 1; }
            else eq_out[b - 1] = 1;
        }
        i = e + 1;
    }
    return OR_OK;
}

/* §IV.B-b, Fig. 3: complete binary search tree stored implicitly,
 * node i has children 2i+1, 2i+2.  With b = 2^h buckets and sorted splitters
 * s_1..s_{b-1}, the node at depth d, position p (index 2^d - 1 + p) holds
 * s_{(2p+1) * 2^(h-1-d)}, so an in-order traversal yields the sorted order. */
int oracle_heap_tree(int dt, const void* splitters, int b, void* tree_out) {
    size_t S = elem_size(dt);
    int h = 0;
    while ((1 << h) < b) ++h;
    if (!S || b < 2 || (1 << h) != b) return OR_EINVAL;
    for (int d = 0; d < h; ++d)
        for (int p = 0; p < (1 << d); ++p) {
            int i1 = (2 * p + 1) << (h - 1 - d);  /* 1-based splitter index */
            memcpy((char*)tree_out + (size_t)((1 << d) - 1 + p) * S,
                   (const char*)splitters + (size_t)(i1 - 1) * S, S);
        }
    return OR_OK;
}

/* Fig. 4: i = 0; for each level i = 2i + (x < tree[i] ? 1 : 2);
 * bucket = i - (tree_width - 1), tree_width = b. */
int oracle_tree_bucket(int dt, const void* tree, int b, const void* x) {
    size_t S = elem_size(dt);
    int h = 0;
    while ((1 << h) < b) ++h;
    int i = 0;
    for (int l = 0; l < h; ++l)
        i = 2 * i + (oracle_cmp(dt, x, (const char*)tree + (size_t)i * S) < 0 ? 1 : 2);
    return i - (b - 1);
}

/* §II.A: n_i = number of elements in bucket i (Fig. 4 line 7). */
int oracle_count_buckets(int dt, const void* data, int64_t n, const void* tree, int b,
                         int64_t* counts_out, uint8_t* oracles_out /* may be NULL */) {
    size_t S = elem_size(dt);
    if (!S) return OR_EINVAL;
    for (int j = 0; j < b; ++j) counts_out[j] = 0;
    for (int64_t i = 0; i < n; ++i) {
        int bk = oracle_tree_bucket(dt, tree, b, (const char*)data + (size_t)i * S);
        counts_out[bk]++;
        if (oracles_out) oracles_out[i] = (uint8_t)bk; /* Fig. 4 line 8 */
    }
    return OR_OK;
}

/* §IV.B-c: extract the elements of one bucket, contiguously, in
 * input order (reading R15: stable compaction).  Returns the count. */
int64_t oracle_filter_bucket(int dt, const void* data, int64_t n, const uint8_t* oracles,
                             int bucket, void* out) {
    size_t S = elem_size(dt);
    int64_t m = 0;
    for (int64_t i = 0; i < n; ++i)
        if (oracles[i] == (uint8_t)bucket) {
            memcpy((char*)out + (size_t)m * S, (const char*)data + (size_t)i * S, S);
            ++m;
        }
    return m;
}

/* §II.C, §V.G L888-893 (readings R11, R12): one level; after the
 * count the splitter ranks r_i are known; return the splitter s_i whose rank
 * r_i = #{x < s_i} is closest to k (ties: smaller i) and its exact rank.
 * Candidates are the original splitters (no equality fix-up: there is no
 * filter or recursion).  Sample: s slots drawn with replacement at level 0.
 * The ranks come from a sorted copy of the data and a lower-bound search
 * (a library sort as a step; the GPU computes them as bucket prefix sums). */
int oracle_approx_select(int dt, const void* data, int64_t n, int64_t k, int b, int64_t s,
                         uint64_t seed, void* out, int64_t* rank_out, int64_t* index_out) {
    size_t S = elem_size(dt);
    if (!S || !data || n < 1 || k < 0 || k >= n || b < 2 || s < 1) return OR_EINVAL;
    int64_t* idx = (int64_t*)malloc((size_t)s * sizeof(int64_t));
    char* sample = (char*)malloc((size_t)s * S);
    char* spl = (char*)malloc((size_t)(b - 1) * S);
    char* sorted = (char*)malloc((size_t)n * S);
    if (!idx || !sample || !spl || !sorted) { free(idx); free(sample); free(spl); free(sorted); return OR_ENOMEM; }
    oracle_sample_indices(seed, 0, n, 0, s, idx);
    for (int64_t j = 0; j < s; ++j) memcpy(sample + (size_t)j * S, (const char*)data + (size_t)idx[j] * S, S);
    oracle_pick_splitters(dt, sample, s, b, spl);
    memcpy(sorted, data, (size_t)n * S);
    sort_copy(dt, sorted, n);
    int best = -1;
    int64_t best_err = 0, best_rank = 0;
    for (int i = 1; i < b; ++i) {
        const void* si = spl + (size_t)(i - 1) * S;
        /* r_i = #{x < s_i}: first position in the sorted copy not below s_i */
        int64_t lo = 0, hi = n;
        while (lo < hi) {
            int64_t mid = lo + (hi - lo) / 2;
            if (oracle_cmp(dt, sorted + (size_t)mid * S, si) < 0) lo = mid + 1; else hi = mid;
        }
        int64_t err = lo > k ? lo - k : k - lo;
        if (best < 0 || err < best_err) { best = i; best_err = err; best_rank = lo; }
    }
    memcpy(out, spl + (size_t)(best - 1) * S, S);
    if (rank_out) *rank_out = best_rank;
    if (index_out) *index_out = best;
    free(idx); free(sample); free(spl); free(sorted);
    return OR_OK;
}

/* One SampleSelect level followed by recursion, exactly as Fig. 1 L95-127
 * (with reading R6: the bucket holding rank k is the unique j with
 * r_j <= k < r_{j+1}).  A slow mirror of the method used to pin the method
 * itself against oracle_select (same answer) and to report the level sizes.
 * levels_out[l] = n_l for each level entered; returns the number of levels. */
int oracle_sampleselect(int dt, const void* data, int64_t n, int64_t k, int b, int64_t s,
                        int64_t base_case, uint64_t seed, void* out,
                        int64_t* levels_out, int max_levels) {
    size_t S = elem_size(dt);
    if (!S || n < 1 || k < 0 || k >= n || b < 4 || b > 256 || s < 1) return -OR_EINVAL;
    char* cur = (char*)malloc((size_t)n * S);
    char* nxt = (char*)malloc((size_t)n * S);
    uint8_t* orc = (uint8_t*)malloc((size_t)n);
    int64_t* idx = (int64_t*)malloc((size_t)s * sizeof(int64_t));
    char* sample = (char*)malloc((size_t)s * S);
    char* spl = (char*)malloc((size_t)(b - 1) * S);
    char* tree = (char*)malloc((size_t)(b - 1) * S);
    int64_t* counts = (int64_t*)malloc((size_t)b * sizeof(int64_t));
    uint8_t* eq = (uint8_t*)malloc((size_t)b);
    int lv = 0;
    memcpy(cur, data, (size_t)n * S);
    for (;;) {
        if (lv < max_levels && levels_out) levels_out[lv] = n;
        if (n <= base_case) {                              /* Fig. 1 lines 2-5 */
            sort_copy(dt, cur, n);
            memcpy(out, cur + (size_t)k * S, S);
            ++lv;
            break;
        }
        oracle_sample_indices(seed, lv, n, 0, s, idx);    /* line 7 */
        for (int64_t j = 0; j < s; ++j) memcpy(sample + (size_t)j * S, cur + (size_t)idx[j] * S, S);
        oracle_pick_splitters(dt, sample, s, b, spl);
        oracle_equality_fixup(dt, spl, b, eq);
        oracle_heap_tree(dt, spl, b, tree);
        oracle_count_buckets(dt, cur, n, tree, b, counts, orc);   /* line 9 */
        int64_t r = 0; int j = 0;                                 /* lines 11-13 */
        while (!(r <= k && k < r + counts[j])) { r += counts[j]; ++j; }
        ++lv;
        if (eq[j]) {                                       /* §IV.C early exit */
            /* lower-bound splitter of bucket j: the original value v */
            const char* lower = spl + (size_t)(j - 1) * S;
            memcpy(out, lower, S);
            break;
        }
        n = oracle_filter_bucket(dt, cur, n, orc, j, nxt); /* line 15 */
        k -= r;                                            /* line 16 */
        char* t = cur; cur = nxt; nxt = t;
    }
    free(cur); free(nxt); free(orc); free(idx); free(sample); free(spl); free(tree); free(counts); free(eq);
    return lv;
}
