// sanitize_driver.cu -- drives every kernel of libsampleselect.so through the
// C ABI at small sizes, for compute-sanitizer (memcheck / racecheck /
// synccheck / initcheck) runs without Python in the process:
//   nvcc -O2 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I include \
//        -o build/sanitize_driver scripts/sanitize_driver.cu \
//        -Lpaper_conf_ipps_ribizela19_b200 -lsampleselect -Xlinker -rpath=$PWD/paper_conf_ipps_ribizela19_b200
//   compute-sanitizer --tool memcheck build/sanitize_driver
// Every exact result is also compared with a sort of the host copy
// (std::nth_element on the order-preserving keys); exit code != 0 on a mismatch.
// compute-sanitizer is closed on the GPU pool (it refuses to run), so the
// driver checks memory itself: every device buffer it hands the library sits
// between two 256-byte guard bands filled with 0xA5 and checked after the
// calls (an out-of-bounds write shows as a changed guard byte), the input is
// compared with its host copy afterwards (no call may write it), and the
// top-k output is compared, as a sorted multiset, with the host's.
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <thread>
#include <vector>
#include <cuda_runtime.h>
#include "sampleselect.h"

static int g_fail = 0;
#define CHECK(x)                                                                            \
    do {                                                                                    \
        ss_status s_ = (x);                                                                 \
        if (s_) {                                                                           \
            std::printf("FAIL %s:%d %s -> %s\n", __FILE__, __LINE__, #x, ss_status_string(s_)); \
            ++g_fail;                                                                       \
        }                                                                                   \
    } while (0)

template <typename T> uint64_t key_of(T v) {
    if (sizeof(T) == 4) {
        uint32_t u;
        std::memcpy(&u, &v, 4);
        if (std::is_floating_point<T>::value) return (u >> 31) ? ~u : (u | 0x80000000u);
        return u ^ 0x80000000u;
    }
    uint64_t u;
    std::memcpy(&u, &v, 8);
    if (std::is_floating_point<T>::value) return (u >> 63) ? ~u : (u | 0x8000000000000000ull);
    return u ^ 0x8000000000000000ull;
}

template <typename T> T ref_select(const std::vector<T>& x, int64_t k) {
    std::vector<uint64_t> keys(x.size());
    for (size_t i = 0; i < x.size(); ++i) keys[i] = key_of(x[i]) << 0;
    std::vector<size_t> idx(x.size());
    for (size_t i = 0; i < idx.size(); ++i) idx[i] = i;
    std::nth_element(idx.begin(), idx.begin() + k, idx.end(), [&](size_t a, size_t b) { return keys[a] < keys[b]; });
    return x[idx[k]];
}

template <typename T> std::vector<T> make(size_t n, int kind, unsigned seed) {
    std::mt19937_64 g(seed);
    std::vector<T> x(n);
    for (size_t i = 0; i < n; ++i) {
        if (kind == 0) x[i] = (T)(std::uniform_real_distribution<double>(-1e6, 1e6)(g));
        else x[i] = (T)(g() % 16);                    // 16 distinct values
    }
    return x;
}

// device buffer of `bytes` between two guard bands
constexpr size_t GUARD = 256;
struct Guarded {
    unsigned char* base = nullptr;
    size_t bytes = 0;
    const char* name = "";
    void* ptr() const { return base + GUARD; }
};
static std::vector<Guarded> g_bufs;
static void* galloc(size_t bytes, const char* name) {
    Guarded gb;
    gb.bytes = bytes;
    gb.name = name;
    cudaMalloc(&gb.base, bytes + 2 * GUARD);
    cudaMemset(gb.base, 0xA5, bytes + 2 * GUARD);
    g_bufs.push_back(gb);
    return gb.ptr();
}
static void gcheck_free() {
    cudaDeviceSynchronize();
    for (const Guarded& gb : g_bufs) {
        std::vector<unsigned char> h(2 * GUARD);
        cudaMemcpy(h.data(), gb.base, GUARD, cudaMemcpyDeviceToHost);
        cudaMemcpy(h.data() + GUARD, gb.base + GUARD + gb.bytes, GUARD, cudaMemcpyDeviceToHost);
        for (size_t i = 0; i < h.size(); ++i)
            if (h[i] != 0xA5) {
                std::printf("GUARD %s: byte %s%zu changed\n", gb.name, i < GUARD ? "-" : "+",
                            i < GUARD ? GUARD - i : i - GUARD);
                ++g_fail;
                break;
            }
        cudaFree(gb.base);
    }
    g_bufs.clear();
}

template <typename T> ss_dtype dt_of() {
    if (std::is_same<T, float>::value) return SS_FLOAT32;
    if (std::is_same<T, double>::value) return SS_FLOAT64;
    if (std::is_same<T, int32_t>::value) return SS_INT32;
    return SS_INT64;
}

template <typename T> void run_dtype(ss_context* ctx, size_t n, int kind) {
    const ss_dtype dt = dt_of<T>();
    std::vector<T> x = make<T>(n, kind, (unsigned)(n * 7 + kind));
    T* d = (T*)galloc((n + 4) * sizeof(T), "input");
    cudaMemcpy(d + 1, x.data(), n * sizeof(T), cudaMemcpyHostToDevice);   // misaligned view: d + 1
    const int64_t ks[] = {0, (int64_t)n / 2, (int64_t)n - 1, (int64_t)n / 3};
    for (int fused = 0; fused < 2; ++fused) {
        ss_config cfg;
        ss_get_config(ctx, &cfg);
        cfg.fused_filter = fused;
        cfg.spec_min_n = 1 << 14;
        ss_set_config(ctx, &cfg);
        for (int64_t k : ks) {
            T v;
            CHECK(ss_select(ctx, dt, d + 1, (int64_t)n, k, &v, nullptr));
            if (key_of(v) != key_of(ref_select(x, k))) {
                std::printf("MISMATCH select n=%zu k=%lld fused=%d\n", n, (long long)k, fused);
                ++g_fail;
            }
        }
    }
    T v;
    int64_t r;
    for (int b : {64, 1024}) CHECK(ss_approx_select(ctx, dt, d + 1, (int64_t)n, (int64_t)n / 2, b, &v, &r, nullptr));
    // top-k: the output buffer is exactly n - k elements (both paths: one pass and two passes)
    for (int64_t m : {(int64_t)std::min<size_t>(1000, n), (int64_t)n / 3}) {
        for (int onep = 0; onep < 2; ++onep) {
            ss_config cfg;
            ss_get_config(ctx, &cfg);
            cfg.upper_onepass = onep;
            ss_set_config(ctx, &cfg);
            T* up = (T*)galloc((size_t)m * sizeof(T), "select_upper out");
            CHECK(ss_select_upper(ctx, dt, d + 1, (int64_t)n, (int64_t)n - m, up, &v, nullptr));
            std::vector<T> got((size_t)m);
            cudaMemcpy(got.data(), up, (size_t)m * sizeof(T), cudaMemcpyDeviceToHost);
            std::vector<uint64_t> gk(got.size()), rk;
            for (size_t i = 0; i < got.size(); ++i) gk[i] = key_of(got[i]);
            for (const T& e : x) rk.push_back(key_of(e));
            std::sort(gk.begin(), gk.end());
            std::sort(rk.begin(), rk.end());
            if (!std::equal(gk.begin(), gk.end(), rk.end() - m)) {
                std::printf("MISMATCH select_upper n=%zu m=%lld onepass=%d\n", n, (long long)m, onep);
                ++g_fail;
            }
        }
    }
    T* out = (T*)galloc(n * sizeof(T), "filter out");
    std::vector<int64_t> mk = {1, (int64_t)n / 5, (int64_t)n / 2, (int64_t)n - 2, 7, (int64_t)n / 3};
    std::vector<T> mv(mk.size());
    CHECK(ss_select_multi(ctx, dt, d + 1, (int64_t)n, (int32_t)mk.size(), mk.data(), mv.data(), nullptr));
    for (size_t i = 0; i < mk.size(); ++i)
        if (key_of(mv[i]) != key_of(ref_select(x, mk[i]))) {
            std::printf("MISMATCH select_multi n=%zu k=%lld\n", n, (long long)mk[i]);
            ++g_fail;
        }
    int64_t nl[64];
    int32_t lv;
    CHECK(ss_quickselect(ctx, dt, d + 1, (int64_t)n, (int64_t)n / 2, &v, nl, 64, &lv, nullptr));
    // steps: sample -> tree -> count (+ oracle bytes) -> filter -> search; ablation modes
    const int s = 4096, b = 256;
    void* keys = galloc(s * sizeof(T), "sample keys");
    void* tree = galloc((b - 1) * sizeof(T), "tree");
    void* spl = galloc((b - 1) * sizeof(T), "splitters");
    uint8_t* eq = (uint8_t*)galloc(b, "eq flags");
    void* tot = galloc(b * 8, "totals");
    void* orc = galloc(n + 16, "oracle bytes");
    void* srch = galloc(32, "search row");
    CHECK(ss_step_sample(ctx, dt, d + 1, (int64_t)n, 0, 0, s, keys, nullptr));
    CHECK(ss_step_tree(ctx, dt, keys, s, b, 1, tree, spl, eq, nullptr));
    CHECK(ss_step_count(ctx, dt, d + 1, (int64_t)n, tree, b, (uint64_t*)tot, (uint8_t*)orc, nullptr));
    uint64_t* cnt = (uint64_t*)galloc(8, "filter count");
    CHECK(ss_step_filter(ctx, dt, d + 1, (int64_t)n, (uint8_t*)orc, 3, out, cnt, nullptr));
    CHECK(ss_step_search(ctx, (uint64_t*)tot, b, (int64_t)n / 2, eq, (int64_t*)srch, nullptr));
    for (int mode = 0; mode < 5; ++mode)
        CHECK(ss_step_count_ablation(ctx, dt, d + 1, (int64_t)n, tree, b, mode, (uint64_t*)tot, nullptr));
    CHECK(ss_step_keys_to_values(ctx, dt, spl, b - 1, spl, nullptr));
    cudaDeviceSynchronize();
    std::vector<T> after(n);
    cudaMemcpy(after.data(), d + 1, n * sizeof(T), cudaMemcpyDeviceToHost);
    if (std::memcmp(after.data(), x.data(), n * sizeof(T))) {
        std::printf("INPUT WRITTEN n=%zu\n", n);
        ++g_fail;
    }
    gcheck_free();
}

// the sharded path on two virtual ranks (one host thread + context each)
template <typename T> void run_sharded(size_t n) {
    ss_local_group* g = nullptr;
    CHECK(ss_local_group_create(2, &g));
    std::vector<T> x0 = make<T>(n, 0, 11), x1 = make<T>(n / 3, 0, 12);
    std::vector<T> all(x0);
    all.insert(all.end(), x1.begin(), x1.end());
    const int64_t k = (int64_t)all.size() / 2;
    const T ref = ref_select(all, k);
    auto worker = [&](int r) {
        ss_context* c = nullptr;
        if (ss_create(0, &c)) { ++g_fail; return; }
        ss_config cfg;
        ss_get_config(c, &cfg);
        cfg.shard_gather_log2 = 12;
        ss_set_config(c, &cfg);
        CHECK(ss_comm_init_local(c, g, r));
        const std::vector<T>& x = r ? x1 : x0;
        T* d = nullptr;
        cudaMalloc(&d, x.size() * sizeof(T));
        cudaMemcpy(d, x.data(), x.size() * sizeof(T), cudaMemcpyHostToDevice);
        cudaStream_t st;
        cudaStreamCreate(&st);
        T v;
        CHECK(ss_select_sharded(c, dt_of<T>(), d, (int64_t)x.size(), k, &v, st));
        if (key_of(v) != key_of(ref)) { std::printf("MISMATCH sharded rank %d\n", r); ++g_fail; }
        cudaStreamDestroy(st);
        cudaFree(d);
        ss_destroy(c);
    };
    std::thread t0(worker, 0), t1(worker, 1);
    t0.join();
    t1.join();
    ss_local_group_destroy(g);
}

int main(int argc, char** argv) {
    const size_t n = argc > 1 ? (size_t)std::atoll(argv[1]) : (size_t)(1 << 16) + 5;
    ss_context* ctx = nullptr;
    if (ss_create(0, &ctx)) { std::printf("no device\n"); return 2; }
    for (int kind = 0; kind < 2; ++kind) {
        run_dtype<float>(ctx, n, kind);
        run_dtype<double>(ctx, n, kind);
        run_dtype<int32_t>(ctx, n, kind);
        run_dtype<int64_t>(ctx, n, kind);
    }
    run_dtype<float>(ctx, 1000, 0);       // base case only
    ss_destroy(ctx);
    run_sharded<float>(n);
    run_sharded<int64_t>(n);
    std::printf("sanitize_driver: %s (%d failures)\n", g_fail ? "FAILED" : "ok", g_fail);
    return g_fail ? 1 : 0;
}
