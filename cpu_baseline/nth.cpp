// cpu_baseline/nth.cpp -- the CPU baselines bench.py reports next to the GPU
// (BASELINE.md "CPU baseline plan"): std::nth_element on one
// core -- the paper's own correctness reference (§IV.H) --
// and libstdc++'s parallel-mode __gnu_parallel::nth_element on all host cores.
// Not part of the product path and not the test oracle (oracle/): a timing
// helper only.  Each repetition restores the input first (nth_element
// permutes it); only the nth_element call is timed.
#include <parallel/algorithm>
#include <algorithm>
#include <chrono>
#include <cstdint>
#include <cstring>
#include <vector>
#include <omp.h>

namespace {
template <typename T>
double run(const T* x, int64_t n, int64_t k, int parallel, int reps, T* out) {
    std::vector<T> w((size_t)n);
    double best = 1e300;
    for (int r = 0; r < reps; ++r) {
        std::memcpy(w.data(), x, sizeof(T) * (size_t)n);
        const auto t0 = std::chrono::steady_clock::now();
        if (parallel)
            __gnu_parallel::nth_element(w.begin(), w.begin() + k, w.end());
        else
            std::nth_element(w.begin(), w.begin() + k, w.end());
        const double s = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
        best = s < best ? s : best;
        *out = w[(size_t)k];
    }
    return best;
}
}  // namespace

extern "C" {
// dtype 0: float32, 1: float64.  Returns the best wall time (s) of `reps`
// repetitions; *out receives element k (for a NaN-free input without mixed
// signed zeros: the exact select's answer).
double cpu_nth_element(int dtype, const void* x, int64_t n, int64_t k, int parallel, int reps, void* out) {
    if (dtype == 0) return run((const float*)x, n, k, parallel, reps, (float*)out);
    return run((const double*)x, n, k, parallel, reps, (double*)out);
}
int cpu_threads(void) { return omp_get_max_threads(); }
}
