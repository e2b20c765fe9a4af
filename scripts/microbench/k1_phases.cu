// Microbenchmark: in-kernel cycle counts of the one-CTA building blocks
// (sample sort, tree build, base-case radix select).  Not part of the product.
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a --expt-relaxed-constexpr \
//        -I../../include -I../../paper_conf_ipps_ribizela19_b200/csrc -o k1p k1_phases.cu
#include <cstdio>
#include <vector>
#include <random>
#include "kernels.cuh"
using namespace ss;
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1);} } while (0)

template <int MODE>
__global__ void __launch_bounds__(1024) probe(const u32* __restrict__ src, u32 s, int reps, long long* cyc, u32* out,
                                              const float* data, u64 n) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    u32* keys = reinterpret_cast<u32*>(smem_raw);
    __shared__ u32 spl_s[MAX_B];
    __shared__ u32 hist[32 * 256];
    __shared__ u32 misc[16];
    __shared__ u32 red[64];
    __syncthreads();
    long long t0 = clock64();
    u32 acc = 0;
    for (int r = 0; r < reps; ++r) {
        if (MODE == 0) {          // sort only (keys from global, L2-resident)
            block_sort_keys<u32>(keys, s, [&](u32 j) { return src[j] ^ (u32)r; });
        } else if (MODE == 1) {   // gather random samples only
            const u64 base = level_base(0x5A17 + r, 0);
            for (u32 j = threadIdx.x; j < s; j += blockDim.x) keys[j] = load_key(data + sample_index(base, j, n));
            __syncthreads();
        } else if (MODE == 2) {   // gather + sort + tree (= K1)
            const u64 base = level_base(0x5A17 + r, 0);
            block_sort_keys<u32>(keys, s, [&](u32 j) { return load_key(data + sample_index(base, j, n)); });
            block_build_tree<u32>(keys, s, 256, 1, spl_s, out, out + 1024, (uint8_t*)(out + 2048));
            __syncthreads();
        } else if (MODE == 3) {   // base case radix select of s keys
            u32 v = block_radix_select<float>(data + r, s, s / 2, hist, misc, red);
            acc += v;
            __syncthreads();
        }
        acc += keys[threadIdx.x % s];
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) { cyc[0] = t1 - t0; }
    if (acc == 0x12345) out[0] = acc;
}

template <int MODE>
void run(const char* name, u32 s, const u32* src, const float* data, u64 n, long long* cyc, u32* out) {
    CK(cudaFuncSetAttribute(probe<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536));
    const int reps = 20;
    probe<MODE><<<1, 1024, 65536>>>(src, s, reps, cyc, out, data, n);
    CK(cudaDeviceSynchronize());
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a);
    probe<MODE><<<1, 1024, 65536>>>(src, s, reps, cyc, out, data, n);
    cudaEventRecord(b);
    CK(cudaDeviceSynchronize());
    float ms; cudaEventElapsedTime(&ms, a, b);
    long long c; CK(cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost));
    printf("%-28s s=%5u: %8.0f cycles/rep  (%.2f us/rep at 1.965 GHz; kernel %.1f us for %d reps)\n", name, s,
           (double)c / reps, (double)c / reps / 1965.0, ms * 1e3, reps);
}

int main() {
    const u64 n = 1ull << 28;
    float* data; CK(cudaMalloc(&data, n * 4));
    std::vector<float> h(1 << 20);
    std::mt19937 rng(1);
    std::uniform_real_distribution<float> U(0, 1);
    for (auto& x : h) x = U(rng);
    for (u64 o = 0; o < n; o += h.size()) CK(cudaMemcpy(data + o, h.data(), h.size() * 4, cudaMemcpyHostToDevice));
    u32* src; CK(cudaMalloc(&src, 16384 * 4));
    std::vector<u32> hs(16384);
    for (auto& x : hs) x = rng();
    CK(cudaMemcpy(src, hs.data(), hs.size() * 4, cudaMemcpyHostToDevice));
    long long* cyc; CK(cudaMalloc(&cyc, 64));
    u32* out; CK(cudaMalloc(&out, 4096 * 4));
    for (u32 s : {1024u, 4096u, 16384u}) {
        run<0>("sort only", s, src, data, n, cyc, out);
        run<1>("gather only (2^28 src)", s, src, data, n, cyc, out);
        run<2>("gather+sort+tree (2^28)", s, src, data, n, cyc, out);
        run<2>("gather+sort+tree (2^20)", s, src, data, 1u << 20, cyc, out);
    }
    for (u32 s : {1024u, 3712u, 16384u}) run<3>("base radix select (U[0,1))", s, src, data, n, cyc, out);
    // narrow range: values 0.5 + [0, 1e-4)
    for (auto& x : h) x = 0.5f + 1e-4f * U(rng);
    CK(cudaMemcpy(data, h.data(), h.size() * 4, cudaMemcpyHostToDevice));
    for (u32 s : {1024u, 3712u, 15000u, 16384u}) run<3>("base radix select (narrow)", s, src, data, n, cyc, out);
    return 0;
}
