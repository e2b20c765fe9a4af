// Microbenchmark: K2 classify/count with the tree walk vs a prefix-LUT start.
// Not part of the product; used to choose the K2 design.
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o k2lut k2_lut.cu
// Data: 2^28 fp32 keys (order-preserving transform of U[0,1) or N(0,1) floats);
// splitters are the i/b percentiles of a 4096-element sample (as K1 builds).
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdint>
#include <cstring>
#include <random>
#include <vector>
#include <cuda_runtime.h>

typedef unsigned int u32;
typedef unsigned long long u64;
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1);} } while (0)

__device__ __forceinline__ uint4 ldg_stream(const uint4* p) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}
__device__ __forceinline__ u32 cstep(u32 p, u32 key, u32 t) {
    u32 r;
    asm("{ .reg .u32 d; sub.cc.u32 d, %1, %2; addc.u32 %0, %3, %3; }" : "=r"(r) : "r"(key), "r"(t), "r"(p));
    return r;
}
__device__ __forceinline__ u32 to_key(u32 u) { return u ^ ((u32)((int)u >> 31) | 0x80000000u); }

struct LutParams { u32 sh; int base; u32 cells; };

// MODE 0: tree walk (levels 0,1 registers, 2..4 heap, >=5 lane-replicated) [current K2]
// MODE 1: LUT(cells) -> hi, bucket = hi - [key < spl[hi]], flagged cells walk
// MODE 2: LUT + replicated spl (per lane)
// MODE 3: no classification (bucket = key >> 24) -- floor
template <int H, int MODE, int LOGC, int TPB>
__global__ void __launch_bounds__(TPB) k2(const uint4* __restrict__ in, u64 nvec, const u32* __restrict__ tree_g,
    const u32* __restrict__ spl_g, const unsigned short* __restrict__ lut_g, LutParams lp,
    uint8_t* __restrict__ orc, u32* __restrict__ out_counts, u32* flagged) {
    constexpr u32 B = 1u << H;
    constexpr u32 W = TPB / 32;
    constexpr u32 C = 1u << LOGC;
    extern __shared__ __align__(16) u32 sm[];
    u32* tree = sm;                               // B
    constexpr u32 REP_WORDS = (H > 5) ? (((1u << H) - 32u) * 32u) : 0u;
    u32* rep = tree + B;                          // replicated levels (MODE 0 only)
    u32* hist = rep + ((MODE == 0 || MODE == 4 || MODE == 5) ? REP_WORDS : 0);   // W * B
    u32* spl = hist + W * B;                      // B (+ pad) or B*32 replicated
    unsigned short* lut = reinterpret_cast<unsigned short*>(spl + (MODE == 2 ? B * 32 : B));
    const u32 lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (u32 i = threadIdx.x; i < B; i += TPB) tree[i] = (i < B - 1) ? tree_g[i] : 0;
    for (u32 i = threadIdx.x; i < W * B; i += TPB) hist[i] = 0;
    if (MODE == 0 || MODE == 4 || MODE == 5)
        for (u32 d = 5; d < H; ++d)
            for (u32 w = threadIdx.x; w < (1u << d) * 32; w += TPB)
                rep[((1u << d) - 32) * 32 + w] = tree_g[(1u << d) - 1 + (w >> 5)];
    if (MODE == 1) for (u32 i = threadIdx.x; i < B; i += TPB) spl[i] = spl_g[i];
    if (MODE == 2) for (u32 i = threadIdx.x; i < B * 32; i += TPB) spl[i] = spl_g[i >> 5];
    if (MODE == 1 || MODE == 2)
        for (u32 i = threadIdx.x; i < C / 8; i += TPB) reinterpret_cast<uint4*>(lut)[i] = reinterpret_cast<const uint4*>(lut_g)[i];
    __syncthreads();
    const u32 r0 = tree[0], r1 = tree[1], r2 = tree[2];
    // lane-resident splitters for shuffle levels: level l node (lane mod 2^l)
    const u32 s2 = tree[3 + (lane & 3)], s3 = tree[7 + (lane & 7)], s4 = tree[15 + (lane & 15)], s5 = tree[31 + lane];
    const u32 r3 = tree[3], r4 = tree[4], r5 = tree[5], r6 = tree[6];
    u32* my_hist = hist + warp * B;
    const u32 sbase = (u32)__cvta_generic_to_shared(spl) + lane * 4;
    auto walk = [&](u32 key) -> u32 {
        u32 p = cstep(0u, key, r0);
        p = cstep(p, key, p ? r2 : r1);
#pragma unroll
        for (int l = 2; l < H; ++l) {
            u32 t;
            if (MODE == 0 && l >= 5) t = rep[((1u << l) - 32) * 32 + p * 32 + lane];
            else t = tree[(1u << l) - 1 + p];
            p = cstep(p, key, t);
        }
        return p;
    };
    u32 nflag = 0;
    auto classify = [&](u32 key) -> u32 {
        if (MODE == 3) return key >> 24 >> (8 - H);
        if (MODE == 4 || MODE == 5) {
            u32 p = cstep(0u, key, r0);
            p = cstep(p, key, p ? r2 : r1);
            if (MODE == 4) p = cstep(p, key, __shfl_sync(0xffffffffu, s2, p));
            else p = cstep(p, key, (p & 2) ? ((p & 1) ? r6 : r5) : ((p & 1) ? r4 : r3));
            p = cstep(p, key, __shfl_sync(0xffffffffu, s3, p));
            p = cstep(p, key, __shfl_sync(0xffffffffu, s4, p));
            p = cstep(p, key, __shfl_sync(0xffffffffu, s5, p));
#pragma unroll
            for (int l = 6; l < H; ++l) p = cstep(p, key, rep[((1u << l) - 32) * 32 + p * 32 + lane]);
            return p;
        }
        if (MODE == 0) return walk(key);
        int c = (int)(key >> lp.sh) - lp.base;
        c = min(max(c, 0), (int)C - 1);
        u32 e = lut[c];
        if (e & 0x8000u) { ++nflag; return walk(key); }
        u32 t;
        if (MODE == 1) t = spl[e];
        else {
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(t) : "r"(sbase + e * 128));
        }
        return e - (key < t ? 1u : 0u);
    };
    const u64 stride = (u64)gridDim.x * TPB;
    u64 v = (u64)blockIdx.x * TPB + threadIdx.x;
    for (; v + 3 * stride < nvec; v += 4 * stride) {
        uint4 q[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) q[u] = ldg_stream(in + v + u * stride);
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            u32 b0 = classify(to_key(q[u].x)), b1 = classify(to_key(q[u].y));
            u32 b2 = classify(to_key(q[u].z)), b3 = classify(to_key(q[u].w));
            atomicAdd(&my_hist[b0], 1u); atomicAdd(&my_hist[b1], 1u);
            atomicAdd(&my_hist[b2], 1u); atomicAdd(&my_hist[b3], 1u);
            *reinterpret_cast<u32*>(orc + (v + u * stride) * 4) = b0 | (b1 << 8) | (b2 << 16) | (b3 << 24);
        }
    }
    for (; v < nvec; v += stride) {
        uint4 q = ldg_stream(in + v);
        u32 b0 = classify(to_key(q.x)), b1 = classify(to_key(q.y)), b2 = classify(to_key(q.z)), b3 = classify(to_key(q.w));
        atomicAdd(&my_hist[b0], 1u); atomicAdd(&my_hist[b1], 1u);
        atomicAdd(&my_hist[b2], 1u); atomicAdd(&my_hist[b3], 1u);
        *reinterpret_cast<u32*>(orc + v * 4) = b0 | (b1 << 8) | (b2 << 16) | (b3 << 24);
    }
    if (nflag) atomicAdd(flagged, nflag);
    __syncthreads();
    for (u32 j = threadIdx.x; j < B; j += TPB) {
        u32 s = 0;
        for (u32 w = 0; w < W; ++w) s += hist[w * B + j];
        out_counts[blockIdx.x * B + j] = s;
    }
}

__global__ void read_only(const uint4* __restrict__ in, u64 nvec, u32* sink) {
    const u64 stride = (u64)gridDim.x * blockDim.x;
    u32 acc = 0;
    for (u64 v = (u64)blockIdx.x * blockDim.x + threadIdx.x; v < nvec; v += stride) {
        uint4 q = ldg_stream(in + v);
        acc ^= q.x ^ q.y ^ q.z ^ q.w;
    }
    if (acc == 0xdeadbeef) sink[0] = acc;
}

struct Ctx {
    uint4* in; u64 nvec; u32* tree; u32* spl; unsigned short* lut; uint8_t* orc; u32* counts; u32* flag; int sms;
    cudaEvent_t e0, e1;
    std::vector<u64> ref;   // reference bucket totals
    LutParams lp;
};

template <typename F>
float timeit(Ctx& c, F f, int reps = 5) {
    f();
    CK(cudaDeviceSynchronize());
    CK(cudaEventRecord(c.e0));
    for (int r = 0; r < reps; ++r) f();
    CK(cudaEventRecord(c.e1));
    CK(cudaEventSynchronize(c.e1));
    float ms;
    CK(cudaEventElapsedTime(&ms, c.e0, c.e1));
    CK(cudaGetLastError());
    return ms / reps;
}

template <int H, int MODE, int LOGC, int TPB>
void run(Ctx& c, const char* name) {
    constexpr u32 B = 1u << H;
    constexpr u32 REP_WORDS = (H > 5) ? (((1u << H) - 32u) * 32u) : 0u;
    size_t smem = (B + ((MODE == 0 || MODE == 4 || MODE == 5) ? REP_WORDS : 0) + (TPB / 32) * B + (MODE == 2 ? B * 32 : B)) * 4;
    if (MODE == 1 || MODE == 2) smem += (2u << LOGC);
    auto kern = k2<H, MODE, LOGC, TPB>;
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int occ = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, TPB, smem));
    if (occ == 0) { printf("%-36s (does not fit: smem %zu)\n", name, smem); return; }
    int grid = occ * c.sms;
    CK(cudaMemset(c.flag, 0, 4));
    float ms = timeit(c, [&] { kern<<<grid, TPB, smem>>>(c.in, c.nvec, c.tree, c.spl, c.lut, c.lp, c.orc, c.counts, c.flag); });
    u32 nflag = 0;
    CK(cudaMemcpy(&nflag, c.flag, 4, cudaMemcpyDeviceToHost));
    double n = c.nvec * 4.0;
    std::vector<u32> h((size_t)grid * B);
    CK(cudaMemcpy(h.data(), c.counts, h.size() * 4, cudaMemcpyDeviceToHost));
    bool ok = true;
    if (MODE != 3) {
        for (u32 j = 0; j < B; ++j) {
            u64 s = 0;
            for (int g = 0; g < grid; ++g) s += h[(size_t)g * B + j];
            if (s != c.ref[j]) ok = false;
        }
    }
    printf("%-36s occ=%d smem=%6zu %8.1f us %7.1f GB/s(5B/el) %.3e el/s flagged/run=%.4f%% %s\n", name, occ, smem,
           ms * 1e3, n * 5.0 / (ms * 1e-3) / 1e9, n / (ms * 1e-3), 100.0 * nflag / 6.0 / n, ok ? "ok" : "COUNTS WRONG");
}

static u32 key_of(float f) { u32 u; memcpy(&u, &f, 4); return u ^ ((u32)((int)u >> 31) | 0x80000000u); }

void setup(Ctx& c, int H, int LOGC, bool normal, std::vector<u32>& hostkeys, bool regen) {
    const u64 n = c.nvec * 4;
    if (regen) {
        std::mt19937_64 rng(normal ? 7 : 5);
        std::vector<float> x(n);
        std::uniform_real_distribution<float> U(0.f, 1.f);
        std::normal_distribution<float> N(0.f, 1.f);
        for (u64 i = 0; i < n; ++i) x[i] = normal ? N(rng) : U(rng);
        CK(cudaMemcpy(c.in, x.data(), n * 4, cudaMemcpyHostToDevice));
        hostkeys.resize(n);
        for (u64 i = 0; i < n; ++i) hostkeys[i] = key_of(x[i]);
    }
    const u32 b = 1u << H;
    std::mt19937_64 rng(99);
    std::vector<u32> smp(4096);
    for (auto& s : smp) s = hostkeys[rng() % n];
    std::sort(smp.begin(), smp.end());
    std::vector<u32> spl(b + 1), tree(b);
    spl[0] = 0;
    for (u32 i = 1; i < b; ++i) spl[i] = smp[(u64)i * 4096 / b];
    spl[b] = 0xFFFFFFFFu;
    for (int d = 0; d < H; ++d)
        for (u32 p = 0; p < (1u << d); ++p) tree[(1u << d) - 1 + p] = spl[(2 * p + 1) << (H - 1 - d)];
    CK(cudaMemcpy(c.tree, tree.data(), b * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(c.spl, spl.data(), b * 4, cudaMemcpyHostToDevice));
    // LUT over [s_1, s_{b-1}] in key space
    const u32 C = 1u << LOGC;
    u32 sh = 1;
    while (((spl[b - 1] >> sh) - (spl[1] >> sh)) >= C) ++sh;
    int base = (int)(spl[1] >> sh);
    std::vector<unsigned short> lut(C);
    u64 nf = 0;
    for (u32 cc = 0; cc < C; ++cc) {
        u64 start = cc == 0 ? 0 : ((u64)(cc + base) << sh);
        u64 end = cc == C - 1 ? 0xFFFFFFFFull : (((u64)(cc + base + 1) << sh) - 1);
        u32 hi = (u32)(std::upper_bound(spl.begin() + 1, spl.begin() + b, (u32)end) - (spl.begin() + 1));
        u32 lo = (u32)(std::upper_bound(spl.begin() + 1, spl.begin() + b, (u32)start) - (spl.begin() + 1));
        lut[cc] = (unsigned short)(hi | (hi - lo >= 2 ? 0x8000u : 0u));
        nf += hi - lo >= 2;
    }
    CK(cudaMemcpy(c.lut, lut.data(), C * 2, cudaMemcpyHostToDevice));
    c.lp = {sh, base, C};
    c.ref.assign(b, 0);
    for (u64 i = 0; i < n; ++i) {
        u32 k = hostkeys[i];
        c.ref[std::upper_bound(spl.begin() + 1, spl.begin() + b, k) - (spl.begin() + 1)]++;
    }
    printf("-- %s b=%u cells=2^%d sh=%u base=%d flagged cells=%llu\n", normal ? "normal" : "uniform", b, LOGC, sh, base, nf);
}

#define RUN(H, M, LC, T) run<H, M, LC, T>(c, "b=2^" #H " mode=" #M " cells=2^" #LC " tpb=" #T)

int main() {
    Ctx c;
    CK(cudaDeviceGetAttribute(&c.sms, cudaDevAttrMultiProcessorCount, 0));
    const u64 n = 1ull << 28;
    c.nvec = n / 4;
    CK(cudaMalloc(&c.in, n * 4));
    CK(cudaMalloc(&c.orc, n));
    CK(cudaMalloc(&c.tree, 1024 * 4));
    CK(cudaMalloc(&c.spl, 1025 * 4));
    CK(cudaMalloc(&c.lut, 65536 * 2));
    CK(cudaMalloc(&c.counts, 4096 * 1024 * 4));
    CK(cudaMalloc(&c.flag, 64));
    CK(cudaEventCreate(&c.e0));
    CK(cudaEventCreate(&c.e1));
    std::vector<u32> hk;
    float ms = timeit(c, [&] { read_only<<<c.sms * 8, 256>>>(c.in, c.nvec, c.flag); });
    printf("read_only %8.1f us %7.1f GB/s\n", ms * 1e3, n * 4.0 / (ms * 1e-3) / 1e9);
    for (int normal = 0; normal < 2; ++normal) {
        setup(c, 8, 12, normal, hk, true);
        RUN(8, 0, 12, 512);
        RUN(8, 4, 12, 512);
        RUN(8, 5, 12, 512);
        RUN(8, 3, 12, 512);
        RUN(8, 2, 12, 512);
    }
    return 0;
}
