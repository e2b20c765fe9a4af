// Microbenchmark of classify/count inner-loop designs for K2 on B200.
// Not part of the product; used to choose the K2 design.
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o k2v k2_variants.cu
// Data: 2^28 u32 keys uniform over the full range (1 GiB > L2), splitters
// s_i = i * 2^32 / b (equiprobable buckets).
#include <cstdio>
#include <cstdint>
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

// WALK 0: heap tree in smem, Fig. 4 walk.
// WALK 1: levels 0,1 in registers, rest in smem heap.
// WALK 2: levels 0,1 in registers, levels 2..4 smem heap, levels >= 5 lane-replicated.
// WALK 3: no walk (bucket = key >> (32-H)) -- isolates histogram/oracle cost.
// HIST 0: none; 1: ATOMS on one CTA histogram; 2: packed u8 per-lane counters
//          [bucket/4][lane] with periodic warp-reduce flush; 3: per-lane u32 [bucket][lane] (b<=128).
template <int H, int WALK, int HIST, bool ORC, int TPB>
__global__ void __launch_bounds__(TPB) k2(const uint4* __restrict__ in, u64 nvec, const u32* __restrict__ tree_g,
                                          uint8_t* __restrict__ orc, u32* __restrict__ out_counts, u32* sink) {
    constexpr u32 B = 1u << H;
    extern __shared__ u32 sm[];
    u32* tree = sm;                         // B words (heap)
    u32* rep = sm + B;                      // replicated levels >= 5: sum_{d>=5} 2^d * 32 words
    constexpr u32 REP_WORDS = (H > 5) ? (((1u << H) - 32u) * 32u) : 0u;
    u32* hist = rep + REP_WORDS;            // B words
    u32* lanec = hist + B;                  // per-lane counters
    const u32 lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (u32 i = threadIdx.x; i < B; i += TPB) { tree[i] = (i < B - 1) ? tree_g[i] : 0; hist[i] = 0; }
    if (WALK == 2 || WALK == 5) {
        for (u32 d = 5; d < H; ++d)
            for (u32 w = threadIdx.x; w < (1u << d) * 32; w += TPB) {
                u32 node = w >> 5;
                u32 off = ((1u << d) - 32) * 32;  // sum_{e=5}^{d-1} 2^e*32
                rep[off + w] = tree_g[(1u << d) - 1 + node];
            }
    }
    if (HIST == 2) for (u32 w = threadIdx.x; w < (B / 4) * TPB; w += TPB) lanec[w] = 0;
    if (HIST == 3) for (u32 w = threadIdx.x; w < B * TPB; w += TPB) lanec[w] = 0;
    __syncthreads();
    const u32 r0 = tree[0], r1 = tree[1], r2 = tree[2];
    u32* my_lanec2 = lanec + warp * (B / 4) * 32 + lane;
    u32* my_lanec3 = lanec + warp * B * 32 + lane;
    u32 acc = 0;

    const u32 d12 = r2 - r1;
    const u32 lane4 = lane * 4;
    auto cstep = [](u32 p, u32 key, u32 t) -> u32 {
        u32 r;
        asm("{ .reg .u32 d; sub.cc.u32 d, %1, %2; addc.u32 %0, %3, %3; }" : "=r"(r) : "r"(key), "r"(t), "r"(p));
        return r;
    };
    auto classify = [&](u32 key) -> u32 {
        if (WALK == 3) return key >> (32 - H);
        if (WALK >= 4) {
            u32 p = 0;
            int l = 0;
            if (WALK != 6) {
                p = cstep(0u, key, r0);
                p = cstep(p, key, r1 + p * d12);
                l = 2;
            }
#pragma unroll
            for (; l < H; ++l) {
                u32 t;
                if (WALK == 5 && l >= 5) {
                    const u32 off = ((1u << l) - 32) * 32;
                    t = *reinterpret_cast<const u32*>(reinterpret_cast<const char*>(rep + off) + p * 128 + lane4);
                } else {
                    t = tree[(1u << l) - 1 + p];
                }
                p = cstep(p, key, t);
            }
            return p;
        }
        u32 i;
        int l0;
        if (WALK == 0) { i = 0; l0 = 0; }
        else {
            u32 c0 = key >= r0;
            u32 t1 = c0 ? r2 : r1;
            u32 c1 = key >= t1;
            i = 3 + 2 * c0 + c1;
            l0 = 2;
        }
        if (WALK == 2) {
#pragma unroll
            for (int l = l0; l < H && l < 5; ++l) i = 2 * i + 1 + (key >= tree[i] ? 1u : 0u);
            if (H > 5) {
                u32 node = i - 31;   // position within level 5
#pragma unroll
                for (int d = 5; d < H; ++d) {
                    const u32 off = ((1u << d) - 32) * 32;
                    u32 t = rep[off + node * 32 + lane];
                    node = 2 * node + (key >= t ? 1u : 0u);
                }
                return node;  // position at level H = bucket
            }
            return i - (B - 1);
        } else {
#pragma unroll
            for (int l = l0; l < H; ++l) i = 2 * i + 1 + (key >= tree[i] ? 1u : 0u);
            return i - (B - 1);
        }
    };
    auto count = [&](u32 bk) {
        if (HIST == 0) acc ^= bk;
        if (HIST == 1) atomicAdd(&hist[bk], 1u);
        if (HIST == 2) { u32* p = my_lanec2 + (bk >> 2) * 32; *p += 1u << ((bk & 3) << 3); }
        if (HIST == 3) { u32* p = my_lanec3 + bk * 32; *p += 1u; }
    };
    auto flush2 = [&]() {
        __syncwarp();
        for (u32 q = 0; q < B / 4; ++q) {
            u32 w = my_lanec2[q * 32];
            my_lanec2[q * 32] = 0;
            u32 lo = __reduce_add_sync(0xffffffffu, w & 0x00FF00FFu);
            u32 hi = __reduce_add_sync(0xffffffffu, (w >> 8) & 0x00FF00FFu);
            if (lane == 0) {
                atomicAdd(&hist[4 * q + 0], lo & 0xFFFF);
                atomicAdd(&hist[4 * q + 2], lo >> 16);
                atomicAdd(&hist[4 * q + 1], hi & 0xFFFF);
                atomicAdd(&hist[4 * q + 3], hi >> 16);
            }
        }
        __syncwarp();
    };
    const u64 stride = (u64)gridDim.x * TPB;
    u64 v = (u64)blockIdx.x * TPB + threadIdx.x;
    int it = 0;
    for (; v + 3 * stride < nvec; v += 4 * stride) {
        uint4 q[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) q[u] = ldg_stream(in + v + u * stride);
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            u32 b0 = classify(q[u].x), b1 = classify(q[u].y), b2 = classify(q[u].z), b3 = classify(q[u].w);
            count(b0); count(b1); count(b2); count(b3);
            if (ORC) *reinterpret_cast<u32*>(orc + (v + u * stride) * 4) = b0 | (b1 << 8) | (b2 << 16) | (b3 << 24);
        }
        if (HIST == 2 && ++it == 15) { it = 0; flush2(); }
    }
    for (; v < nvec; v += stride) {
        uint4 q = ldg_stream(in + v);
        u32 b0 = classify(q.x), b1 = classify(q.y), b2 = classify(q.z), b3 = classify(q.w);
        count(b0); count(b1); count(b2); count(b3);
        if (ORC) *reinterpret_cast<u32*>(orc + v * 4) = b0 | (b1 << 8) | (b2 << 16) | (b3 << 24);
    }
    if (HIST == 2) flush2();
    if (HIST == 3) {
        __syncwarp();
        for (u32 bk = 0; bk < B; ++bk) {
            u32 s = __reduce_add_sync(0xffffffffu, my_lanec3[bk * 32]);
            if (lane == 0) atomicAdd(&hist[bk], s);
        }
    }
    __syncthreads();
    for (u32 i = threadIdx.x; i < B; i += TPB) out_counts[blockIdx.x * B + i] = hist[i];
    if (HIST == 0 && acc == 0xdeadbeef) sink[0] = acc;
}

// plain streaming baselines
__global__ void read_only(const uint4* __restrict__ in, u64 nvec, u32* sink) {
    const u64 stride = (u64)gridDim.x * blockDim.x;
    u32 acc = 0;
    for (u64 v = (u64)blockIdx.x * blockDim.x + threadIdx.x; v < nvec; v += stride) {
        uint4 q = ldg_stream(in + v);
        acc ^= q.x ^ q.y ^ q.z ^ q.w;
    }
    if (acc == 0xdeadbeef) sink[0] = acc;
}
__global__ void read_write_bytes(const uint4* __restrict__ in, u64 nvec, uint8_t* orc) {
    const u64 stride = (u64)gridDim.x * blockDim.x;
    for (u64 v = (u64)blockIdx.x * blockDim.x + threadIdx.x; v < nvec; v += stride) {
        uint4 q = ldg_stream(in + v);
        *reinterpret_cast<u32*>(orc + v * 4) = (q.x >> 24) | ((q.y >> 24) << 8) | ((q.z >> 24) << 16) | (q.w & 0xFF000000u);
    }
}

struct Ctx {
    uint4* in; u64 nvec; u32* tree; uint8_t* orc; u32* counts; u32* sink; int sms;
    cudaEvent_t e0, e1;
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

template <int H, int WALK, int HIST, bool ORC, int TPB>
void run(Ctx& c, const char* name) {
    constexpr u32 B = 1u << H;
    constexpr u32 REP_WORDS = (H > 5) ? (((1u << H) - 32u) * 32u) : 0u;
    size_t smem = (B + REP_WORDS + B) * 4;
    if (HIST == 2) smem += (size_t)(B / 4) * TPB * 4;
    if (HIST == 3) smem += (size_t)B * TPB * 4;
    auto kern = k2<H, WALK, HIST, ORC, TPB>;
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int occ = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, TPB, smem));
    if (occ == 0) { printf("%-44s b=%4u  (does not fit: smem %zu)\n", name, B, smem); return; }
    int grid = occ * c.sms;
    float ms = timeit(c, [&] { kern<<<grid, TPB, smem>>>(c.in, c.nvec, c.tree, c.orc, c.counts, c.sink); });
    double n = c.nvec * 4.0;
    double bytes = n * (4 + (ORC ? 1 : 0));
    // verify counts (HIST != 0): equiprobable buckets sum to n
    if (HIST) {
        std::vector<u32> h((size_t)grid * B);
        CK(cudaMemcpy(h.data(), c.counts, h.size() * 4, cudaMemcpyDeviceToHost));
        u64 tot = 0;
        for (auto x : h) tot += x;
        if (tot != (u64)n) printf("  !! count mismatch %llu vs %.0f\n", tot, n);
    }
    printf("%-44s b=%4u occ=%d grid=%5d smem=%6zu  %8.1f us  %7.1f GB/s  %.3e el/s\n", name, B, occ, grid, smem,
           ms * 1e3, bytes / (ms * 1e-3) / 1e9, n / (ms * 1e-3));
}

#define RUNH(H, W, HI, O, T) run<H, W, HI, O, T>(c, "walk=" #W " hist=" #HI " orc=" #O " tpb=" #T)

int main() {
    Ctx c;
    CK(cudaDeviceGetAttribute(&c.sms, cudaDevAttrMultiProcessorCount, 0));
    const u64 n = 1ull << 28;
    c.nvec = n / 4;
    CK(cudaMalloc(&c.in, n * 4));
    CK(cudaMalloc(&c.orc, n));
    CK(cudaMalloc(&c.tree, 1024 * 4));
    CK(cudaMalloc(&c.counts, 4096 * 1024 * 4));
    CK(cudaMalloc(&c.sink, 64));
    CK(cudaEventCreate(&c.e0));
    CK(cudaEventCreate(&c.e1));
    {   // random keys
        std::vector<u32> h(n);
        u64 s = 0x12345;
        for (u64 i = 0; i < n; ++i) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; h[i] = (u32)(s >> 16); }
        CK(cudaMemcpy(c.in, h.data(), n * 4, cudaMemcpyHostToDevice));
    }
    auto set_tree = [&](int H) {
        u32 b = 1u << H;
        std::vector<u32> spl(b), tree(b);
        for (u32 i = 1; i < b; ++i) spl[i] = (u32)(((u64)i << 32) / b);
        for (int d = 0; d < H; ++d)
            for (u32 p = 0; p < (1u << d); ++p) tree[(1u << d) - 1 + p] = spl[(2 * p + 1) << (H - 1 - d)];
        CK(cudaMemcpy(c.tree, tree.data(), b * 4, cudaMemcpyHostToDevice));
    };
    int sms = c.sms;
    float ms = timeit(c, [&] { read_only<<<sms * 8, 256>>>(c.in, c.nvec, c.sink); });
    printf("read_only                 %8.1f us  %7.1f GB/s\n", ms * 1e3, n * 4.0 / (ms * 1e-3) / 1e9);
    ms = timeit(c, [&] { read_write_bytes<<<sms * 8, 256>>>(c.in, c.nvec, c.orc); });
    printf("read+oracle write         %8.1f us  %7.1f GB/s\n", ms * 1e3, n * 5.0 / (ms * 1e-3) / 1e9);

    set_tree(8);
    RUNH(8, 4, 1, true, 256);
    RUNH(8, 5, 1, true, 256);
    RUNH(8, 6, 1, true, 256);
    RUNH(8, 5, 1, true, 512);
    RUNH(8, 5, 0, true, 256);
    set_tree(7);
    RUNH(7, 4, 1, true, 256);
    RUNH(7, 5, 1, true, 256);
    RUNH(7, 6, 1, true, 256);
    set_tree(6);
    RUNH(6, 4, 1, true, 256);
    RUNH(6, 5, 1, true, 256);
    RUNH(6, 6, 1, true, 256);
    set_tree(10);
    RUNH(10, 4, 1, false, 256);
    RUNH(10, 6, 1, false, 256);
    RUNH(10, 5, 1, false, 512);
    set_tree(8);
    RUNH(8, 3, 0, true, 256);
    RUNH(8, 3, 1, true, 256);
    RUNH(8, 3, 2, true, 256);
    RUNH(8, 0, 0, true, 256);
    RUNH(8, 1, 0, true, 256);
    RUNH(8, 2, 0, true, 256);
    RUNH(8, 0, 1, true, 512);
    RUNH(8, 0, 1, true, 256);
    RUNH(8, 1, 1, true, 256);
    RUNH(8, 2, 1, true, 256);
    RUNH(8, 1, 2, true, 256);
    RUNH(8, 2, 2, true, 256);
    RUNH(8, 2, 2, true, 128);
    set_tree(7);
    RUNH(7, 3, 1, true, 256);
    RUNH(7, 3, 3, true, 128);
    RUNH(7, 0, 1, true, 256);
    RUNH(7, 1, 1, true, 256);
    RUNH(7, 2, 1, true, 256);
    RUNH(7, 1, 2, true, 256);
    RUNH(7, 2, 2, true, 256);
    RUNH(7, 2, 3, true, 128);
    set_tree(6);
    RUNH(6, 3, 1, true, 256);
    RUNH(6, 3, 3, true, 256);
    RUNH(6, 0, 1, true, 256);
    RUNH(6, 1, 1, true, 256);
    RUNH(6, 2, 1, true, 256);
    RUNH(6, 1, 2, true, 256);
    RUNH(6, 1, 3, true, 256);
    RUNH(6, 2, 3, true, 256);
    set_tree(10);
    RUNH(10, 3, 1, false, 256);
    RUNH(10, 0, 1, false, 256);
    RUNH(10, 1, 1, false, 256);
    RUNH(10, 2, 1, false, 256);
    return 0;
}
