// read_bw.cu -- the read-only HBM ceiling on B200 for the window kernel's
// access pattern (a 1 GiB fp32 stream, every byte read once, almost nothing
// written): 128-bit LDG with D loads in flight per thread vs TMA bulk copies
// (cp.async.bulk) into an S-stage shared-memory ring per CTA.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o read_bw read_bw.cu && ./read_bw
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

typedef unsigned long long u64;
typedef unsigned int u32;

__device__ __forceinline__ uint4 ldg_ef(const uint4* p, u64 pol) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p), "l"(pol));
    return r;
}
__device__ __forceinline__ u64 pol_ef() {
    u64 p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}

// LDG: each warp streams a contiguous run, D vectors per lane in flight
template <int D>
__global__ void __launch_bounds__(1024, 1) ldg_kernel(const uint4* __restrict__ in, u64 nvec, u32* out) {
    const u64 pol = pol_ef();
    const u32 lane = threadIdx.x & 31, warp = threadIdx.x >> 5, NW = blockDim.x >> 5;
    const u64 gw = (u64)blockIdx.x * NW + warp, nw = (u64)gridDim.x * NW;
    const u64 per = (nvec + nw - 1) / nw;
    u64 vb = gw * per, ve = vb + per < nvec ? vb + per : nvec;
    u32 acc = 0;
    uint4 r[D];
    for (; vb + 32 * D <= ve; vb += 32 * D) {
#pragma unroll
        for (int i = 0; i < D; ++i) r[i] = ldg_ef(in + vb + lane + 32 * i, pol);
#pragma unroll
        for (int i = 0; i < D; ++i) acc += (r[i].x < 0x3F000000u) + (r[i].y < 0x3F000000u) + (r[i].z < 0x3F000000u) + (r[i].w < 0x3F000000u);
    }
    for (u64 v = vb + lane; v < ve; v += 32) {
        uint4 q = ldg_ef(in + v, pol);
        acc += (q.x < 0x3F000000u) + (q.w < 0x3F000000u);
    }
    acc = __reduce_add_sync(0xffffffffu, acc);
    if (lane == 0) atomicAdd(out, acc);
}

// TMA ring: thread 0 issues bulk copies of CHUNK bytes into STAGES buffers;
// all threads consume each buffer (LDS.128) and release it by a barrier.
template <int STAGES, int CHUNK>
__global__ void __launch_bounds__(1024, 1) tma_kernel(const char* __restrict__ in, u64 nbytes, u32* out) {
    extern __shared__ __align__(128) unsigned char ring[];
    __shared__ __align__(8) u64 bar[STAGES];
    const u64 pol = pol_ef();
    const u64 nchunks = nbytes / CHUNK;
    const u64 per = (nchunks + gridDim.x - 1) / gridDim.x;
    const u64 c0 = blockIdx.x * per, c1 = c0 + per < nchunks ? c0 + per : nchunks;
    const u32 rb = (u32)__cvta_generic_to_shared(ring), b0 = (u32)__cvta_generic_to_shared(bar);
    auto issue = [&](u64 t) {
        const u32 st = (u32)(t % STAGES);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b0 + st * 8), "r"(CHUNK) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
                     ::"r"(rb + st * CHUNK), "l"(in + (c0 + t) * CHUNK), "r"(CHUNK), "r"(b0 + st * 8), "l"(pol) : "memory");
    };
    if (threadIdx.x == 0) {
        for (int i = 0; i < STAGES; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b0 + i * 8));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (u64 t = 0; t < STAGES && c0 + t < c1; ++t) issue(t);
    }
    __syncthreads();
    u32 acc = 0;
    for (u64 t = 0; c0 + t < c1; ++t) {
        const u32 st = (u32)(t % STAGES), ph = (u32)((t / STAGES) & 1);
        u32 ok;
        do {
            asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                         : "=r"(ok) : "r"(b0 + st * 8), "r"(ph) : "memory");
        } while (!ok);
        for (u32 o = threadIdx.x * 16; o < CHUNK; o += blockDim.x * 16) {
            uint4 q;
            asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(q.x), "=r"(q.y), "=r"(q.z), "=r"(q.w) : "r"(rb + st * CHUNK + o));
            acc += (q.x < 0x3F000000u) + (q.y < 0x3F000000u) + (q.z < 0x3F000000u) + (q.w < 0x3F000000u);
        }
        __syncthreads();
        if (threadIdx.x == 0 && c0 + t + STAGES < c1) issue(t + STAGES);
    }
    acc = __reduce_add_sync(0xffffffffu, acc);
    if ((threadIdx.x & 31) == 0) atomicAdd(out, acc);
}

template <typename F>
float timeit(F f, int reps = 20) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    f();
    cudaDeviceSynchronize();
    float best = 1e9;
    for (int r = 0; r < reps; ++r) {
        cudaEventRecord(a);
        f();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        best = ms < best ? ms : best;
    }
    return best;
}

int main() {
    const u64 n = 1ull << 28, bytes = n * 4;
    char* d;
    u32* out;
    cudaMalloc(&d, bytes);
    cudaMalloc(&out, 4);
    cudaMemset(d, 0x3e, bytes);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const u64 nvec = bytes / 16;
    auto rep = [&](const char* name, float ms) {
        printf("%-28s %8.1f us  %7.1f GB/s\n", name, ms * 1e3, bytes / (ms * 1e-3) / 1e9);
    };
    rep("ldg D=4", timeit([&] { ldg_kernel<4><<<sms, 1024>>>((const uint4*)d, nvec, out); }));
    rep("ldg D=8", timeit([&] { ldg_kernel<8><<<sms, 1024>>>((const uint4*)d, nvec, out); }));
    rep("ldg D=16", timeit([&] { ldg_kernel<16><<<sms, 1024>>>((const uint4*)d, nvec, out); }));
    rep("ldg D=8 2x grid 512thr", timeit([&] { ldg_kernel<8><<<2 * sms, 512>>>((const uint4*)d, nvec, out); }));
#define TMA(S, C)                                                                                     \
    {                                                                                                 \
        cudaFuncSetAttribute(tma_kernel<S, C>, cudaFuncAttributeMaxDynamicSharedMemorySize, S * C);   \
        rep("tma " #S "x" #C, timeit([&] { tma_kernel<S, C><<<sms, 1024, S * C>>>(d, bytes, out); }));   \
    }
    TMA(4, 16384) TMA(8, 16384) TMA(4, 32768) TMA(6, 32768) TMA(3, 65536) TMA(12, 16384)
    cudaError_t e = cudaGetLastError();
    printf("%s\n", cudaGetErrorString(e));
    return 0;
}
