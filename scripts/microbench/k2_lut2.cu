// Microbenchmark: K2 classify/count design space on B200 (not part of the product).
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o k2lut2 k2_lut2.cu
// Classifiers (CLS):
//   0 tree walk as in K2 (levels 0,1 registers, 2..5 warp shuffles, >= 6 lane-replicated smem)
//   1 cell LUT: c = min((max(key, base) - base) >> sh, C-1); m = lut8[c];
//     bucket = m + [key >= R[m]] (R[m] = s_{m+1}); marker m = b-1 (R = 0) -> bucket b -> tree walk
//   2 as 1 with R replicated per lane (R[m*32 + lane]: conflict-free)
//   3 floor: bucket = key >> (32 - H) (no classification)
// Histograms (HIST): 0 per-warp [W][B]; 1 one per CTA laid out [B][32 lanes] (conflict-free);
//   2 none.
// Data: 2^28 fp32 keys of U[0,1) / N(0,1) / 16 distinct values; splitters = percentiles of a
// 4096 sample (b = 256).  Totals are checked against CLS 0 / HIST 0.
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
__device__ __forceinline__ u32 cadd(u32 m, u32 key, u32 t) {   // m + [key >= t]
    u32 r;
    asm("{ .reg .u32 d; sub.cc.u32 d, %1, %2; addc.u32 %0, %3, 0; }" : "=r"(r) : "r"(key), "r"(t), "r"(m));
    return r;
}
__device__ __forceinline__ u32 to_key(u32 u) { return u ^ ((u32)((int)u >> 31) | 0x80000000u); }

struct LutParams { u32 base, sh, dmax; };

template <int H, int CLS, int HIST, int LOGC, int TPB>
__global__ void __launch_bounds__(TPB) k2(const uint4* __restrict__ in, u64 nvec, const u32* __restrict__ tree_g,
    const u32* __restrict__ R_g, const uint8_t* __restrict__ lut_g, LutParams lp,
    uint8_t* __restrict__ orc, u32* __restrict__ out_counts, u32* flagged) {
    constexpr u32 B = 1u << H;
    constexpr u32 W = TPB / 32;
    constexpr u32 C = 1u << LOGC;
    constexpr bool LUT = CLS == 1 || CLS == 2;
    extern __shared__ __align__(16) u32 sm[];
    u32* tree = sm;                                              // B
    constexpr u32 REP_WORDS = (H > 6) ? (((1u << H) - 64u) * 32u) : 0u;   // levels 6.. replicated
    u32* rep = tree + B;
    u32* hist = rep + REP_WORDS;                                 // W*B or B*32
    constexpr u32 HW = HIST == 0 ? W * B : (HIST == 1 ? B * 32 : 0);
    u32* R = hist + HW;                                          // B or B*32
    constexpr u32 RW = CLS == 1 ? B : (CLS == 2 ? B * 32 : 0);
    uint8_t* lut = reinterpret_cast<uint8_t*>(R + RW);           // C bytes
    const u32 lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (u32 i = threadIdx.x; i < B; i += TPB) tree[i] = (i < B - 1) ? tree_g[i] : 0;
    for (u32 i = threadIdx.x; i < HW; i += TPB) hist[i] = 0;
    for (u32 d = 6; d < H; ++d)
        for (u32 w = threadIdx.x; w < (1u << d) * 32; w += TPB) rep[((1u << d) - 64) * 32 + w] = tree_g[(1u << d) - 1 + (w >> 5)];
    if (CLS == 1) for (u32 i = threadIdx.x; i < B; i += TPB) R[i] = R_g[i];
    if (CLS == 2) for (u32 i = threadIdx.x; i < B * 32; i += TPB) R[i] = R_g[i >> 5];
    if (LUT) for (u32 i = threadIdx.x; i < C / 16; i += TPB) reinterpret_cast<uint4*>(lut)[i] = reinterpret_cast<const uint4*>(lut_g)[i];
    __syncthreads();
    const u32 r0 = tree[0], r1 = tree[1], r2 = tree[2];
    const u32 s2 = tree[3 + (lane & 3)], s3 = tree[7 + (lane & 7)], s4 = tree[15 + (lane & 15)], s5 = tree[31 + lane];
    auto walk_div = [&](u32 key) -> u32 {     // divergence-safe walk (no shuffles)
        u32 p = cstep(0u, key, r0);
        p = cstep(p, key, p ? r2 : r1);
#pragma unroll
        for (int l = 2; l < H; ++l) p = cstep(p, key, tree[(1u << l) - 1 + p]);
        return p;
    };
    auto walk_w = [&](u32 key) -> u32 {       // warp-uniform walk
        u32 p = cstep(0u, key, r0);
        p = cstep(p, key, p ? r2 : r1);
        p = cstep(p, key, __shfl_sync(0xffffffffu, s2, p));
        p = cstep(p, key, __shfl_sync(0xffffffffu, s3, p));
        p = cstep(p, key, __shfl_sync(0xffffffffu, s4, p));
        p = cstep(p, key, __shfl_sync(0xffffffffu, s5, p));
#pragma unroll
        for (int l = 6; l < H; ++l) p = cstep(p, key, rep[((1u << l) - 64) * 32 + p * 32 + lane]);
        return p;
    };
    const u32 rbase = (u32)__cvta_generic_to_shared(R) + (CLS == 2 ? lane * 4 : 0);
    const u32 lbase = (u32)__cvta_generic_to_shared(lut);
    u32 nflag = 0;
    auto lut_cls = [&](u32 key) -> u32 {
        u32 d = min(max(key, lp.base) - lp.base, lp.dmax);
        u32 c = d >> lp.sh;
        u32 m;
        asm volatile("ld.shared.u8 %0, [%1];" : "=r"(m) : "r"(lbase + c));
        u32 t;
        asm volatile("ld.shared.u32 %0, [%1];" : "=r"(t) : "r"(rbase + m * (CLS == 2 ? 128u : 4u)));
        return cadd(m, key, t);
    };
    u32* my_hist = HIST == 0 ? hist + warp * B : hist + lane;
    auto count = [&](u32 bk) {
        if (HIST == 0) atomicAdd(&my_hist[bk], 1u);
        if (HIST == 1) atomicAdd(&my_hist[bk * 32], 1u);
    };
    auto quad = [&](uint4 q, u32* o) {
        u32 k0 = to_key(q.x), k1 = to_key(q.y), k2 = to_key(q.z), k3 = to_key(q.w);
        u32 b0, b1, b2, b3;
        if (CLS == 0) { b0 = walk_w(k0); b1 = walk_w(k1); b2 = walk_w(k2); b3 = walk_w(k3); }
        else if (CLS == 3) { b0 = k0 >> (32 - H); b1 = k1 >> (32 - H); b2 = k2 >> (32 - H); b3 = k3 >> (32 - H); }
        else {
            b0 = lut_cls(k0); b1 = lut_cls(k1); b2 = lut_cls(k2); b3 = lut_cls(k3);
            if ((b0 | b1 | b2 | b3) & B) {    // rare: a cell with >= 2 boundaries
                ++nflag;
                if (b0 >= B) b0 = walk_div(k0);
                if (b1 >= B) b1 = walk_div(k1);
                if (b2 >= B) b2 = walk_div(k2);
                if (b3 >= B) b3 = walk_div(k3);
            }
        }
        count(b0); count(b1); count(b2); count(b3);
        *o = __byte_perm(__byte_perm(b0, b1, 0x0040), __byte_perm(b2, b3, 0x0040), 0x5410);
    };
    // per-warp contiguous chunk, 4 vectors per lane in flight
    const u64 units = (u64)gridDim.x * W;
    const u64 unit = (u64)blockIdx.x * W + warp;
    const u64 per = ((nvec + units - 1) / units + 127) / 128 * 128;
    u64 vb = unit * per, ve = min(vb + per, nvec);
    u32* ow = reinterpret_cast<u32*>(orc);
    if (vb + 128 <= ve) {
        uint4 n0 = ldg_stream(in + vb + lane), n1 = ldg_stream(in + vb + 32 + lane);
        uint4 n2 = ldg_stream(in + vb + 64 + lane), n3 = ldg_stream(in + vb + 96 + lane);
        for (;;) {
            const uint4 a0 = n0, a1 = n1, a2 = n2, a3 = n3;
            u32* o = ow + vb + lane;
            vb += 128;
            const bool more = vb + 128 <= ve;
            if (more) {
                n0 = ldg_stream(in + vb + lane); n1 = ldg_stream(in + vb + 32 + lane);
                n2 = ldg_stream(in + vb + 64 + lane); n3 = ldg_stream(in + vb + 96 + lane);
            }
            quad(a0, o); quad(a1, o + 32); quad(a2, o + 64); quad(a3, o + 96);
            if (!more) break;
        }
    }
    for (; vb < ve; vb += 32) {   // (nvec is a multiple of 32 here)
        quad(ldg_stream(in + vb + lane), ow + vb + lane);
    }
    if (nflag) atomicAdd(flagged, nflag);
    __syncthreads();
    for (u32 j = threadIdx.x; j < B; j += TPB) {
        u32 s = 0;
        if (HIST == 0) for (u32 w = 0; w < W; ++w) s += hist[w * B + j];
        if (HIST == 1) for (u32 l = 0; l < 32; ++l) s += hist[j * 32 + ((l + j) & 31)];
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
__global__ void read_write(const uint4* __restrict__ in, u64 nvec, u32* __restrict__ orc) {
    const u64 stride = (u64)gridDim.x * blockDim.x;
    for (u64 v = (u64)blockIdx.x * blockDim.x + threadIdx.x; v < nvec; v += stride) {
        uint4 q = ldg_stream(in + v);
        orc[v] = (q.x >> 24) | ((q.y >> 24) << 8) | ((q.z >> 24) << 16) | ((q.w >> 24) << 24);
    }
}

struct Ctx {
    uint4* in; u64 nvec; u32* tree; u32* R; uint8_t* lut; uint8_t* orc; u32* counts; u32* flag; int sms;
    cudaEvent_t e0, e1;
    std::vector<u64> ref;
    LutParams lp;
};

template <typename F>
float timeit(Ctx& c, F f, int reps = 10) {
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

template <int H, int CLS, int HIST, int LOGC, int TPB>
void run(Ctx& c, const char* name, bool set_ref = false) {
    constexpr u32 B = 1u << H, W = TPB / 32;
    constexpr u32 REP_WORDS = (H > 6) ? (((1u << H) - 64u) * 32u) : 0u;
    size_t smem = (B + REP_WORDS + (HIST == 0 ? W * B : (HIST == 1 ? B * 32 : 0)) +
                   (CLS == 1 ? B : (CLS == 2 ? B * 32 : 0))) * 4;
    if (CLS == 1 || CLS == 2) smem += (1u << LOGC);
    auto kern = k2<H, CLS, HIST, LOGC, TPB>;
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int occ = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, TPB, smem));
    if (occ == 0) { printf("%-40s (does not fit: smem %zu)\n", name, smem); return; }
    int grid = occ * c.sms;
    CK(cudaMemset(c.flag, 0, 4));
    float ms = timeit(c, [&] { kern<<<grid, TPB, smem>>>(c.in, c.nvec, c.tree, c.R, c.lut, c.lp, c.orc, c.counts, c.flag); });
    u32 nflag = 0;
    CK(cudaMemcpy(&nflag, c.flag, 4, cudaMemcpyDeviceToHost));
    double n = c.nvec * 4.0;
    std::vector<u32> h((size_t)grid * B);
    CK(cudaMemcpy(h.data(), c.counts, h.size() * 4, cudaMemcpyDeviceToHost));
    std::vector<u64> tot(B, 0);
    for (u32 j = 0; j < B; ++j) for (int g = 0; g < grid; ++g) tot[j] += h[(size_t)g * B + j];
    const char* st = "";
    if (set_ref) { c.ref = tot; st = "(ref)"; }
    else if (HIST != 2 && CLS != 3) st = (tot == c.ref) ? "ok" : "COUNTS WRONG";
    printf("%-40s occ=%d smem=%6zu %8.1f us %7.1f GB/s(5B/el) %.3e el/s fallback-quads/run=%.4f%% %s\n", name, occ, smem,
           ms * 1e3, n * 5.0 / (ms * 1e-3) / 1e9, n / (ms * 1e-3), 100.0 * nflag / 11.0 / (n / 4), st);
}

static u32 key_of(float f) { u32 u; memcpy(&u, &f, 4); return u ^ ((u32)((int)u >> 31) | 0x80000000u); }

// LUT of C cells over the key range of the splitters (see CLS 1)
void build_lut(Ctx& c, const std::vector<u32>& spl, u32 b, int LOGC) {
    const u32 C = 1u << LOGC;
    const u32 s1 = spl[1], sb = spl[b - 1];
    const u32 base = s1 ? s1 - 1 : 0;
    u32 sh = 0;
    while (((u64)(sb - base) >> sh) > C - 2) ++sh;
    auto bucket = [&](u64 x) -> u32 {   // #{s_i <= x}
        return (u32)(std::upper_bound(spl.begin() + 1, spl.begin() + b, (u32)x) - (spl.begin() + 1));
    };
    std::vector<uint8_t> lut(C);
    u64 multi = 0;
    for (u32 cc = 0; cc < C; ++cc) {
        u64 lo = cc == 0 ? 0 : (u64)base + ((u64)cc << sh);
        if (lo > 0xFFFFFFFFull) { lut[cc] = (uint8_t)(b - 2); continue; }
        u64 hi = cc == C - 1 ? 0xFFFFFFFFull : (u64)base + ((u64)(cc + 1) << sh) - 1;
        if (hi > 0xFFFFFFFFull) hi = 0xFFFFFFFFull;
        u32 vlo = bucket(lo), vhi = bucket(hi);
        u32 m;
        if (vhi == vlo) m = vlo < b - 1 ? vlo : b - 2;
        else if (vhi == vlo + 1) m = vlo;
        else { m = b - 1; ++multi; }
        lut[cc] = (uint8_t)m;
    }
    std::vector<u32> R(b);
    for (u32 m = 0; m + 1 < b; ++m) R[m] = spl[m + 1];
    R[b - 1] = 0;
    CK(cudaMemcpy(c.lut, lut.data(), C, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(c.R, R.data(), b * 4, cudaMemcpyHostToDevice));
    c.lp = {base, sh, ((C - 1) << sh) | ((1u << sh) - 1)};
    if (((u64)(C - 1) << sh) + ((1ull << sh) - 1) > 0xFFFFFFFFull) c.lp.dmax = 0xFFFFFFFFu;
    printf("   LUT 2^%d cells: base=%08x sh=%u multi-boundary cells=%llu\n", LOGC, base, sh, multi);
}

std::vector<u32> setup(Ctx& c, int H, int kind) {
    const u64 n = c.nvec * 4;
    std::mt19937_64 rng(5 + kind);
    std::vector<float> x(n);
    std::uniform_real_distribution<float> U(0.f, 1.f);
    std::normal_distribution<float> N(0.f, 1.f);
    for (u64 i = 0; i < n; ++i) x[i] = kind == 0 ? U(rng) : kind == 1 ? N(rng) : (float)(rng() % 16);
    CK(cudaMemcpy(c.in, x.data(), n * 4, cudaMemcpyHostToDevice));
    const u32 b = 1u << H;
    std::vector<u32> smp(4096);
    for (auto& s : smp) s = key_of(x[rng() % n]);
    std::sort(smp.begin(), smp.end());
    std::vector<u32> spl(b + 1), tree(b);
    spl[0] = 0;
    for (u32 i = 1; i < b; ++i) spl[i] = smp[(u64)i * 4096 / b];
    spl[b] = 0xFFFFFFFFu;
    for (int d = 0; d < H; ++d)
        for (u32 p = 0; p < (1u << d); ++p) tree[(1u << d) - 1 + p] = spl[(2 * p + 1) << (H - 1 - d)];
    CK(cudaMemcpy(c.tree, tree.data(), b * 4, cudaMemcpyHostToDevice));
    static const char* names[] = {"uniform", "normal", "16-distinct"};
    printf("-- %s b=%u\n", names[kind], b);
    return spl;
}

#define RUN(H, CLS, HI, LC, T) run<H, CLS, HI, LC, T>(c, "cls=" #CLS " hist=" #HI " cells=2^" #LC " tpb=" #T)

int main() {
    Ctx c;
    CK(cudaDeviceGetAttribute(&c.sms, cudaDevAttrMultiProcessorCount, 0));
    const u64 n = 1ull << 28;
    c.nvec = n / 4;
    CK(cudaMalloc(&c.in, n * 4));
    CK(cudaMalloc(&c.orc, n));
    CK(cudaMalloc(&c.tree, 1024 * 4));
    CK(cudaMalloc(&c.R, 1024 * 4));
    CK(cudaMalloc(&c.lut, 1 << 17));
    CK(cudaMalloc(&c.counts, 4096 * 1024 * 4));
    CK(cudaMalloc(&c.flag, 64));
    CK(cudaEventCreate(&c.e0));
    CK(cudaEventCreate(&c.e1));
    float ms = timeit(c, [&] { read_only<<<c.sms * 8, 256>>>(c.in, c.nvec, c.flag); });
    printf("read_only  %8.1f us %7.1f GB/s\n", ms * 1e3, n * 4.0 / (ms * 1e-3) / 1e9);
    ms = timeit(c, [&] { read_write<<<c.sms * 8, 256>>>(c.in, c.nvec, (u32*)c.orc); });
    printf("read+write %8.1f us %7.1f GB/s (5 B/el)\n", ms * 1e3, n * 5.0 / (ms * 1e-3) / 1e9);
    for (int kind = 0; kind < 3; ++kind) {
        std::vector<u32> spl = setup(c, 8, kind);
        run<8, 0, 0, 15, 512>(c, "cls=0 hist=0 (tree walk, current)", true);
        RUN(8, 0, 1, 15, 512);
        RUN(8, 0, 1, 15, 1024);
        for (int lc : {12, 13, 14, 15, 16}) {
            build_lut(c, spl, 256, lc);
            if (lc == 12) { RUN(8, 2, 1, 12, 512); RUN(8, 2, 1, 12, 1024); }
            if (lc == 13) { RUN(8, 2, 1, 13, 512); RUN(8, 2, 1, 13, 1024); }
            if (lc == 14) { RUN(8, 2, 1, 14, 512); RUN(8, 2, 1, 14, 1024); }
            if (lc == 15) { RUN(8, 2, 1, 15, 512); RUN(8, 2, 1, 15, 1024); }
            if (lc == 16) { RUN(8, 2, 1, 16, 512); RUN(8, 2, 1, 16, 1024); RUN(8, 1, 1, 16, 1024); }
        }
    }
    return 0;
}
