#pragma once
// driver.cuh -- level driver (Layer 1): the context, the per-call control of
// the kernels of one SampleSelect level, and the per-dtype operations the C ABI
// (abi.cu) dispatches to.  Compiled once per dtype (inst_<dtype>.cu defines
// SS_INST_T before including this file), so the kernel templates of one dtype
// live in one translation unit and the four build in parallel; abi.cu includes
// it without SS_INST_T for the context and the shared helpers only.  Everything
// here has internal linkage except the op_* entry points at the end.
//
// The driver follows Fig. 1 (L95-127) with the recursion control kept on the
// device (§IV.E): per call it enqueues an init kernel and, per
// expected level, K1 (sample/tree or base case) -> K2 (count + fused K3/K4
// tail) -> K5 (filter), all reading their data-dependent sizes from
// device-resident LevelCtl blocks and exiting early once the answer is known.
// A final K1 either finishes the base case or flags "incomplete", in which
// case (rare: an unlucky sample) more levels are enqueued.  One device->host
// copy per call returns the answer; there is no per-level host round trip.
#include <algorithm>
#include <chrono>
#include <cmath>
#include <atomic>
#include <cstddef>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>
#include <utility>
#include <vector>
#include <type_traits>

#include "kernels.cuh"
#include "quickselect.cuh"
#include "comm.cuh"
#include "sampleselect.h"

using namespace ss;

struct ExactPlan {
    int b0, bd, s, s_deep;
    int sfs[SS_MAX_LEVELS];           // sample size of each fused level
    bool dir_plan[SS_MAX_LEVELS];     // level l is directed by level l-1's histogram (R28): no K1w
    u32 B;
    int L;                            // levels [.., L) are enqueued, then the final K1
    bool spec_plan[SS_MAX_LEVELS];    // level l is a fused level
    const void* sample0;              // sample keys of level lev_first gathered ahead (or NULL)
    int lev_first;
    void* out0;                       // top-k call: level 0 writes its window here (d_win), else NULL
    u32 kw_grid[SS_MAX_LEVELS];       // fused level l's window_kernel grid (0: one CTA per SM)
};

// ss_select_multi: per-rank tails run as exact calls on child contexts, each
// on its own stream, up to MULTI_CH at a time
constexpr int MULTI_CH = 8;

// A launched exact call (run_exact_begin) waiting for its result hand-off
// (run_exact_end): what the host needs for the rare extra rounds.
struct ExactCall {
    const void* d;
    void* up_out;
    u64 n, k;
    void* h_result;
    bool up;
    int L;
    u32 B;
    int b0, bd;
    double t_in;
    ExactPlan plan;
};

#ifndef SS_USE_GRAPHS
#define SS_USE_GRAPHS 1
#endif
struct ss_context {
    int device = 0;
    int sms = 0;
    ss_config cfg{};
    ss_stats stats{};
    std::string err;
    uint8_t* d_oracles = nullptr;
    size_t cap_oracles = 0;
    void* d_buf[2] = {nullptr, nullptr};
    size_t cap_buf[2] = {0, 0};
    void* d_stage = nullptr;
    size_t cap_stage = 0;
    LevelCtl* d_ctl = nullptr;
    SelectResult* d_res = nullptr;
    u64* d_totals = nullptr;     // [SS_MAX_LEVELS][MAX_B]
    u32* d_cta_counts = nullptr; // [MAX_GRID][MAX_B]
    u64* d_tree = nullptr;       // [SS_MAX_LEVELS][MAX_B] keys (u32 keys use the same bytes)
    u64* d_spl = nullptr;
    uint8_t* d_eq = nullptr;     // [SS_MAX_LEVELS][MAX_B]
    u64* d_sorted = nullptr;     // [SS_MAX_LEVELS][MAX_S] sorted sample keys (wide K1)
    u64* d_sample0 = nullptr;    // [MAX_S] level-0 sample keys (gathered by the init kernel)
    u64* d_presample = nullptr;  // [SS_MAX_LEVELS][MAX_S] sample keys gathered by a fused level's tail
    uint8_t* d_image = nullptr;  // [SS_MAX_LEVELS][K2_IMAGE_SLOT] count-kernel images (tree_image_kernel)
    SelectResult* h_res = nullptr;   // mapped pinned mirror of d_res (written by publish_kernel)
    SelectResult* h_res_dev = nullptr;
    u32 seq = 0;                     // publishes issued (host count, lockstep with *d_seq)
    u32* d_seq = nullptr;            // device publish counter
    // CUDA graphs of whole calls (init + levels + final K1 + publish), one per
    // (dtype, n, plan); the rank k and the input pointer are patched into the
    // init node (level 0's kernels read the input from LevelCtl::src)
    struct GraphEntry {
        bool used = false;
        u64 key = 0;                          // hash of what the captured chain bakes in (graph_launch):
                                              // dtype, plan, sample sizes, seed, ...; n itself is patched
        cudaGraph_t graph = nullptr;       // kept: the init node handle belongs to it
        cudaGraphExec_t exec = nullptr;
        cudaGraphNode_t init_node = nullptr;
        cudaKernelNodeParams init_params{};
        void* init_args[16] = {};
        unsigned char init_store[256] = {};   // backing store of the init kernel's arguments
        size_t k_offset = 0;                  // where k lives in init_store
        size_t n_offset = 0;                  // where n lives in init_store
        size_t d_offset = 0;                  // where the input pointer lives in init_store
        size_t up_offset = 0;                 // where the top-k output pointer lives
        int kernels = 0;
        u64 stamp = 0;
    } graphs[8];
    u64 graph_clock = 0;
    cudaStream_t cap_st = nullptr;   // capture stream (graphs are captured off the caller's stream)
    bool use_graphs = SS_USE_GRAPHS != 0;   // (-DSS_USE_GRAPHS=0: every call launches its kernels directly)
    // record of the last ss_step_count (per-CTA counts feed ss_step_filter)
    const void* step_ptr = nullptr;
    u64 step_n = 0;
    int step_b = 0;
    int step_dt = -1;
    u32 step_grid = 0;
    // profile=1: event pairs around every kernel, slot (level, kernel)
    cudaEvent_t ev[SS_MAX_LEVELS][3][2] = {};
    bool ev_used[SS_MAX_LEVELS][3] = {};
    bool ev_ready = false;
    double prof_sum[SS_MAX_LEVELS][3] = {};   // accumulated device ms per (level, kernel)
    long long prof_cnt[SS_MAX_LEVELS][3] = {};
    long long launches_total = 0;
    long long calls_total = 0;
    int launches = 0;
    int64_t h2d = 0, d2h = 0;   // bytes copied by the current call
    // SS_HOST_TIMING=1: host-side phase times of run_exact, printed by ss_destroy
    unsigned long long* d_upper_cnt = nullptr;  // ss_select_upper: #{x > result}
    cudaEvent_t ev_upper[2] = {nullptr, nullptr};
    unsigned upper_attr = 0;                    // bit dt_code: gather kernel smem attribute set
    unsigned mf_attr = 0;                       // bit dt_code: multi_filter_kernel smem attribute set
    // ss_select_multi: scratch (sample keys, tree, splitters, eq, totals, search
    // results, bucket counts, one value) and the extracted buckets
    unsigned char* d_multi_scratch = nullptr;
    void* d_multi = nullptr;
    size_t cap_multi = 0;
    ss_context* mchild[MULTI_CH] = {};          // child contexts of the per-rank tails
    cudaStream_t mchild_st[MULTI_CH] = {};
    cudaEvent_t ev_mfork = nullptr, ev_mjoin[MULTI_CH] = {};
    unsigned char* h_mpin = nullptr;            // pinned staging: ranks in, search rows out, slot tables
    // ss_quickselect: device control block, ping-pong level
    // buffers (level 0 writes up to n - 1 elements), batch-end host mirror
    QsCtl* d_qs = nullptr;
    QsCtl* h_qs = nullptr;
    void* d_qsbuf[2] = {nullptr, nullptr};
    size_t cap_qsbuf = 0;
    cudaEvent_t ev_qs[2] = {nullptr, nullptr};
    // ss_select_sharded: the communicator, the exchange buffers
    // (sizes, per-rank counts, sample keys), the gather send/receive buffers
    ss_comm::ShardComm* comm = nullptr;
    u64 dist_n_plan = 0;             // size of the union seen by the last sharded call (0: exchange first)
    void* d_dist = nullptr;
    size_t cap_dist = 0;
    void* d_gather[2] = {nullptr, nullptr};
    size_t cap_gather[2] = {0, 0};
    int k2_occ[4][11] = {};          // count_kernel<T, H> resident CTAs per SM (per dtype, H)
    bool kw_attr[4][3] = {};         // window_kernel<T, APX, UP> shared-memory attribute set
    // ss_select_upper one-pass path: level 0's window, kept for the top-k tail
    // (level 1 reads it; deeper levels ping-pong in d_buf)
    void* d_win = nullptr;
    size_t cap_win = 0;
    bool up_used = false;            // the last run_exact ran the one-pass top-k path
    ExactCall call{};                // the exact call in flight (run_exact_begin .. run_exact_end)
    bool shared_gpu = false;         // a child context of ss_select_multi: small levels on part of the GPU
    bool host_timing = false;
    double ht[5] = {};
    long long ht_n = 0;
};
static inline double now_us() {
    return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

static constexpr u32 MAX_GRID = 2048;
static constexpr int MAX_S = 16384;
// sample sizes up to this are ranked by the wide K1 (s/32 CTAs, s^2 pairs);
// larger samples (approximate b = 1024) use the one-CTA bitonic K1
static constexpr int WIDE_K1_MAX_S = 4096;

namespace {

struct DevGuard {
    int prev = -1;
    explicit DevGuard(int d) {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (prev != d) cudaSetDevice(d);
    }
    ~DevGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

ss_status fail(ss_context* c, ss_status s, const std::string& msg) {
    if (c) c->err = msg;
    return s;
}

#define CK(call)                                                                              \
    do {                                                                                      \
        cudaError_t e_ = (call);                                                              \
        if (e_ != cudaSuccess) {                                                              \
            (void)cudaGetLastError();                                                         \
            return fail(c, e_ == cudaErrorMemoryAllocation ? SS_ERR_OUT_OF_MEMORY : SS_ERR_CUDA, \
                        std::string(#call) + ": " + cudaGetErrorString(e_));                  \
        }                                                                                     \
    } while (0)

#define CKLAUNCH(what) CK(cudaGetLastError())

// Launch with programmatic stream serialisation (PDL): the kernel may become
// resident while its predecessor on the stream finishes; it waits for the
// predecessor's completion inside (pdl_wait) before reading its results.
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                       Args&&... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}

template <typename T> constexpr int dt_code() {
    return std::is_same<T, float>::value ? 1 : std::is_same<T, double>::value ? 2 : std::is_same<T, int>::value ? 3 : 4;
}

int log2i(int b) {
    int h = 0;
    while ((1 << h) < b) ++h;
    return h;
}
bool pow2(long long x) { return x > 0 && (x & (x - 1)) == 0; }

size_t dt_size(ss_dtype dt) {
    switch (dt) {
    case SS_FLOAT32: case SS_INT32: return 4;
    case SS_FLOAT64: case SS_INT64: return 8;
    default: return 0;
    }
}

int sample_size(const ss_config& cfg, int b) {
    if (cfg.sample_size > 0) return cfg.sample_size;
    return std::max(4096, std::min(16 * b, 16384));
}

ss_status grow(ss_context* c, void** p, size_t* cap, size_t need) {
    if (*cap >= need && *p) return SS_OK;
    if (*p) {
        cudaFree(*p);
        *p = nullptr;
        *cap = 0;
    }
    for (auto& e : c->graphs) {   // captured graphs hold the old buffer addresses
        if (e.exec) cudaGraphExecDestroy(e.exec);
        if (e.graph) cudaGraphDestroy(e.graph);
        e = ss_context::GraphEntry();
    }
    size_t alloc = need + need / 16 + 256;
    CK(cudaMalloc(p, alloc));
    *cap = alloc;
    return SS_OK;
}

// Grow *p to `need` bytes keeping its first `keep` bytes (a stream-ordered
// device copy; the old block is freed once the copy is done).
ss_status grow_keep(ss_context* c, void** p, size_t* cap, size_t need, size_t keep, cudaStream_t st) {
    if (*cap >= need && *p) return SS_OK;
    void* old = *p;
    *p = nullptr;
    *cap = 0;
    ss_status rc = grow(c, p, cap, need);
    if (rc) return rc;
    if (old) {
        if (keep) CK(cudaMemcpyAsync(*p, old, keep, cudaMemcpyDeviceToDevice, st));
        CK(cudaStreamSynchronize(st));
        cudaFree(old);
    }
    return SS_OK;
}

// Device bytes the context owns (ss_stats.workspace_bytes).
size_t workspace_bytes(const ss_context* c);

// count/filter grid: resident CTAs of the count kernel x #SMs (one wave)
// (the occupancy is cached per context: a context belongs to one device and
// one host thread, so no cache is shared between threads)
template <typename T, int H>
u32 count_grid(ss_context* c) {
    int& occ = c->k2_occ[dt_code<T>() - 1][H];
    if (!occ) {
        int o = 0;
        typedef typename Traits<T>::Key K;
        cudaFuncSetAttribute(count_kernel<T, H>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)count_smem_bytes<H, K>());
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, count_kernel<T, H>, K2_THREADS,
                                                      count_smem_bytes<H, K>());
        occ = o > 0 ? o : 1;
    }
    u32 per = (u32)std::max(1, std::min(c->cfg.ctas_per_sm, occ));
    return std::min<u32>(per * (u32)c->sms, MAX_GRID);
}

template <typename T>
ss_status launch_count(ss_context* c, int H, const T* in, CountArgs& a, cudaStream_t st) {
#define SS_COUNT_CASE(h)                                                     \
    case h:                                                                  \
        a.grid = count_grid<T, h>(c);                                        \
        CK(launch_pdl(count_kernel<T, h>, dim3(a.grid), dim3(K2_THREADS),    \
            count_smem_bytes<h, typename Traits<T>::Key>(), st, in, a));     \
        break;
    switch (H) {
        SS_COUNT_CASE(2) SS_COUNT_CASE(3) SS_COUNT_CASE(4) SS_COUNT_CASE(5) SS_COUNT_CASE(6)
        SS_COUNT_CASE(7) SS_COUNT_CASE(8) SS_COUNT_CASE(9) SS_COUNT_CASE(10)
    default: return fail(c, SS_ERR_INVALID_ARGUMENT, "b must be a power of two in [4, 1024]");
    }
#undef SS_COUNT_CASE
    CKLAUNCH("count_kernel");
    return SS_OK;
}

// fused count + filter kernel: one CTA per SM, KW_SMEM bytes (TMA ring + stash)
template <typename T, bool APX = false, bool UP = false>
ss_status launch_window(ss_context* c, int /*H*/, const T* in, CountArgs a, cudaStream_t st) {
    if (!a.grid) a.grid = (u32)c->sms * (u32)KW_MINB;   // (a small planned level may take fewer CTAs)
    bool& attr_set = c->kw_attr[dt_code<T>() - 1][APX ? 1 : UP ? 2 : 0];
    if (!attr_set) {
        CK(cudaFuncSetAttribute(window_kernel<T, APX, UP>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)KW_SMEM));
        attr_set = true;
    }
    CK(launch_pdl(window_kernel<T, APX, UP>, dim3(a.grid), dim3(KW_THREADS), KW_SMEM, st, in, a));
    CKLAUNCH("window_kernel");
    return SS_OK;
}

template <typename T>
u32 grid_for(ss_context* c, int H) {
    switch (H) {
    case 2: return count_grid<T, 2>(c);
    case 3: return count_grid<T, 3>(c);
    case 4: return count_grid<T, 4>(c);
    case 5: return count_grid<T, 5>(c);
    case 6: return count_grid<T, 6>(c);
    case 7: return count_grid<T, 7>(c);
    case 8: return count_grid<T, 8>(c);
    case 9: return count_grid<T, 9>(c);
    default: return count_grid<T, 10>(c);
    }
}

// K1's dynamic smem holds the s sample keys (the base case keeps its keys in registers)
template <typename T>
size_t k1_smem(int s, u32 B) {            // the sample, or the base case's B keys
    typedef typename Traits<T>::Key K;
    return (size_t)std::max<u32>((u32)s, B) * sizeof(K);
}

template <typename T>
ss_status set_k1_attrs(ss_context* c) {
    typedef typename Traits<T>::Key K;
    CK(cudaFuncSetAttribute(sample_tree_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)(16384 * sizeof(K))));
    CK(cudaFuncSetAttribute(filter_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)FILTER_SMEM));
    CK(cudaFuncSetAttribute(sample_rank_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)(16384 * sizeof(K))));
    CK(cudaFuncSetAttribute(sample_chunk_sort_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)(K1C_CHUNK * sizeof(K))));
    CK(cudaFuncSetAttribute(sample_merge_rank_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)(16384 * sizeof(K))));
    CK(cudaFuncSetAttribute(qs_pivot_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)(16384 * sizeof(K))));
    CK(cudaFuncSetAttribute(wsel_cluster_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)(WC_KEYS * sizeof(K))));
    return SS_OK;
}

ss_status ensure_small(ss_context* c) {
    if (c->d_ctl) return SS_OK;
    CK(cudaMalloc(&c->d_ctl, sizeof(LevelCtl) * (SS_MAX_LEVELS + 1)));
    CK(cudaMalloc(&c->d_res, sizeof(SelectResult)));
    CK(cudaMalloc(&c->d_totals, sizeof(u64) * SS_MAX_LEVELS * MAX_B));
    CK(cudaMalloc(&c->d_cta_counts, sizeof(u32) * (size_t)MAX_GRID * MAX_B));
    CK(cudaMalloc(&c->d_tree, sizeof(u64) * SS_MAX_LEVELS * MAX_B));
    CK(cudaMalloc(&c->d_spl, sizeof(u64) * SS_MAX_LEVELS * MAX_B));
    CK(cudaMalloc(&c->d_eq, (size_t)SS_MAX_LEVELS * MAX_B));
    CK(cudaMalloc(&c->d_sorted, sizeof(u64) * SS_MAX_LEVELS * MAX_S));
    CK(cudaMalloc(&c->d_sample0, sizeof(u64) * MAX_S));
    CK(cudaMalloc(&c->d_presample, sizeof(u64) * SS_MAX_LEVELS * MAX_S));
    CK(cudaMalloc(&c->d_image, K2_IMAGE_SLOT * SS_MAX_LEVELS));
    CK(cudaHostAlloc(&c->h_res, sizeof(SelectResult), cudaHostAllocMapped));
    std::memset(c->h_res, 0, sizeof(SelectResult));
    CK(cudaHostGetDevicePointer((void**)&c->h_res_dev, c->h_res, 0));
    CK(cudaMalloc(&c->d_seq, sizeof(u32)));
    CK(cudaMemset(c->d_seq, 0, sizeof(u32)));
    CK(cudaStreamCreateWithFlags(&c->cap_st, cudaStreamNonBlocking));
    return SS_OK;
}

ss_status prof_init(ss_context* c) {
    if (c->ev_ready) return SS_OK;
    for (int l = 0; l < SS_MAX_LEVELS; ++l)
        for (int q = 0; q < 3; ++q)
            for (int e = 0; e < 2; ++e) CK(cudaEventCreate(&c->ev[l][q][e]));
    c->ev_ready = true;
    return SS_OK;
}

// Record the start (e=0) / end (e=1) event of kernel q at level l.
inline void mark(ss_context* c, int l, int q, int e, cudaStream_t st) {
    if (!c->cfg.profile || c->cfg.profile == 3 || l >= SS_MAX_LEVELS) return;
    if (c->cfg.profile == 2 && !(l == 0 && q == 1)) return;   // dominant kernel only
    cudaEventRecord(c->ev[l][q][e], st);
    if (e) c->ev_used[l][q] = true;
}

// bytes of the result block read back per call (the timeline only in profile=3)
size_t res_bytes(const ss_context* c) {
    return c->cfg.profile == 3 ? sizeof(SelectResult) : offsetof(SelectResult, tl_on);
}

// Enqueue the result hand-off and wait for it: the publish kernel writes the
// result block into the mapped host mirror and then the new sequence number;
// the host spins on that word (checking the stream for errors now and then).
ss_status enqueue_publish(ss_context* c, cudaStream_t st) {
    const u32 nwords = (u32)(res_bytes(c) / 4);
    const u32 seq_word = (u32)(offsetof(SelectResult, seq) / 4);
    CK(launch_pdl(publish_kernel, dim3(1), dim3(128), 0, st, reinterpret_cast<const u32*>(c->d_res),
                  reinterpret_cast<u32*>(c->h_res_dev), nwords, seq_word, c->d_seq));
    CKLAUNCH("publish_kernel");
    ++c->launches;
    return SS_OK;
}

ss_status wait_publish(ss_context* c, cudaStream_t st) {
    const u32 seq = ++c->seq;
    c->d2h += res_bytes(c);
    volatile u32* flag = &c->h_res->seq;
    for (u64 spin = 1;; ++spin) {
        if (*flag == seq) break;
        if ((spin & 1023) == 0) {
            const cudaError_t e = cudaStreamQuery(st);
            if (e != cudaSuccess && e != cudaErrorNotReady) CK(e);
            if (e == cudaSuccess && *flag != seq) return fail(c, SS_ERR_INTERNAL, "result hand-off lost");
        }
    }
    std::atomic_thread_fence(std::memory_order_acquire);
    return SS_OK;
}

void prof_collect(ss_context* c) {
    if (c->cfg.profile == 3) {
        const SelectResult& r = *c->h_res;
        for (int l = 0; l < SS_MAX_LEVELS; ++l)
            for (int q = 0; q < 3; ++q) {
                const u64 a = ~r.tl[l * 3 + q][0], b = r.tl[l * 3 + q][1];
                const bool ran = r.tl[l * 3 + q][0] != 0 && b != 0;
                c->stats.tl_us[l][q][0] = ran ? (float)((double)(long long)(a - r.t_init) * 1e-3) : -1.f;
                c->stats.tl_us[l][q][1] = ran ? (float)((double)(long long)(b - r.t_init) * 1e-3) : -1.f;
                const float ms = ran ? (float)((double)(long long)(b - a) * 1e-6) : 0.f;
                c->stats.ms_kernel[l][q] = ms;
                if (ran) {
                    c->prof_sum[l][q] += ms;
                    c->prof_cnt[l][q] += 1;
                }
            }
        return;
    }
    for (int l = 0; l < SS_MAX_LEVELS; ++l)
        for (int q = 0; q < 3; ++q) {
            float ms = 0.f;
            if (c->cfg.profile && c->ev_used[l][q])
                cudaEventElapsedTime(&ms, c->ev[l][q][0], c->ev[l][q][1]);
            c->stats.ms_kernel[l][q] = ms;
            c->prof_sum[l][q] += ms;
            if (c->cfg.profile && c->ev_used[l][q]) c->prof_cnt[l][q] += 1;
            c->ev_used[l][q] = false;
        }
    (void)cudaGetLastError();
}

struct SpecCfg { u64 min_n; float z, max_frac; };
SpecCfg spec_params(const ss_context* c) {
    SpecCfg p;
    p.min_n = c->cfg.fused_filter ? (u64)c->cfg.spec_min_n : ~0ull;
    p.z = c->cfg.spec_z;
    p.max_frac = c->cfg.spec_max_frac;
    return p;
}

// Fused-level sample sizes (K1w): the configured sample_size if set (at least
// 1024), else at level 0 16384 for large inputs -- the window is ~6 z /
// sqrt(s) of the level, and level 0's window decides the largest write and
// the next level's size -- and 4096 up to 2^25 elements, where K1w's cost
// (12.5 vs 7.8 us on B200) outweighs the larger window (measured device time
// 2^16: 30 -> 26 us, 2^20: 40.6 -> 37.6 us, 2^24: 51 -> 47 us); deeper, the
// smallest of 4096 / 8192 / 16384 whose expected window fits the base case
// (saving a whole level), else 4096.
constexpr u64 SMALL_L0_SAMPLE_MAX_N = (u64)1 << 25;
inline int fused_sample(const ss_config& cfg, int level, u64 n) {
    if (cfg.sample_size > 0) return std::max(1024, std::min(cfg.sample_size, 16384));
    return level || n <= SMALL_L0_SAMPLE_MAX_N ? 4096 : 16384;
}

inline double window_frac(float z, int s) {
    return (2.0 * (z * 0.5 * std::sqrt((double)s) + 2.0) + 1.0) / s;
}

// The planned levels of an exact call.  A paper level keeps ~1.5 / b of its
// input (the bucket holding k is size-biased, ~1.1 for s / b = 16; 1.5 is
// slack); a fused level keeps its window (<= window_frac of it, plus chunk
// padding); a directed level (reading R28: its window is the key bin of the
// previous fused level's histogram that holds its rank) keeps one of KW_HB
// bins (4 / KW_HB planned: the bins split the window's key range, not its
// elements).  Levels with at least spec_min_n elements (host estimate) are
// fused when fused_filter is on, and the fused levels after the first are
// directed; sf_plan[l] is a fused level's sample size.  An under-estimate is
// caught on the device (the final level flags "incomplete") and more levels
// are enqueued.
int expected_levels(const ss_context* c, u64 n, int b0, int bd, u32 B, bool* spec_plan, int* sf_plan,
                    bool* dir_plan, double* est = nullptr) {
    const SpecCfg sp = spec_params(c);
    const double pad = (double)c->sms * 32.0;
    int L = 0;
    double m = (double)n;
    bool prev_fused = false;
    while (m > (double)B && L < SS_MAX_LEVELS - 2) {
        const int b = L ? bd : b0;
        int sf = fused_sample(c->cfg, L, n);
        if (L && c->cfg.sample_size <= 0)
            for (int cand = 4096; cand <= 16384; cand *= 2)
                if (m * 1.1 * window_frac(sp.z, cand) + pad / 2 <= (double)B) {
                    sf = cand;
                    break;
                }
        const double f = window_frac(sp.z, sf);
        const bool dir = prev_fused && c->cfg.directed;
        const bool spec = dir || (sp.min_n != ~0ull && m >= (double)sp.min_n && f <= sp.max_frac);
        if (spec_plan) spec_plan[L] = spec;
        if (sf_plan) sf_plan[L] = sf;
        if (dir_plan) dir_plan[L] = dir;
        if (est) est[L] = m;
        m = dir ? m * 4.0 / KW_HB + pad : spec ? m * 1.2 * f + pad : m * 1.5 / b;
        prev_fused = spec;
        ++L;
    }
    return L;
}

template <typename T>
ss_status launch_k1(ss_context* c, const T* in, int lev, int s, int b, int fixup, u32 B, int final_level,
                    cudaStream_t st, void* sorted_out = nullptr) {
    typedef typename Traits<T>::Key K;
    K* tree = reinterpret_cast<K*>(c->d_tree) + (size_t)lev * MAX_B;
    K* spl = reinterpret_cast<K*>(c->d_spl) + (size_t)lev * MAX_B;
    uint8_t* eq = c->d_eq + (size_t)lev * MAX_B;
    mark(c, lev, 0, 0, st);
    CK(launch_pdl(sample_tree_kernel<T>, dim3(1), dim3(K1_THREADS), k1_smem<T>(s, B), st,
                  in, c->d_ctl + lev, c->d_res, tree, spl, eq, s, b, fixup, B, (u64)c->cfg.seed, lev,
                  final_level, reinterpret_cast<K*>(sorted_out)));
    CKLAUNCH("sample_tree_kernel");
    mark(c, lev, 0, 1, st);
    ++c->launches;
    return SS_OK;
}

// Wide K1: gather + rank the level's sample on s/32 CTAs (or the base case).
template <typename T>
ss_status launch_k1_wide(ss_context* c, const T* in, int lev, int s, u32 B, cudaStream_t st,
                         const void* presampled = nullptr) {
    typedef typename Traits<T>::Key K;
    K* sorted = reinterpret_cast<K*>(c->d_sorted) + (size_t)lev * MAX_S;
    mark(c, lev, 0, 0, st);
    CK(launch_pdl(sample_rank_kernel<T>, dim3(((u32)s + 31u) / 32u), dim3(K1R_THREADS),
                  k1_smem<T>(s, B), st,
                  in, c->d_ctl + lev, c->d_res, sorted, s, B, (u64)c->cfg.seed, lev,
                  reinterpret_cast<const K*>(presampled)));
    CKLAUNCH("sample_rank_kernel");
    mark(c, lev, 0, 1, st);
    ++c->launches;
    return SS_OK;
}

// K1b: the level's tree + count-kernel image from the wide K1's sorted sample.
template <typename T>
ss_status launch_image(ss_context* c, int H, int lev, int s, int fixup, cudaStream_t st) {
    typedef typename Traits<T>::Key K;
    const K* sorted = reinterpret_cast<const K*>(c->d_sorted) + (size_t)lev * MAX_S;
    uint8_t* image = c->d_image + (size_t)lev * K2_IMAGE_SLOT;
    K* tree = reinterpret_cast<K*>(c->d_tree) + (size_t)lev * MAX_B;
    K* spl = reinterpret_cast<K*>(c->d_spl) + (size_t)lev * MAX_B;
    uint8_t* eq = c->d_eq + (size_t)lev * MAX_B;
    const int lut_on = c->cfg.classify == 0;
#define SS_IMG_CASE(h)                                                                                     \
    case h:                                                                                                \
        CK(launch_pdl(tree_image_kernel<T, h>, dim3(IMG_CTAS), dim3(1024), 0, st, sorted, s, fixup, lut_on, \
                      c->d_ctl + lev, c->d_res, image, tree, spl, eq));                                    \
        break;
    switch (H) {
        SS_IMG_CASE(2) SS_IMG_CASE(3) SS_IMG_CASE(4) SS_IMG_CASE(5) SS_IMG_CASE(6)
        SS_IMG_CASE(7) SS_IMG_CASE(8) SS_IMG_CASE(9) SS_IMG_CASE(10)
    default: return fail(c, SS_ERR_INVALID_ARGUMENT, "b must be a power of two in [4, 1024]");
    }
#undef SS_IMG_CASE
    CKLAUNCH("tree_image_kernel");
    ++c->launches;
    return SS_OK;
}

// The exact chain of Fig. 1 (L95-127) from level lev0 to the plan's L.  A
// paper level is K1 (sample + sort, or the base case), the tree image, K2
// (count + K3/K4 tail) and K5 (filter); a fused level (spec_plan) is K1w (the
// window straight from the sample, wsel_cluster_kernel) and the fused
// count + filter pass (window_kernel) -- nothing else is enqueued behind it:
// a miss halts the chain (SelectResult::halt) and the host re-runs that level
// the paper's way.  Every kernel reads its sizes from the device-resident
// LevelCtl of its level and exits early once the answer is known; the chain
// ends with the final K1 (base case, or the "incomplete" flag when an unlucky
// sample left more than B elements).  Level p.lev_first reads `first_in`;
// level l > p.lev_first reads the buffer level l-1 wrote (d_buf[(l-1) & 1]).


constexpr double KW_CTA_ELEMS = 32768.0;     // elements per window CTA on a small planned level

// The buffer level `lev` writes (and level lev + 1 reads).
inline void* level_out(const ss_context* c, const ExactPlan& p, int lev) {
    return lev == 0 && p.out0 ? p.out0 : c->d_buf[lev & 1];
}

inline int plan_sample(const ExactPlan& p, int lev) {
    if (p.spec_plan[lev]) return p.sfs[lev];
    return lev ? p.s_deep : p.s;
}

template <typename T>
ss_status launch_wsel(ss_context* c, const T* in, int lev, int s, u32 B, const void* pre, int final_level,
                      cudaStream_t q) {
    typedef typename Traits<T>::Key K;
    const SpecCfg sp = spec_params(c);
    mark(c, lev, 0, 0, q);
    CK(launch_pdl(wsel_cluster_kernel<T>, dim3(WC_CTAS), dim3(WC_THREADS), WC_KEYS * sizeof(K), q, in,
                  c->d_ctl + lev, c->d_ctl + lev + 1, c->d_res, reinterpret_cast<const K*>(pre), (u32)s, B,
                  (u64)c->cfg.seed, lev, sp.z, sp.max_frac, final_level));
    CKLAUNCH("wsel_cluster_kernel");
    mark(c, lev, 0, 1, q);
    ++c->launches;
    return SS_OK;
}

template <typename T>
ss_status enqueue_exact_levels(ss_context* c, const ExactPlan& p, const T* first_in, int lev0, cudaStream_t q) {
    typedef typename Traits<T>::Key K;
    ss_status rc;
    const T* in = lev0 > p.lev_first ? reinterpret_cast<const T*>(level_out(c, p, lev0 - 1)) : first_in;
    const u64 cap_limit = std::min(std::min(c->cap_buf[0], c->cap_buf[1]), p.out0 ? c->cap_win : ~(size_t)0) /
                          sizeof(T);          // elements per level buffer
    int lev = lev0;
    for (; lev < p.L; ++lev) {
        const int b = lev ? p.bd : p.b0, H = log2i(b);
        const int sl = plan_sample(p, lev);
        const int sl_next = lev + 1 < p.L ? plan_sample(p, lev + 1) : 0;
        // a fused level's tail gathers the next level's sample from its output
        K* pre_next = lev + 1 < p.L && !p.dir_plan[lev + 1] && (p.spec_plan[lev + 1] || sl_next <= WIDE_K1_MAX_S)
                          ? reinterpret_cast<K*>(c->d_presample) + (size_t)(lev + 1) * MAX_S : nullptr;
        const void* pre_this = lev == p.lev_first ? p.sample0
                               : (lev > 0 && p.spec_plan[lev - 1]
                                      ? (const void*)(reinterpret_cast<K*>(c->d_presample) + (size_t)lev * MAX_S)
                                      : nullptr);
        if (p.spec_plan[lev]) {               // fused level: K1w + count/filter in one pass
            const void* pre_buf = pre_this ? pre_this
                                           : (const void*)(reinterpret_cast<K*>(c->d_presample) + (size_t)lev * MAX_S);
            if (!p.dir_plan[lev] && (rc = launch_wsel<T>(c, in, lev, sl, p.B, pre_buf, 0, q))) return rc;
            const SpecCfg sp = spec_params(c);
            CountArgs w{};
            w.ctl = c->d_ctl + lev;
            w.ctl_next = c->d_ctl + lev + 1;
            w.res = c->d_res;
            w.level = lev;
            w.tail = TAIL_EXACT;
            w.cap_out = level_out(c, p, lev);  // the window = the next level's input
            w.spec_min_n = sp.min_n;
            w.spec_z = sp.z;
            w.spec_max_frac = sp.max_frac;
            w.sample_next = pre_next;
            w.s_next = sl_next;
            w.seed = (u64)c->cfg.seed;
            w.halt_on_miss = 1;
            w.cap_limit = cap_limit;
            w.hist = lev + 1 < p.L && p.dir_plan[lev + 1];
            w.dir_level = p.dir_plan[lev];
            w.totals = c->d_totals + (size_t)lev * MAX_B;   // the hist bins (zeroed by init)
            w.grid = p.kw_grid[lev];
            mark(c, lev, 1, 0, q);
            if (lev == 0 && p.out0) {          // top-k: also stream the keys above the window out
                if ((rc = launch_window<T, false, true>(c, H, in, w, q))) return rc;
            } else if ((rc = launch_window<T>(c, H, in, w, q))) {
                return rc;
            }
            mark(c, lev, 1, 1, q);
            ++c->launches;
            in = reinterpret_cast<const T*>(level_out(c, p, lev));
            continue;
        }
        const u32 grid = grid_for<T>(c, H);
        const bool wide = sl <= WIDE_K1_MAX_S;
        CountArgs a{};
        if (wide) a.image = c->d_image + (size_t)lev * K2_IMAGE_SLOT;
        a.ctl = c->d_ctl + lev;
        a.ctl_next = c->d_ctl + lev + 1;
        a.res = c->d_res;
        a.tree = reinterpret_cast<K*>(c->d_tree) + (size_t)lev * MAX_B;
        a.spl = reinterpret_cast<K*>(c->d_spl) + (size_t)lev * MAX_B;
        a.eq = c->d_eq + (size_t)lev * MAX_B;
        a.oracles = c->d_oracles;
        a.cta_counts = c->d_cta_counts;
        a.totals = c->d_totals + (size_t)lev * MAX_B;
        a.lut = c->cfg.classify == 0;
        a.lut_stats = lev == 0 ? c->d_res->lut_stats : nullptr;
        a.level = lev;
        a.tail = TAIL_EXACT;
        a.cap_limit = cap_limit;
        if (wide) {
            if ((rc = launch_k1_wide<T>(c, in, lev, sl, p.B, q, pre_this))) return rc;
            if (lev == 0) {
                if ((rc = launch_image<T>(c, H, lev, sl, 1, q))) return rc;
            } else {
                // small deeper level: each count CTA builds the tree from
                // the sorted sample itself and walks it (no image kernel,
                // no lookup table)
                a.image = nullptr;
                a.sorted = reinterpret_cast<K*>(c->d_sorted) + (size_t)lev * MAX_S;
                a.s = sl;
                a.fixup = 1;
                a.lut = 0;
            }
        } else if ((rc = launch_k1<T>(c, in, lev, sl, b, 1, p.B, 0, q))) {
            return rc;
        }
        mark(c, lev, 1, 0, q);
        if ((rc = launch_count<T>(c, H, in, a, q))) return rc;
        mark(c, lev, 1, 1, q);
        ++c->launches;
        if (a.grid != grid) return fail(c, SS_ERR_INTERNAL, "grid mismatch");
        T* out = reinterpret_cast<T*>(level_out(c, p, lev));
        FilterArgs f{};
        f.ctl = c->d_ctl + lev;
        f.res = c->d_res;
        f.oracles = c->d_oracles;
        f.cta_counts = c->d_cta_counts;
        f.b_count = (u32)b;
        f.grid = grid;
        f.level = lev;
        mark(c, lev, 2, 0, q);
        CK(launch_pdl(filter_kernel<T>, dim3(grid), dim3(K5_THREADS), FILTER_SMEM, q, in, out, f));
        CKLAUNCH("filter_kernel");
        mark(c, lev, 2, 1, q);
        ++c->launches;
        in = out;
    }
    // the final level: the base case on one cluster (or the "incomplete" flag)
    return launch_wsel<T>(c, in, lev, 0, p.B, nullptr, 1, q);
}

// Launch a call's chain as one cached CUDA graph keyed on `key` (everything
// the captured kernels bake in: dtype, plan, sample sizes, seed ...): captured
// on first use (enqueue(capture stream)), then replayed with n, k, the input
// and the top-k output patched into its init node -- the only kernel that
// takes them as arguments (the others read LevelCtl).
template <typename T, typename F>
ss_status graph_launch(ss_context* c, u64 key, u64 n, u64 k, const T* d, void* up, F&& enqueue, cudaStream_t st) {
    typedef typename Traits<T>::Key K;
    ss_context::GraphEntry* ge = nullptr;
    for (auto& e : c->graphs)
        if (e.used && e.key == key) ge = &e;
    if (!ge) {
        ss_context::GraphEntry* slot = nullptr;           // a free entry, else the least recently used
        for (auto& e : c->graphs)
            if (!e.used) { slot = &e; break; }
        if (!slot) {
            slot = &c->graphs[0];
            for (auto& e : c->graphs)
                if (e.stamp < slot->stamp) slot = &e;
        }
        if (slot->exec) cudaGraphExecDestroy(slot->exec);
        if (slot->graph) cudaGraphDestroy(slot->graph);
        *slot = ss_context::GraphEntry();
        const int launches0 = c->launches;
        CK(cudaStreamBeginCapture(c->cap_st, cudaStreamCaptureModeThreadLocal));
        const ss_status rc2 = enqueue(c->cap_st);
        cudaGraph_t g = nullptr;
        const cudaError_t ec = cudaStreamEndCapture(c->cap_st, &g);
        if (rc2) {
            if (g) cudaGraphDestroy(g);
            return rc2;
        }
        CK(ec);
        cudaGraphExec_t ex = nullptr;
        const cudaError_t ei = cudaGraphInstantiate(&ex, g, 0);
        // the init node: the graph's only kernel node running init_kernel<T>
        size_t nn = 0;
        cudaGraphGetNodes(g, nullptr, &nn);
        std::vector<cudaGraphNode_t> nodes(nn);
        cudaGraphGetNodes(g, nodes.data(), &nn);
        cudaGraphNode_t init_node = nullptr;
        cudaKernelNodeParams ip{};
        for (auto nd : nodes) {
            cudaGraphNodeType ty;
            cudaGraphNodeGetType(nd, &ty);
            if (ty != cudaGraphNodeTypeKernel) continue;
            cudaKernelNodeParams kp{};
            if (cudaGraphKernelNodeGetParams(nd, &kp) == cudaSuccess &&
                kp.func == reinterpret_cast<void*>(init_kernel<T>)) {
                init_node = nd;
                ip = kp;
            }
        }
        if (ei != cudaSuccess || !init_node) {
            cudaGraphDestroy(g);
            if (ex) cudaGraphExecDestroy(ex);
            (void)cudaGetLastError();
            return fail(c, SS_ERR_CUDA, "graph capture of the level chain failed");
        }
        slot->used = true;
        slot->key = key;
        slot->exec = ex;
        slot->init_node = init_node;
        slot->kernels = c->launches - launches0;
        // private copy of the init arguments (n index 5, k 6, input 8, top-k output 12)
        slot->init_params = ip;
        size_t off = 0;
        const size_t sizes[13] = {sizeof(LevelCtl*), sizeof(int), sizeof(u64*), sizeof(int), sizeof(SelectResult*),
                                  sizeof(u64), sizeof(u64), sizeof(int), sizeof(const T*), sizeof(int), sizeof(u64),
                                  sizeof(K*), sizeof(void*)};
        for (int i = 0; i < 13; ++i) {
            off = (off + 7) & ~(size_t)7;
            std::memcpy(slot->init_store + off, ip.kernelParams[i], sizes[i]);
            slot->init_args[i] = slot->init_store + off;
            if (i == 5) slot->n_offset = off;
            if (i == 6) slot->k_offset = off;
            if (i == 8) slot->d_offset = off;
            if (i == 12) slot->up_offset = off;
            off += sizes[i];
        }
        slot->init_params.kernelParams = slot->init_args;
        slot->init_params.extra = nullptr;
        slot->graph = g;
        ge = slot;
        c->launches = launches0;
    } else {
        u64 kk = k, nn = n;
        const T* dd = d;
        if (std::memcmp(ge->init_store + ge->k_offset, &kk, sizeof(u64)) ||
            std::memcmp(ge->init_store + ge->n_offset, &nn, sizeof(u64)) ||
            std::memcmp(ge->init_store + ge->d_offset, &dd, sizeof(const T*)) ||
            std::memcmp(ge->init_store + ge->up_offset, &up, sizeof(void*))) {   // (unchanged: no update)
            std::memcpy(ge->init_store + ge->k_offset, &kk, sizeof(u64));
            std::memcpy(ge->init_store + ge->n_offset, &nn, sizeof(u64));
            std::memcpy(ge->init_store + ge->d_offset, &dd, sizeof(const T*));
            std::memcpy(ge->init_store + ge->up_offset, &up, sizeof(void*));
            CK(cudaGraphExecKernelNodeSetParams(ge->exec, ge->init_node, &ge->init_params));
        }
    }
    ge->stamp = ++c->graph_clock;
    CK(cudaGraphLaunch(ge->exec, st));
    c->launches += ge->kernels;
    return SS_OK;
}

// top-k tail: the window's keys above the answer, then the copies of it
template <typename T>
ss_status enqueue_upper_tail(ss_context* c, bool up, cudaStream_t q) {
    if (!up) return SS_OK;
    CK(launch_pdl(upper_window_kernel<T>, dim3((u32)c->sms * 2), dim3(UW_THREADS), 0, q,
                  reinterpret_cast<const T*>(c->d_win), c->d_ctl, (const SelectResult*)c->d_res));
    CKLAUNCH("upper_window_kernel");
    CK(launch_pdl(upper_tail_fill_kernel<T>, dim3((u32)c->sms * 4), dim3(256), 0, q, c->d_ctl, c->d_res));
    CKLAUNCH("upper_tail_fill_kernel");
    c->launches += 2;
    return SS_OK;
}

// An exact call in two halves: run_exact_begin plans it and launches the
// planned chain (one graph launch) without waiting; run_exact_end waits for the
// result hand-off, runs the rare extra rounds and fills the stats.  Callers
// with independent selects (ss_select_multi) launch several on their own
// contexts and streams before waiting on any.
template <typename T>
ss_status run_exact_begin(ss_context* c, const T* d, u64 n, u64 k, void* h_result, cudaStream_t st,
                          T* up_out = nullptr) {
    typedef typename Traits<T>::Key K;
    const double t_in = c->host_timing ? now_us() : 0.0;
    // reading R7: level 0 draws s = clamp(16 b, 4096, 16384) samples (or the
    // configured size); deeper levels hold n_l ~ n / b elements and draw
    // S_DEEP = max(1024, b) -- a quarter of the sort, ~1.25x the bucket size
    // level 0 uses b_exact buckets, deeper levels b_deep (default: the same)
    const int b0 = c->cfg.b_exact, bd = c->cfg.b_deep ? c->cfg.b_deep : b0;
    const int s = sample_size(c->cfg, b0);
    const int s_deep = std::min(sample_size(c->cfg, bd), std::max(1024, bd));
    const u32 B = (u32)c->cfg.base_case;
    ss_status rc;
    if ((rc = ensure_small(c))) return rc;
    if (c->cfg.profile && (rc = prof_init(c))) return rc;
    c->launches = 0;
    c->d2h = 0;
    bool spec_plan[SS_MAX_LEVELS] = {};
    int sf_plan[SS_MAX_LEVELS] = {};
    bool dir_plan[SS_MAX_LEVELS] = {};
    double est[SS_MAX_LEVELS] = {};
    int L = expected_levels(c, n, b0, bd, B, spec_plan, sf_plan, dir_plan, est);
    const int sf = sf_plan[0] ? sf_plan[0] : fused_sample(c->cfg, 0, n);
    // top-k (§IV.I): a fused level 0 also streams the keys above its window to
    // up_out and keeps its window in d_win for the tail kernels
    const bool up = up_out && L > 0 && spec_plan[0];
    c->up_used = up;
    // workspace (reading R16: the paper keeps aux storage <= n/4 elements):
    // the two level buffers hold the planned level-1 survivors with 2x slack
    // (a level whose survivors would not fit halts before writing past them;
    // the host grows the buffers to n and re-runs it), the oracle bytes the
    // largest planned paper level
    {
        const double f0 = window_frac(spec_params(c).z, sf);
        const double est1 = L == 0 ? 0.0 : spec_plan[0] ? (double)n * 1.2 * f0 + (double)c->sms * 4096.0
                                                         : (double)n * 1.5 / b0;
        const u64 cap_el = std::min<u64>(n, std::max<u64>((u64)(2.0 * est1), (u64)1 << 20));
        for (int i = 0; i < 2; ++i)
            if ((rc = grow(c, &c->d_buf[i], &c->cap_buf[i], cap_el * sizeof(T)))) return rc;
        if (up && (rc = grow(c, &c->d_win, &c->cap_win, cap_el * sizeof(T)))) return rc;
        bool paper_deep = false;
        for (int l = 1; l < L; ++l) paper_deep |= !spec_plan[l];
        const u64 orc = L > 0 && !spec_plan[0] ? n : paper_deep ? cap_el : 0;
        if ((rc = grow(c, (void**)&c->d_oracles, &c->cap_oracles, orc + 64))) return rc;
    }
    // level 0's sample is gathered by the init kernel (spread over the grid)
    // when K1w or the wide K1 takes it from memory
    const int s_init = L > 0 && spec_plan[0] ? sf : s;
    const bool pre0 = L > 0 && (spec_plan[0] || s <= WIDE_K1_MAX_S);
    K* sample0 = pre0 ? reinterpret_cast<K*>(c->d_sample0) : nullptr;
    const int tl_on = c->cfg.profile == 3;
    // totals of every planned level are zeroed by init; levels beyond the plan
    // (the rare "incomplete" fallback) are zeroed before they run
    auto enqueue_init = [&](cudaStream_t q) -> ss_status {
        CK(launch_pdl(init_kernel<T>, dim3(pre0 ? ((u32)s_init + 255u) / 256u : 1u), dim3(256), 0, q, c->d_ctl,
                      (int)(SS_MAX_LEVELS + 1), c->d_totals, (int)((L + 1) * MAX_B), c->d_res, n, k, tl_on, d,
                      s_init, (u64)c->cfg.seed, sample0, up ? (void*)up_out : nullptr));
        CKLAUNCH("init_kernel");
        ++c->launches;
        return SS_OK;
    };
    ExactPlan plan{};
    plan.b0 = b0; plan.bd = bd; plan.s = s; plan.s_deep = s_deep; plan.B = B; plan.L = L;
    std::copy(sf_plan, sf_plan + SS_MAX_LEVELS, plan.sfs);
    std::copy(dir_plan, dir_plan + SS_MAX_LEVELS, plan.dir_plan);
    std::copy(spec_plan, spec_plan + SS_MAX_LEVELS, plan.spec_plan);
    plan.sample0 = sample0;
    plan.lev_first = 0;
    plan.out0 = up ? c->d_win : nullptr;
    // on a child context of ss_select_multi (several selects in flight
    // together) a small fused level runs on a quarter of the SMs or more,
    // ~KW_CTA_ELEMS elements per CTA, so the per-rank tails share the GPU
    // instead of queueing behind each other's full-GPU grids (measured: m = 8
    // 0.72 -> 0.68 ms; a lone small select is faster on the full grid)
    for (int l = 0; l < L && c->shared_gpu; ++l) {
        const u32 full = (u32)c->sms * (u32)KW_MINB, quarter = std::max<u32>(1, full / 4);
        const double want = std::ceil(est[l] / KW_CTA_ELEMS);
        plan.kw_grid[l] = want >= (double)full ? 0u : std::max<u32>(quarter, (u32)want);
    }
    auto enqueue_levels = [&](int lev0, cudaStream_t q) -> ss_status {
        plan.L = L;
        return enqueue_exact_levels<T>(c, plan, d, lev0, q);
    };
    // the planned part of the call: one CUDA graph launch (events of
    // profile 1/2 cannot live in a graph: those calls launch directly).  The
    // chain depends on n only through the plan (every kernel reads its level's
    // size from the LevelCtl): graphs are keyed on the plan's signature and
    // n, k, the input and output pointers are patched into the init node.
    const bool graph = c->use_graphs && c->cfg.profile != 1 && c->cfg.profile != 2;
    if (graph) {
        u64 key = 1469598103934665603ull;
        auto mix = [&](u64 v) { key = (key ^ v) * 1099511628211ull; };
        mix(1);                                // exact chain
        mix((u64)dt_code<T>());
        mix((u64)L);
        mix((u64)s_init);
        mix((u64)pre0);
        for (int l = 0; l < L; ++l)
            mix((u64)spec_plan[l] | (u64)dir_plan[l] << 1 | (u64)(u32)sf_plan[l] << 2 | (u64)plan.kw_grid[l] << 20);
        mix((u64)b0); mix((u64)bd); mix((u64)s); mix((u64)s_deep); mix((u64)B);
        mix((u64)tl_on); mix(c->cfg.seed); mix((u64)up);
        auto enqueue_all = [&](cudaStream_t q) -> ss_status {
            ss_status r2 = enqueue_init(q);
            if (!r2) r2 = enqueue_levels(0, q);
            if (!r2) r2 = enqueue_upper_tail<T>(c, up, q);
            if (!r2) r2 = enqueue_publish(c, q);
            return r2;
        };
        if (c->host_timing) c->ht[0] += now_us() - t_in;
        const double t_l = c->host_timing ? now_us() : 0.0;
        if ((rc = graph_launch<T>(c, key, n, k, d, up ? (void*)up_out : nullptr, enqueue_all, st))) return rc;
        if (c->host_timing) c->ht[1] += now_us() - t_l;
    } else {
        if ((rc = enqueue_init(st))) return rc;
        if ((rc = enqueue_levels(0, st))) return rc;
        if ((rc = enqueue_upper_tail<T>(c, up, st))) return rc;
        if ((rc = enqueue_publish(c, st))) return rc;
    }
    ExactCall& ec = c->call;
    ec.d = d;
    ec.up_out = up_out;
    ec.n = n;
    ec.k = k;
    ec.h_result = h_result;
    ec.up = up;
    ec.L = L;
    ec.B = B;
    ec.b0 = b0;
    ec.bd = bd;
    ec.t_in = t_in;
    ec.plan = plan;
    return SS_OK;
}

template <typename T>
ss_status run_exact_end(ss_context* c, cudaStream_t st) {
    ExactCall& ec = c->call;
    const T* d = reinterpret_cast<const T*>(ec.d);
    const u64 n = ec.n;
    const bool up = ec.up;
    int L = ec.L;
    const u32 B = ec.B;
    const int b0 = ec.b0, bd = ec.bd;
    const double t_in = ec.t_in;
    ExactPlan& plan = ec.plan;
    ss_status rc;
    auto enqueue_levels = [&](int lev0, cudaStream_t q) -> ss_status {
        plan.L = L;
        return enqueue_exact_levels<T>(c, plan, d, lev0, q);
    };
    const double t_w = c->host_timing ? now_us() : 0.0;
    if ((rc = wait_publish(c, st))) return rc;
    if (c->host_timing) c->ht[2] += now_us() - t_w;
    const double t_s = c->host_timing ? now_us() : 0.0;
    // rare: a fused level's window missed rank k (halt), or an unlucky sample
    // left more than B elements after the planned levels (incomplete)
    int extra_rounds = 0;
    for (;;) {
        const SelectResult& h = *c->h_res;
        if (h.halt) {
            // re-run the halted level lh the paper's way at level index lh + 2
            // (its input is level lh's input; index lh + 2 writes the buffer
            // the halted level wrote, never the one it reads)
            ++extra_rounds;
            const int lh = (h.halt & 0xFFFF) - 1, lev_new = lh + 2;
            const u64 nh = (u64)h.n_level[lh];
            if (h.halt & SS_HALT_OVERFLOW) {        // grow the level buffers to n, keeping level lh's input
                const size_t keep = lh ? (size_t)nh * sizeof(T) : 0;
                const int bi = (lh - 1) & 1;
                if ((rc = grow_keep(c, &c->d_buf[bi], &c->cap_buf[bi], n * sizeof(T), lh ? keep : 0, st))) return rc;
                if ((rc = grow_keep(c, &c->d_buf[bi ^ 1], &c->cap_buf[bi ^ 1], n * sizeof(T), 0, st))) return rc;
                if (up && (rc = grow_keep(c, &c->d_win, &c->cap_win, n * sizeof(T), lh == 1 ? keep : 0, st)))
                    return rc;
                if (up) plan.out0 = c->d_win;
            }
            if ((rc = grow(c, (void**)&c->d_oracles, &c->cap_oracles, nh + 64))) return rc;
            double m = (double)nh;
            int L2 = lev_new;
            while (m > (double)B && L2 < SS_MAX_LEVELS - 2) {
                m = m * 1.5 / (L2 ? bd : b0);
                ++L2;
            }
            if (L2 >= SS_MAX_LEVELS - 2) return fail(c, SS_ERR_INTERNAL, "recursion too deep after a halt");
            CK(cudaMemsetAsync(&c->d_res->done, 0, sizeof(int), st));
            CK(cudaMemsetAsync(&c->d_res->halt, 0, sizeof(int), st));
            CK(cudaMemcpyAsync(c->d_ctl + lev_new, c->d_ctl + lh + 1, sizeof(LevelCtl), cudaMemcpyDeviceToDevice, st));
            CK(cudaMemsetAsync(c->d_totals + (size_t)lev_new * MAX_B, 0, sizeof(u64) * MAX_B * (L2 - lev_new + 1), st));
            std::fill(plan.spec_plan, plan.spec_plan + SS_MAX_LEVELS, false);
            std::fill(plan.dir_plan, plan.dir_plan + SS_MAX_LEVELS, false);
            plan.lev_first = lev_new;
            plan.sample0 = nullptr;
            plan.L = L = L2;
            const T* first_in = lh == 0 ? d : reinterpret_cast<const T*>(level_out(c, plan, lh - 1));
            if ((rc = enqueue_exact_levels<T>(c, plan, first_in, lev_new, st))) return rc;
        } else if (!h.done) {
            ++extra_rounds;
            if (!h.incomplete || L >= SS_MAX_LEVELS - 2)
                return fail(c, SS_ERR_INTERNAL, "recursion did not terminate");
            CK(cudaMemsetAsync(&c->d_res->incomplete, 0, sizeof(int), st));
            CK(cudaMemsetAsync(c->d_totals + (size_t)L * MAX_B, 0, sizeof(u64) * MAX_B, st));
            const int lev0 = L;
            L = L + 1;
            if ((rc = enqueue_levels(lev0, st))) return rc;
        } else {
            break;
        }
        if ((rc = enqueue_publish(c, st))) return rc;
        if ((rc = wait_publish(c, st))) return rc;
    }
    if (up && extra_rounds) {                  // the tail kernels of the graph saw an unfinished call
        if ((rc = enqueue_upper_tail<T>(c, up, st))) return rc;
        if ((rc = enqueue_publish(c, st))) return rc;
        if ((rc = wait_publish(c, st))) return rc;
    }
    const SelectResult& r = *c->h_res;
    std::memcpy(ec.h_result, &r.bits, sizeof(T));
    ss_stats& S = c->stats;
    std::memset(&S, 0, sizeof(S));
    S.levels = r.levels;
    S.equality_exit = r.eq_exit;
    S.lut_ctas = (int32_t)r.lut_stats[0];
    S.lut_marker = (int32_t)r.lut_stats[1];
    S.spec_levels = (int32_t)r.spec_levels;
    S.fused_levels = (int32_t)r.fused_levels;
    S.incomplete_rounds = extra_rounds;
    S.workspace_bytes = (int64_t)workspace_bytes(c);
    if (r.spec_err) return fail(c, SS_ERR_INTERNAL, "fused filter: captured count != window total");
    double bytes = 0;
    const double Sz = (double)sizeof(T);
    for (int l = 0; l <= r.levels && l < SS_MAX_LEVELS; ++l) {
        S.n_level[l] = r.n_level[l];
        S.bucket[l] = r.bucket[l];
    }
    for (int l = 0; l < r.levels; ++l) {
        const double nl = (double)r.n_level[l], nn = (double)r.n_level[l + 1];
        const bool last_eq = r.eq_exit && l == r.levels - 1;
        if (r.spec_levels >> l & 1) {
            bytes += Sz * nl;                           // the fused pass reads the level once
            if (!last_eq && (r.fused_levels >> l & 1)) bytes += Sz * nn;   // and writes the window
            continue;                                   // (a miss halts: the level is re-run from its input)
        }
        bytes += Sz * nl + nl;                          // count: read + oracle write
        if (!last_eq) bytes += nl + 2.0 * Sz * nn;      // oracle read + gather + write
    }
    if (!r.eq_exit) bytes += Sz * (double)r.n_level[r.levels];  // base case reads its input
    S.bytes_algorithmic = bytes;
    S.launches = c->launches;
    S.h2d_bytes = c->h2d;
    S.d2h_bytes = c->d2h;
    c->launches_total += c->launches;
    c->calls_total += 1;
    prof_collect(c);
    if (c->host_timing) {
        c->ht[3] += now_us() - t_s;
        c->ht[4] += now_us() - t_in;
        ++c->ht_n;
    }
    return SS_OK;
}

template <typename T>
ss_status run_exact(ss_context* c, const T* d, u64 n, u64 k, void* h_result, cudaStream_t st, T* up_out = nullptr) {
    const ss_status rc = run_exact_begin<T>(c, d, n, k, h_result, st, up_out);
    return rc ? rc : run_exact_end<T>(c, st);
}

template <typename T>
ss_status run_approx(ss_context* c, const T* d, u64 n, u64 k, int b, void* h_result, int64_t* h_rank,
                     cudaStream_t st) {
    typedef typename Traits<T>::Key K;
    const int H = log2i(b);
    const int s = c->cfg.sample_size > 0 ? c->cfg.sample_size : sample_size(c->cfg, b);
    if (s < b) return fail(c, SS_ERR_INVALID_ARGUMENT, "sample_size must be >= b");
    ss_status rc;
    if ((rc = ensure_small(c))) return rc;
    if (c->cfg.profile && (rc = prof_init(c))) return rc;
    c->launches = 0;
    c->d2h = 0;
    const bool merge = s > WIDE_K1_MAX_S && s % (int)K1C_CHUNK == 0;   // chunk sort + merge rank
    const bool wide = s <= WIDE_K1_MAX_S || merge;
    K* sample0 = s <= WIDE_K1_MAX_S ? reinterpret_cast<K*>(c->d_sample0) : nullptr;
    // fused one-pass window (approx_window in kernels.cuh) on large inputs;
    // the paper's full count runs only if it cannot decide
    const SpecCfg sp = spec_params(c);
    const bool fw = sp.min_n != ~0ull && n >= sp.min_n;
    K* sorted0 = reinterpret_cast<K*>(c->d_sorted);
    const int tl_on = c->cfg.profile == 3;
    auto enqueue_head = [&](cudaStream_t q) -> ss_status {   // init, the sorted sample
        CK(launch_pdl(init_kernel<T>, dim3(sample0 ? ((u32)s + 255u) / 256u : 1u), dim3(256), 0, q, c->d_ctl, 2,
                      c->d_totals, (int)MAX_B, c->d_res, n, k, tl_on, d, s, (u64)c->cfg.seed, sample0,
                      (void*)nullptr));
        CKLAUNCH("init_kernel");
        ++c->launches;
        if (merge) {
            K* chunks = reinterpret_cast<K*>(c->d_sorted) + MAX_S;   // level 1's slot: scratch here
            mark(c, 0, 0, 0, q);
            CK(launch_pdl(sample_chunk_sort_kernel<T>, dim3((u32)s / K1C_CHUNK), dim3(1024), K1C_CHUNK * sizeof(K), q,
                          d, c->d_ctl, c->d_res, chunks, (u64)c->cfg.seed, 0));
            CKLAUNCH("sample_chunk_sort_kernel");
            CK(launch_pdl(sample_merge_rank_kernel<T>, dim3((u32)s / 1024u), dim3(1024), (size_t)s * sizeof(K), q,
                          c->d_ctl, c->d_res, chunks, s, sorted0, 0));
            CKLAUNCH("sample_merge_rank_kernel");
            mark(c, 0, 0, 1, q);
            c->launches += 2;
        } else if (wide) {
            if ((rc = launch_k1_wide<T>(c, d, 0, s, 0, q, sample0))) return rc;
        } else if ((rc = launch_k1<T>(c, d, 0, s, b, 0, 0, 0, q, fw ? sorted0 : nullptr))) {
            return rc;
        }
        return SS_OK;
    };
    CountArgs a{};
    if (wide) a.image = c->d_image;
    a.ctl = c->d_ctl;
    a.ctl_next = c->d_ctl + 1;
    a.res = c->d_res;
    a.tree = reinterpret_cast<K*>(c->d_tree);
    a.spl = reinterpret_cast<K*>(c->d_spl);
    a.eq = c->d_eq;
    a.oracles = nullptr;
    a.cta_counts = nullptr;
    a.totals = c->d_totals;
    a.lut = c->cfg.classify == 0;
    a.lut_stats = c->d_res->lut_stats;
    a.level = 0;
    a.tail = TAIL_APPROX;
    auto enqueue_window = [&](cudaStream_t q) -> ss_status {
        CountArgs w = a;
        w.sorted = sorted0;
        w.s = s;
        w.b = b;
        w.spec_min_n = sp.min_n;
        w.spec_z = sp.z;
        w.spec_max_frac = 1.0f;
        mark(c, 0, 1, 0, q);
        if ((rc = launch_window<T, true>(c, H, d, w, q))) return rc;
        mark(c, 0, 1, 1, q);
        ++c->launches;
        return SS_OK;
    };
    auto enqueue_count = [&](cudaStream_t q) -> ss_status {   // the paper's level-0 count (+ K3/K4 tail)
        if (!fw) mark(c, 0, 1, 0, q);
        if (wide && (rc = launch_image<T>(c, H, 0, s, 0, q))) return rc;
        if ((rc = launch_count<T>(c, H, d, a, q))) return rc;
        if (!fw) mark(c, 0, 1, 1, q);
        ++c->launches;
        return SS_OK;
    };
    const bool graph = fw && c->use_graphs && c->cfg.profile != 1 && c->cfg.profile != 2;
    if (graph) {
        // the one-pass window decides almost always: one graph (init, sample
        // sort, window, publish); the count runs after the hand-off only when
        // the window could not decide (the kernels read n and k from LevelCtl)
        u64 key = 1469598103934665603ull;
        auto mix = [&](u64 v) { key = (key ^ v) * 1099511628211ull; };
        mix(2);                                // approximate chain
        mix((u64)dt_code<T>()); mix((u64)s); mix((u64)b); mix((u64)tl_on); mix(c->cfg.seed);
        mix((u64)merge); mix((u64)wide); mix((u64)c->cfg.classify);
        auto enqueue_all = [&](cudaStream_t q) -> ss_status {
            ss_status r2 = enqueue_head(q);
            if (!r2) r2 = enqueue_window(q);
            if (!r2) r2 = enqueue_publish(c, q);
            return r2;
        };
        if ((rc = graph_launch<T>(c, key, n, k, d, nullptr, enqueue_all, st))) return rc;
        if ((rc = wait_publish(c, st))) return rc;
        if (!c->h_res->done) {
            if ((rc = enqueue_count(st))) return rc;
            if ((rc = enqueue_publish(c, st))) return rc;
            if ((rc = wait_publish(c, st))) return rc;
        }
    } else {
        if ((rc = enqueue_head(st))) return rc;
        if (fw && (rc = enqueue_window(st))) return rc;
        if ((rc = enqueue_count(st))) return rc;
        if ((rc = enqueue_publish(c, st))) return rc;
        if ((rc = wait_publish(c, st))) return rc;
    }
    const SelectResult& r = *c->h_res;
    if (!r.done) return fail(c, SS_ERR_INTERNAL, "approximate select produced no result");
    std::memcpy(h_result, &r.bits, sizeof(T));
    if (h_rank) *h_rank = r.rank;
    ss_stats& S = c->stats;
    std::memset(&S, 0, sizeof(S));
    S.levels = 1;
    S.spec_levels = (int32_t)r.spec_levels;
    S.fused_levels = (int32_t)r.fused_levels;
    S.lut_ctas = (int32_t)r.lut_stats[0];
    S.lut_marker = (int32_t)r.lut_stats[1];
    S.n_level[0] = (int64_t)n;
    S.bucket[0] = (int32_t)r.split_index;
    S.bytes_algorithmic = (double)sizeof(T) * (double)n;
    S.launches = c->launches;
    S.h2d_bytes = c->h2d;
    S.d2h_bytes = c->d2h;
    c->launches_total += c->launches;
    c->calls_total += 1;
    prof_collect(c);
    return SS_OK;
}

template <typename T>
ss_status launch_ablation(ss_context* c, const T* d, u64 n, const void* tree, int h, int mode, u64* totals,
                          cudaStream_t st) {
    typedef typename Traits<T>::Key K;
    const u32 grid = (u32)c->sms * 2;
    const K* tr = (const K*)tree;
    unsigned long long* tt = (unsigned long long*)totals;
    switch (mode) {
        case ABL_SHARED: ablation_count_kernel<T, ABL_SHARED><<<grid, ABL_THREADS, 0, st>>>(d, n, tr, h, tt); break;
        case ABL_SHARED_WA: ablation_count_kernel<T, ABL_SHARED_WA><<<grid, ABL_THREADS, 0, st>>>(d, n, tr, h, tt); break;
        case ABL_SHARED_FIG6: ablation_count_kernel<T, ABL_SHARED_FIG6><<<grid, ABL_THREADS, 0, st>>>(d, n, tr, h, tt); break;
        case ABL_GLOBAL: ablation_count_kernel<T, ABL_GLOBAL><<<grid, ABL_THREADS, 0, st>>>(d, n, tr, h, tt); break;
        default: ablation_count_kernel<T, ABL_GLOBAL_WA><<<grid, ABL_THREADS, 0, st>>>(d, n, tr, h, tt); break;
    }
    CK(cudaGetLastError());
    c->launches_total += 1;
    return SS_OK;
}

// Top-k fusion (§IV.I; reading R22).  One pass (upper_onepass, the
// paper's design: the filter "copies not only elements from the target
// bucket, but also from all buckets containing larger elements"): the fused
// level 0 streams the keys above its window straight to d_out while it copies
// the window; the select finishes on the window, and the tail kernels append
// the window's keys > result and the copies of result -- all inside the call's
// graph.  Otherwise (level 0 not a fused hit, or upper_onepass = 0): the exact
// select, then one streaming pass that appends the elements > result to d_out,
// then the copies of result that fill it up to n-k.
#ifndef SS_UPPER_ONEPASS_MAX_FRAC
#define SS_UPPER_ONEPASS_MAX_FRAC 0.25
#endif
constexpr double UPPER_ONEPASS_MAX_FRAC = SS_UPPER_ONEPASS_MAX_FRAC;
template <typename T>
ss_status run_upper(ss_context* c, const T* d, u64 n, u64 k, T* d_out, void* h_result, cudaStream_t st) {
    typedef typename Traits<T>::Key K;
    // the one-pass path appends the keys above level 0's window with one
    // global atomic per warp flush: measured at n = 2^28 fp32 it wins while
    // the output is small and loses to the two passes (select + a streaming
    // gather with CTA-staged appends) once n - k is a large part of n
    const bool one = c->cfg.upper_onepass && (double)(n - k) <= UPPER_ONEPASS_MAX_FRAC * (double)n;
    ss_status rc = run_exact<T>(c, d, n, k, h_result, st, one ? d_out : nullptr);
    if (rc) return rc;
    const u64 m = n - k;
    {
        const SelectResult& r = *c->h_res;
        const bool l0_ok = (r.spec_levels & 1) && ((r.fused_levels & 1) || (r.eq_exit && r.levels == 1));
        if (c->up_used && l0_ok) {
            const u64 greater = r.upper_cnt;
            if (greater >= m && m > 0) return fail(c, SS_ERR_INTERNAL, "select_upper: #{x > result} >= n-k");
            c->stats.upper_greater = (int64_t)greater;
            c->stats.upper_onepass = 1;
            // + the output, + the tail's read of level 0's window
            c->stats.bytes_algorithmic += (double)sizeof(T) * ((double)m + (double)r.n_level[1] * (r.fused_levels & 1));
            return SS_OK;
        }
    }
    if (!c->d_upper_cnt) CK(cudaMalloc(&c->d_upper_cnt, sizeof(unsigned long long)));
    const bool prof = c->cfg.profile != 0;
    if (prof && !c->ev_upper[0]) {
        CK(cudaEventCreate(&c->ev_upper[0]));
        CK(cudaEventCreate(&c->ev_upper[1]));
    }
    T v;
    std::memcpy(&v, h_result, sizeof(T));
    K vb;
    std::memcpy(&vb, &v, sizeof(T));
    const K kv = Traits<T>::to_key(vb);
    CK(cudaMemsetAsync(c->d_upper_cnt, 0, sizeof(unsigned long long), st));
    constexpr u64 EPV = 16 / sizeof(T);
    const u64 tiles = (n / EPV + (u64)UG_THREADS * UG_VEC - 1) / ((u64)UG_THREADS * UG_VEC);
    const u32 grid = (u32)std::max<u64>(1, std::min<u64>(tiles, (u64)c->sms * UG_MINB));
    if (prof) CK(cudaEventRecord(c->ev_upper[0], st));
    if (!(c->upper_attr >> dt_code<T>() & 1)) {   // stage > 48 KB-safe default: opt in once per (context device, dtype)
        CK(cudaFuncSetAttribute(upper_gather_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, UG_STAGE_BYTES));
        c->upper_attr |= 1u << dt_code<T>();
    }
    upper_gather_kernel<T><<<grid, UG_THREADS, UG_STAGE_BYTES, st>>>(d, n, kv, d_out, c->d_upper_cnt);
    CK(cudaGetLastError());
    if (prof) CK(cudaEventRecord(c->ev_upper[1], st));
    upper_fill_kernel<T><<<(u32)c->sms * 4, 256, 0, st>>>(d_out, m, v, c->d_upper_cnt);
    CK(cudaGetLastError());
    unsigned long long greater = 0;
    CK(cudaMemcpyAsync(&greater, c->d_upper_cnt, sizeof(greater), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    if (greater >= m && m > 0) return fail(c, SS_ERR_INTERNAL, "select_upper: #{x > result} >= n-k");
    c->stats.upper_greater = (int64_t)greater;
    c->stats.bytes_algorithmic += (double)sizeof(T) * ((double)n + (double)m);   // one read + the output
    c->stats.launches += 2;
    c->stats.d2h_bytes += (int64_t)sizeof(greater);
    c->launches_total += 2;
    if (prof) {
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, c->ev_upper[0], c->ev_upper[1]));
        c->stats.ms_upper_gather = ms;
    }
    return SS_OK;
}

// Multi-rank selection (§VI "multiple ... selection",
// reading R23): m ranks share one sample, one splitter tree and ONE count
// pass over the input (the dominant K2 pass, §IV.G); one launch searches the
// bucket of every rank; every distinct bucket holding a rank is extracted in
// one pass over the oracle bytes (multi_filter_kernel); each rank then
// finishes with the single-rank select on its bucket (rank k - r_j, Fig. 1).
// An equality bucket answers its ranks with its splitter (§IV.C).  One host
// round trip (the search rows, which size the extraction); the per-rank
// selects run as exact calls on child contexts, each on its own stream, all
// launched (one graph launch each) before the host waits on any.
constexpr int MULTI_MAX = 1024;
constexpr u64 MULTI_MIN_N = (u64)1 << 20;   // below: one select per rank is cheaper
// Below 4 ranks the per-rank fused selects win: each is one ~0.22 ms pass at
// n = 2^28 fp32, the shared path's count + extraction alone ~0.33 ms.
constexpr int MULTI_MIN_M = 4;

// the child contexts (same device and config, no profiling) and their streams
inline ss_status multi_children(ss_context* c, int want) {
    if (!c->ev_mfork) CK(cudaEventCreateWithFlags(&c->ev_mfork, cudaEventDisableTiming));
    ss_config cc = c->cfg;
    cc.profile = 0;
    for (int i = 0; i < want && i < MULTI_CH; ++i) {
        if (!c->mchild[i]) {
            ss_status rc = ss_create(c->device, &c->mchild[i]);
            if (rc) return fail(c, rc, "select_multi: child context");
            c->mchild[i]->shared_gpu = true;
            CK(cudaStreamCreateWithFlags(&c->mchild_st[i], cudaStreamNonBlocking));
            CK(cudaEventCreateWithFlags(&c->ev_mjoin[i], cudaEventDisableTiming));
        }
        if (std::memcmp(&c->mchild[i]->cfg, &cc, sizeof(cc))) {
            ss_status rc = ss_set_config(c->mchild[i], &cc);
            if (rc) return fail(c, rc, c->mchild[i]->err.c_str());
        }
    }
    return SS_OK;
}

// The per-rank selects of a multi-rank call: exact calls on child contexts,
// MULTI_CH at a time, each on its own stream after `st`'s work so far; the
// caller's stream waits for them at the end.
struct MultiTail {
    const void* in;
    u64 n, k;
    unsigned char* out;   // host result slot
};
// After a failed tail the children may hold launched calls nobody waits for
// (their publish counters would run ahead of the host's): drop them all; the
// next multi-rank call creates fresh ones.
inline void multi_children_reset(ss_context* c) {
    for (int i = 0; i < MULTI_CH; ++i) {
        if (c->mchild_st[i]) cudaStreamSynchronize(c->mchild_st[i]);
        if (c->mchild[i]) ss_destroy(c->mchild[i]);
        if (c->mchild_st[i]) cudaStreamDestroy(c->mchild_st[i]);
        if (c->ev_mjoin[i]) cudaEventDestroy(c->ev_mjoin[i]);
        c->mchild[i] = nullptr;
        c->mchild_st[i] = nullptr;
        c->ev_mjoin[i] = nullptr;
    }
}

template <typename T>
ss_status run_tails(ss_context* c, const std::vector<MultiTail>& tails, cudaStream_t st, double* bytes,
                    int* launches) {
    const int nt = (int)tails.size();
    if (!nt) return SS_OK;
    ss_status rc;
    if ((rc = multi_children(c, nt))) return rc;
    auto failed = [&](ss_context* ch, ss_status r) -> ss_status {
        const std::string msg = ch->err;
        multi_children_reset(c);
        return fail(c, r, msg.c_str());
    };
    CK(cudaEventRecord(c->ev_mfork, st));
    const int nch = std::min(nt, MULTI_CH);
    for (int w0 = 0; w0 < nt; w0 += nch) {
        const int wn = std::min(nch, nt - w0);
        for (int q = 0; q < wn; ++q) {
            const MultiTail& t = tails[w0 + q];
            ss_context* ch = c->mchild[q];
            if (w0 == 0) CK(cudaStreamWaitEvent(c->mchild_st[q], c->ev_mfork, 0));
            if ((rc = run_exact_begin<T>(ch, reinterpret_cast<const T*>(t.in), t.n, t.k, t.out, c->mchild_st[q])))
                return failed(ch, rc);
        }
        for (int q = 0; q < wn; ++q) {
            ss_context* ch = c->mchild[q];
            if ((rc = run_exact_end<T>(ch, c->mchild_st[q]))) return failed(ch, rc);
            *bytes += ch->stats.bytes_algorithmic;
            *launches += ch->stats.launches;
        }
    }
    for (int q = 0; q < nch; ++q) {            // later work on the caller's stream follows the tails
        CK(cudaEventRecord(c->ev_mjoin[q], c->mchild_st[q]));
        CK(cudaStreamWaitEvent(st, c->ev_mjoin[q], 0));
    }
    return SS_OK;
}

template <typename T>
ss_status run_multi(ss_context* c, ss_dtype dt, const T* d, u64 n, int m, const int64_t* ks, void* h_res,
                    cudaStream_t st) {
    typedef typename Traits<T>::Key K;
    unsigned char* outb = (unsigned char*)h_res;
    ss_status rc;
    double bytes = 0;
    int launches = 0;
    if (n < MULTI_MIN_N || m < MULTI_MIN_M) {
        for (int i = 0; i < m; ++i) {
            if ((rc = run_exact<T>(c, d, n, (u64)ks[i], outb + (size_t)i * sizeof(T), st))) return rc;
            bytes += c->stats.bytes_algorithmic;
            launches += c->stats.launches;
        }
        c->stats.bytes_algorithmic = bytes;
        c->stats.launches = launches;
        return SS_OK;
    }
    const int b = std::min(c->cfg.b_exact, 256);
    const int s = c->cfg.sample_size > 0 ? c->cfg.sample_size : sample_size(c->cfg, b);
    // device scratch layout (8-byte slots)
    const size_t o_keys = 0, o_tree = o_keys + (size_t)MAX_S * 8, o_spl = o_tree + (size_t)MAX_B * 8,
                 o_tot = o_spl + (size_t)MAX_B * 8, o_srch = o_tot + (size_t)MAX_B * 8,
                 o_ks = o_srch + (size_t)MULTI_MAX * MS_ROW * 8, o_cnt = o_ks + (size_t)MULTI_MAX * 8,
                 o_eq = o_cnt + (size_t)MULTI_MAX * 8, o_lut = o_eq + MAX_B, o_sb = o_lut + 256,
                 o_sbase = o_sb + (size_t)MF_MAX_SLOTS * 4, scratch = o_sbase + (size_t)MF_MAX_SLOTS * 8;
    // pinned host staging (ranks, search rows, slot tables): the copies stay asynchronous
    const size_t p_ks = 0, p_srch = p_ks + (size_t)MULTI_MAX * 8, p_lut = p_srch + (size_t)MULTI_MAX * MS_ROW * 8,
                 p_sb = p_lut + 256, p_sbase = p_sb + (size_t)MF_MAX_SLOTS * 4,
                 pin_bytes = p_sbase + (size_t)MF_MAX_SLOTS * 8;
    if (!c->d_multi_scratch) CK(cudaMalloc(&c->d_multi_scratch, scratch));
    if (!c->h_mpin) CK(cudaMallocHost(&c->h_mpin, pin_bytes));
    unsigned char* S0 = c->d_multi_scratch;
    unsigned char* P0 = c->h_mpin;
    if ((rc = ensure_small(c))) return rc;
    if ((rc = grow(c, (void**)&c->d_oracles, &c->cap_oracles, (size_t)n + 64))) return rc;
    std::memcpy(P0 + p_ks, ks, sizeof(int64_t) * (size_t)m);
    CK(cudaMemcpyAsync(S0 + o_ks, P0 + p_ks, sizeof(int64_t) * (size_t)m, cudaMemcpyHostToDevice, st));
    if ((rc = ss_step_sample(c, dt, d, (int64_t)n, 0, 0, s, S0 + o_keys, st))) return rc;
    if ((rc = ss_step_tree(c, dt, S0 + o_keys, s, b, 1, S0 + o_tree, S0 + o_spl, S0 + o_eq, st))) return rc;
    if ((rc = ss_step_count(c, dt, d, (int64_t)n, S0 + o_tree, b, (uint64_t*)(S0 + o_tot), c->d_oracles, st)))
        return rc;
    multi_search_kernel<T><<<1, 256, 0, st>>>((const u64*)(S0 + o_tot), (u32)b, (const long long*)(S0 + o_ks), m,
                                               S0 + o_eq, (const K*)(S0 + o_spl), (long long*)(S0 + o_srch));
    CK(cudaGetLastError());
    const int64_t* sr = reinterpret_cast<const int64_t*>(P0 + p_srch);
    CK(cudaMemcpyAsync(P0 + p_srch, S0 + o_srch, sizeof(int64_t) * MS_ROW * (size_t)m, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));             // the one host round trip: the rows size the extraction
    int step_launches = 4;
    bytes += (double)sizeof(T) * n + (double)n;   // count: read + oracle bytes
    // distinct buckets, in bucket order; regions of d_multi for the non-equality ones
    std::vector<int> order(m);
    for (int i = 0; i < m; ++i) order[i] = i;
    std::sort(order.begin(), order.end(),
              [&](int a, int bb) { return sr[MS_ROW * (size_t)a] < sr[MS_ROW * (size_t)bb]; });
    std::vector<int64_t> bucket_off(MAX_B, -1);
    size_t total = 0;
    for (int i : order) {
        const int64_t j = sr[MS_ROW * (size_t)i], nj = sr[MS_ROW * (size_t)i + 2], eq = sr[MS_ROW * (size_t)i + 3];
        if (eq || bucket_off[j] >= 0) continue;
        bucket_off[j] = (int64_t)total;
        total += (size_t)nj;
    }
    if ((rc = grow(c, &c->d_multi, &c->cap_multi, std::max<size_t>(total, 1) * sizeof(T)))) return rc;
    u32* slot_bucket = reinterpret_cast<u32*>(P0 + p_sb);
    u64* slot_base = reinterpret_cast<u64*>(P0 + p_sbase);
    int nb = 0;
    for (int j = 0; j < b; ++j)
        if (bucket_off[j] >= 0) {
            if (nb < MF_MAX_SLOTS) {
                slot_bucket[nb] = (u32)j;
                slot_base[nb] = (u64)bucket_off[j];
            }
            ++nb;
        }
    if (nb >= 2 && nb <= MF_MAX_SLOTS && b <= 256) {
        // one pass over the oracle bytes extracts every wanted bucket
        uint8_t* slot_of = P0 + p_lut;
        std::memset(slot_of, 0xFF, 256);
        for (int i = 0; i < nb; ++i) slot_of[slot_bucket[i]] = (uint8_t)i;
        CK(cudaMemcpyAsync(S0 + o_lut, P0 + p_lut, 256 + (size_t)MF_MAX_SLOTS * 12, cudaMemcpyHostToDevice, st));
        if (!(c->mf_attr >> dt_code<T>() & 1)) {
            CK(cudaFuncSetAttribute(multi_filter_kernel<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)MF_SMEM));
            c->mf_attr |= 1u << dt_code<T>();
        }
        multi_filter_kernel<T><<<c->step_grid, MF_THREADS, MF_SMEM, st>>>(
            d, n, c->d_oracles, c->d_cta_counts, (u32)b, c->step_grid, S0 + o_lut, (const u32*)(S0 + o_sb),
            (const u64*)(S0 + o_sbase), (u32)nb, (T*)c->d_multi);
        CK(cudaGetLastError());
        step_launches += 1;
        bytes += (double)n;    // one read of the oracle bytes
    } else {
        for (int j = 0; j < b; ++j) {
            if (bucket_off[j] < 0) continue;
            if ((rc = ss_step_filter(c, dt, d, (int64_t)n, c->d_oracles, (int32_t)j,
                                     (T*)c->d_multi + bucket_off[j], (uint64_t*)(S0 + o_cnt), st)))
                return rc;
            step_launches += 1;
            bytes += (double)n;   // each extraction reads the oracle bytes
        }
    }
    // equality buckets: the value is splitter s_j (row field 4)
    std::vector<int> tails;
    for (int i = 0; i < m; ++i) {
        const int64_t* row = sr + MS_ROW * (size_t)i;
        if (row[3]) {
            std::memcpy(outb + (size_t)i * sizeof(T), &row[4], sizeof(T));
        } else {
            bytes += 2.0 * sizeof(T) * (double)row[2];
            tails.push_back(i);
        }
    }
    // the remaining levels of each rank: single-rank selects on its bucket
    std::vector<MultiTail> tl;
    for (int i : tails) {
        const int64_t* row = sr + MS_ROW * (size_t)i;
        tl.push_back({(const T*)c->d_multi + bucket_off[row[0]], (u64)row[2], (u64)row[1],
                      outb + (size_t)i * sizeof(T)});
    }
    if ((rc = run_tails<T>(c, tl, st, &bytes, &launches))) return rc;
    c->launches_total += step_launches;
    std::memset(&c->stats, 0, sizeof(c->stats));
    c->stats.levels = 1;
    c->stats.n_level[0] = (int64_t)n;
    c->stats.n_level[1] = (int64_t)total;
    c->stats.bytes_algorithmic = bytes;
    c->stats.launches = launches + step_launches;
    c->stats.h2d_bytes = (int64_t)(sizeof(int64_t) * (size_t)m);
    c->stats.d2h_bytes = (int64_t)(sizeof(int64_t) * MS_ROW * (size_t)m);
    return SS_OK;
}

// QuickSelect baseline (quickselect.cuh).
// Levels are enqueued in batches (the first sized to the expected depth, then
// QS_BATCH; pivot -> partition -> decide,
// each early-exiting once the answer is known); one 8-byte-aligned header
// copy per batch tells the host whether to enqueue more.
constexpr int QS_BATCH = 4;
template <typename T>
ss_status run_quick(ss_context* c, const T* d, u64 n, u64 k, void* h_result, int64_t* h_n_level, int32_t cap,
                    int32_t* h_levels, cudaStream_t st) {
    if (n >= ((u64)1 << 32)) return fail(c, SS_ERR_INVALID_ARGUMENT, "quickselect: n must be < 2^32");
    if (!c->d_qs) {
        CK(cudaMalloc(&c->d_qs, sizeof(QsCtl)));
        CK(cudaMallocHost(&c->h_qs, sizeof(QsCtl)));
        CK(cudaEventCreate(&c->ev_qs[0]));
        CK(cudaEventCreate(&c->ev_qs[1]));
    }
    const size_t need = (size_t)n * sizeof(T);
    if (c->cap_qsbuf < need) {
        for (auto& p : c->d_qsbuf) {
            cudaFree(p);
            p = nullptr;
        }
        c->cap_qsbuf = 0;
        CK(cudaMalloc(&c->d_qsbuf[0], need));
        CK(cudaMalloc(&c->d_qsbuf[1], need));
        c->cap_qsbuf = need;
    }
    const u32 B = (u32)std::min<int64_t>(std::max<int64_t>(c->cfg.base_case, 1), (int64_t)BASE_THREADS * BASE_PT);
    constexpr int IPT = (sizeof(T) == 8 && QP_IPT > 16) ? 16 : QP_IPT;   // 8-byte tiles: <= 32 KB static stage
    const u32 grid = (u32)c->sms * qp_minb<T>();
    T* buf[2] = {(T*)c->d_qsbuf[0], (T*)c->d_qsbuf[1]};
    const bool prof = c->cfg.profile != 0;
    if (prof) CK(cudaEventRecord(c->ev_qs[0], st));
    qs_init_kernel<<<1, 1, 0, st>>>(c->d_qs, n, k);
    CK(cudaGetLastError());
    int launches = 1, level = 0, batches = 0;
    // first batch: the expected depth log2(n / B) + 2 of a median pivot; then QS_BATCH at a time
    int batch = 2;
    for (u64 m = n; m > B; m >>= 1) ++batch;
    for (;; batch = QS_BATCH) {
        for (int q = 0; q < batch; ++q, ++level) {
            const T* bin = buf[(level + 1) & 1];      // level l reads buffer (l-1)&1 (level 0: d)
            qs_pivot_kernel<T><<<1, 1024, (size_t)B * sizeof(typename Traits<T>::Key), st>>>(d, bin, c->d_qs, B,
                                                                                          c->cfg.seed, level);
            qs_partition_kernel<T, IPT><<<grid, QP_THREADS, 0, st>>>(d, bin, buf[level & 1], c->d_qs, level);
            qs_decide_kernel<T><<<1, 1, 0, st>>>(c->d_qs, level);
            CK(cudaGetLastError());
            launches += 3;
        }
        CK(cudaMemcpyAsync(c->h_qs, c->d_qs, offsetof(QsCtl, n_level), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        ++batches;
        if (c->h_qs->done) break;
        if (level + QS_BATCH > QS_MAX_LEVELS) return fail(c, SS_ERR_INTERNAL, "quickselect: level limit reached");
    }
    if (prof) CK(cudaEventRecord(c->ev_qs[1], st));
    CK(cudaMemcpyAsync(c->h_qs, c->d_qs, sizeof(QsCtl), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    const QsCtl& h = *c->h_qs;
    std::memcpy(h_result, &h.bits, sizeof(T));
    const int lv = (int)h.levels;
    const int nvalid = lv + (h.eq_exit ? 0 : 1);   // an equality exit has no base-case level
    double bytes = 0;
    for (int l = 0; l < lv; ++l) bytes += (double)sizeof(T) * ((double)h.n_level[l] + (double)h.n_out[l]);
    if (!h.eq_exit) bytes += (double)sizeof(T) * (double)h.n_level[lv];   // base case reads its level
    if (h_levels) *h_levels = lv;
    if (h_n_level)
        for (int l = 0; l < cap && l < QS_MAX_LEVELS; ++l)
            h_n_level[l] = l < nvalid ? (int64_t)h.n_level[l] : 0;
    c->stats = ss_stats{};
    c->stats.levels = std::min(lv, SS_MAX_LEVELS - 1);
    c->stats.equality_exit = (int)h.eq_exit;
    for (int l = 0; l < nvalid && l < SS_MAX_LEVELS; ++l) c->stats.n_level[l] = (int64_t)h.n_level[l];
    c->stats.bytes_algorithmic = bytes;
    c->stats.launches = launches;
    c->stats.d2h_bytes = (int64_t)(offsetof(QsCtl, n_level) * (size_t)batches + sizeof(QsCtl));
    c->launches_total += launches;
    if (prof) {
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, c->ev_qs[0], c->ev_qs[1]));
        c->stats.ms_quick = ms;
    }
    return SS_OK;
}



size_t workspace_bytes(const ss_context* c) {
    size_t b = c->cap_oracles + c->cap_buf[0] + c->cap_buf[1] + c->cap_win + c->cap_stage + c->cap_multi + 2 * c->cap_qsbuf +
               c->cap_gather[0] + c->cap_gather[1] + c->cap_dist;
    if (c->d_ctl)   // the fixed per-context arrays (ensure_small)
        b += sizeof(LevelCtl) * (SS_MAX_LEVELS + 1) + sizeof(SelectResult) + sizeof(u64) * SS_MAX_LEVELS * MAX_B +
             sizeof(u32) * (size_t)MAX_GRID * MAX_B + 2 * sizeof(u64) * SS_MAX_LEVELS * MAX_B +
             (size_t)SS_MAX_LEVELS * MAX_B + sizeof(u64) * SS_MAX_LEVELS * MAX_S + sizeof(u64) * MAX_S +
             sizeof(u64) * SS_MAX_LEVELS * MAX_S + K2_IMAGE_SLOT * SS_MAX_LEVELS;
    return b;
}

#include "sharded.cuh"

}  // namespace

#include "ops.cuh"
