// abi.cu -- the C ABI of include/sampleselect.h: argument checks, context
// lifetime and configuration, and dispatch of each call to the per-dtype
// operations (op_* in ops.cuh, compiled in inst_<dtype>.cu).
#define SS_ABI_TU 1
#include "driver.cuh"

using namespace ss;

namespace {
ss_status check_common(ss_context* c, ss_dtype dt, const void* p, int64_t n, int64_t k, void* out) {
    if (!c) return SS_ERR_INVALID_ARGUMENT;
    if (!dt_size(dt)) return fail(c, SS_ERR_INVALID_ARGUMENT, "unknown dtype");
    if (!p || !out) return fail(c, SS_ERR_INVALID_ARGUMENT, "NULL pointer");
    if (n < 1) return fail(c, SS_ERR_INVALID_ARGUMENT, "n must be >= 1");
    if (k < 0 || k >= n) return fail(c, SS_ERR_INVALID_ARGUMENT, "k must be in [0, n)");
    if (((uintptr_t)p) % dt_size(dt)) return fail(c, SS_ERR_INVALID_ARGUMENT, "data not naturally aligned");
    return SS_OK;
}

template <typename F>
ss_status dispatch(ss_dtype dt, F&& f) {
    switch (dt) {
    case SS_FLOAT32: return f((float*)nullptr);
    case SS_FLOAT64: return f((double*)nullptr);
    case SS_INT32: return f((int*)nullptr);
    case SS_INT64: return f((long long*)nullptr);
    default: return SS_ERR_INVALID_ARGUMENT;
    }
}

ss_status stage_host(ss_context* c, const void* h, size_t bytes, cudaStream_t st) {
    ss_status rc = grow(c, &c->d_stage, &c->cap_stage, bytes);
    if (rc) return rc;
    CK(cudaMemcpyAsync(c->d_stage, h, bytes, cudaMemcpyHostToDevice, st));
    c->h2d = (int64_t)bytes;
    return SS_OK;
}
}  // namespace

// =========================================================== C ABI ========
extern "C" {

int ss_abi_version(void) { return SS_ABI_VERSION; }

const char* ss_status_string(ss_status s) {
    switch (s) {
    case SS_OK: return "SS_OK";
    case SS_ERR_INVALID_ARGUMENT: return "SS_ERR_INVALID_ARGUMENT";
    case SS_ERR_CUDA: return "SS_ERR_CUDA";
    case SS_ERR_OUT_OF_MEMORY: return "SS_ERR_OUT_OF_MEMORY";
    case SS_ERR_NCCL: return "SS_ERR_NCCL";
    case SS_ERR_INTERNAL: return "SS_ERR_INTERNAL";
    default: return "SS_UNKNOWN_STATUS";
    }
}

ss_status ss_create(int device, ss_context** out) {
    if (!out || device < 0) return SS_ERR_INVALID_ARGUMENT;
    *out = nullptr;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device >= ndev) {
        (void)cudaGetLastError();
        return SS_ERR_CUDA;
    }
    ss_context* c = new (std::nothrow) ss_context();
    if (!c) return SS_ERR_OUT_OF_MEMORY;
    c->device = device;
    c->host_timing = std::getenv("SS_HOST_TIMING") != nullptr;
    c->cfg.b_exact = 256;
    c->cfg.b_deep = 0;
    c->cfg.sample_size = 0;
    c->cfg.base_case = 16384;
    c->cfg.ctas_per_sm = 4;
    c->cfg.profile = 0;
    c->cfg.seed = 0x5A17;
    c->cfg.classify = 0;
    c->cfg.fused_filter = 1;
    c->cfg.spec_z = 3.0f;
    c->cfg.spec_min_n = (int64_t)1 << 16;
    c->cfg.spec_max_frac = 0.25f;
    c->cfg.shard_gather_log2 = 0;
    c->cfg.directed = 1;
    c->cfg.upper_onepass = 1;
    DevGuard g(device);
    if (cudaDeviceGetAttribute(&c->sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess) {
        (void)cudaGetLastError();
        delete c;
        return SS_ERR_CUDA;
    }
    ss_status rc = ensure_small(c);
    if (!rc) rc = op_set_attrs(c, (const float*)nullptr);
    if (!rc) rc = op_set_attrs(c, (const double*)nullptr);
    if (!rc) rc = op_set_attrs(c, (const int*)nullptr);
    if (!rc) rc = op_set_attrs(c, (const long long*)nullptr);
    if (!rc && cudaFuncSetAttribute(tree_from_keys_kernel<u32>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)(16384 * sizeof(u32))) != cudaSuccess) rc = SS_ERR_CUDA;
    if (!rc && cudaFuncSetAttribute(tree_from_keys_kernel<u64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)(16384 * sizeof(u64))) != cudaSuccess) rc = SS_ERR_CUDA;
    if (rc) {
        ss_destroy(c);
        return rc;
    }
    *out = c;
    return SS_OK;
}

void ss_destroy(ss_context* c) {
    if (!c) return;
    if (c->host_timing && c->ht_n)
        std::fprintf(stderr, "ss host timing (us/call over %lld exact calls): prep %.2f graph-launch %.2f "
                     "wait %.2f post %.2f total %.2f\n", c->ht_n, c->ht[0] / c->ht_n, c->ht[1] / c->ht_n,
                     c->ht[2] / c->ht_n, c->ht[3] / c->ht_n, c->ht[4] / c->ht_n);
    DevGuard g(c->device);
    delete c->comm;
    cudaFree(c->d_dist);
    cudaFree(c->d_gather[0]);
    cudaFree(c->d_gather[1]);
    cudaFree(c->d_oracles);
    cudaFree(c->d_buf[0]);
    cudaFree(c->d_buf[1]);
    cudaFree(c->d_win);
    cudaFree(c->d_stage);
    cudaFree(c->d_ctl);
    cudaFree(c->d_res);
    cudaFree(c->d_totals);
    cudaFree(c->d_cta_counts);
    cudaFree(c->d_tree);
    cudaFree(c->d_spl);
    cudaFree(c->d_eq);
    cudaFree(c->d_sorted);
    cudaFree(c->d_sample0);
    cudaFree(c->d_presample);
    cudaFree(c->d_image);
    cudaFree(c->d_seq);
    cudaFree(c->d_upper_cnt);
    for (int i = 0; i < MULTI_CH; ++i) {
        if (c->mchild[i]) ss_destroy(c->mchild[i]);
        if (c->mchild_st[i]) cudaStreamDestroy(c->mchild_st[i]);
        if (c->ev_mjoin[i]) cudaEventDestroy(c->ev_mjoin[i]);
    }
    if (c->ev_mfork) cudaEventDestroy(c->ev_mfork);
    if (c->h_mpin) cudaFreeHost(c->h_mpin);
    cudaFree(c->d_multi_scratch);
    cudaFree(c->d_multi);
    cudaFree(c->d_qs);
    cudaFree(c->d_qsbuf[0]);
    cudaFree(c->d_qsbuf[1]);
    if (c->h_qs) cudaFreeHost(c->h_qs);
    for (auto& e : c->ev_qs)
        if (e) cudaEventDestroy(e);
    for (auto& e : c->ev_upper)
        if (e) cudaEventDestroy(e);
    for (auto& e : c->graphs) {
        if (e.exec) cudaGraphExecDestroy(e.exec);
        if (e.graph) cudaGraphDestroy(e.graph);
    }
    if (c->cap_st) cudaStreamDestroy(c->cap_st);
    if (c->h_res) cudaFreeHost(c->h_res);
    if (c->ev_ready)
        for (int l = 0; l < SS_MAX_LEVELS; ++l)
            for (int q = 0; q < 3; ++q)
                for (int e = 0; e < 2; ++e) cudaEventDestroy(c->ev[l][q][e]);
    (void)cudaGetLastError();
    delete c;
}

ss_status ss_get_config(const ss_context* c, ss_config* out) {
    if (!c || !out) return SS_ERR_INVALID_ARGUMENT;
    *out = c->cfg;
    return SS_OK;
}

ss_status ss_set_config(ss_context* c, const ss_config* cfg) {
    if (!c || !cfg) return SS_ERR_INVALID_ARGUMENT;
    if (!pow2(cfg->b_exact) || cfg->b_exact < 4 || cfg->b_exact > 256)
        return fail(c, SS_ERR_INVALID_ARGUMENT, "b_exact must be a power of two in [4, 256]");
    if (cfg->b_deep != 0 && (!pow2(cfg->b_deep) || cfg->b_deep < 4 || cfg->b_deep > 256))
        return fail(c, SS_ERR_INVALID_ARGUMENT, "b_deep must be 0 or a power of two in [4, 256]");
    if (cfg->sample_size != 0 && (!pow2(cfg->sample_size) || cfg->sample_size > 16384 ||
                                  cfg->sample_size < std::max(64, std::max(cfg->b_exact, cfg->b_deep))))
        return fail(c, SS_ERR_INVALID_ARGUMENT, "sample_size must be 0 or a power of two in [max(64, b), 16384]");
    if (!pow2(cfg->base_case) || cfg->base_case < 256 || cfg->base_case > 16384)
        return fail(c, SS_ERR_INVALID_ARGUMENT, "base_case must be a power of two in [256, 16384]");
    if (cfg->profile < 0 || cfg->profile > 3)
        return fail(c, SS_ERR_INVALID_ARGUMENT, "profile must be 0, 1, 2 or 3");
    if (cfg->classify < 0 || cfg->classify > 1)
        return fail(c, SS_ERR_INVALID_ARGUMENT, "classify must be 0 (auto) or 1 (tree walk)");
    if (cfg->ctas_per_sm < 1 || cfg->ctas_per_sm > 16)
        return fail(c, SS_ERR_INVALID_ARGUMENT, "ctas_per_sm must be in [1, 16]");
    if (cfg->fused_filter < 0 || cfg->fused_filter > 1)
        return fail(c, SS_ERR_INVALID_ARGUMENT, "fused_filter must be 0 or 1");
    if (!(cfg->spec_z >= 0.0f && cfg->spec_z <= 64.0f))
        return fail(c, SS_ERR_INVALID_ARGUMENT, "spec_z must be in [0, 64]");
    if (cfg->spec_min_n < 1)
        return fail(c, SS_ERR_INVALID_ARGUMENT, "spec_min_n must be >= 1");
    if (!(cfg->spec_max_frac > 0.0f && cfg->spec_max_frac <= 1.0f))
        return fail(c, SS_ERR_INVALID_ARGUMENT, "spec_max_frac must be in (0, 1]");
    if (cfg->shard_gather_log2 != 0 && (cfg->shard_gather_log2 < 12 || cfg->shard_gather_log2 > 28))
        return fail(c, SS_ERR_INVALID_ARGUMENT, "shard_gather_log2 must be 0 or in [12, 28]");
    if (cfg->directed != 0 && cfg->directed != 1)
        return fail(c, SS_ERR_INVALID_ARGUMENT, "directed must be 0 or 1");
    if (cfg->upper_onepass != 0 && cfg->upper_onepass != 1)
        return fail(c, SS_ERR_INVALID_ARGUMENT, "upper_onepass must be 0 or 1");
    // captured graphs bake in grid sizes and the fused-filter parameters
    const bool regrid = cfg->ctas_per_sm != c->cfg.ctas_per_sm || cfg->classify != c->cfg.classify ||
                        cfg->fused_filter != c->cfg.fused_filter || cfg->spec_z != c->cfg.spec_z ||
                        cfg->spec_min_n != c->cfg.spec_min_n || cfg->spec_max_frac != c->cfg.spec_max_frac ||
                        cfg->directed != c->cfg.directed;
    c->cfg = *cfg;
    if (regrid)                   // captured grid sizes are stale (the other knobs are part of the graph key)
        for (auto& e : c->graphs) {
            if (e.exec) cudaGraphExecDestroy(e.exec);
            if (e.graph) cudaGraphDestroy(e.graph);
            e = ss_context::GraphEntry();
        }
    return SS_OK;
}

ss_status ss_profile_totals(ss_context* c, double* ms_sum, int64_t* count, int64_t* launches,
                            int64_t* calls, int32_t reset) {
    if (!c) return SS_ERR_INVALID_ARGUMENT;
    for (int l = 0; l < SS_MAX_LEVELS; ++l)
        for (int q = 0; q < 3; ++q) {
            if (ms_sum) ms_sum[l * 3 + q] = c->prof_sum[l][q];
            if (count) count[l * 3 + q] = c->prof_cnt[l][q];
            if (reset) { c->prof_sum[l][q] = 0; c->prof_cnt[l][q] = 0; }
        }
    if (launches) *launches = c->launches_total;
    if (calls) *calls = c->calls_total;
    if (reset) { c->launches_total = 0; c->calls_total = 0; }
    return SS_OK;
}

ss_status ss_last_stats(const ss_context* c, ss_stats* out) {
    if (!c || !out) return SS_ERR_INVALID_ARGUMENT;
    *out = c->stats;
    return SS_OK;
}

const char* ss_last_error(const ss_context* c) { return c ? c->err.c_str() : "NULL context"; }

static ss_status select_impl(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, int64_t k,
                             void* h_result, void* stream);

ss_status ss_select(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, int64_t k, void* h_result,
                    void* stream) {
    if (c) c->h2d = 0;
    return select_impl(c, dt, d_data, n, k, h_result, stream);
}

static ss_status select_impl(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, int64_t k,
                             void* h_result, void* stream) {
    ss_status rc = check_common(c, dt, d_data, n, k, h_result);
    if (rc) return rc;
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    try {
        return dispatch(dt, [&](auto* tag) {
            typedef std::remove_pointer_t<decltype(tag)> T;
            return op_exact(c, (const T*)d_data, (u64)n, (u64)k, h_result, st);
        });
    } catch (...) {
        return fail(c, SS_ERR_INTERNAL, "exception in ss_select");
    }
}

ss_status ss_select_host(ss_context* c, ss_dtype dt, const void* h_data, int64_t n, int64_t k,
                         void* h_result, void* stream) {
    ss_status rc = check_common(c, dt, h_data, n, k, h_result);
    if (rc) return rc;
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    if ((rc = stage_host(c, h_data, (size_t)n * dt_size(dt), st))) return rc;
    return select_impl(c, dt, c->d_stage, n, k, h_result, stream);
}

ss_status ss_select_upper(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, int64_t k, void* d_out,
                          void* h_result, void* stream) {
    ss_status rc = check_common(c, dt, d_data, n, k, h_result);
    if (rc) return rc;
    if (!d_out) return fail(c, SS_ERR_INVALID_ARGUMENT, "d_out is NULL");
    const size_t S = dt_size(dt);
    const uintptr_t a0 = (uintptr_t)d_data, a1 = a0 + (size_t)n * S, o0 = (uintptr_t)d_out,
                    o1 = o0 + (size_t)(n - k) * S;
    if (o0 < a1 && a0 < o1) return fail(c, SS_ERR_INVALID_ARGUMENT, "d_out overlaps d_data");
    c->h2d = 0;
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    try {
        return dispatch(dt, [&](auto* tag) {
            typedef std::remove_pointer_t<decltype(tag)> T;
            return op_upper(c, (const T*)d_data, (u64)n, (u64)k, (T*)d_out, h_result, st);
        });
    } catch (...) {
        return fail(c, SS_ERR_INTERNAL, "exception in ss_select_upper");
    }
}

ss_status ss_quickselect(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, int64_t k, void* h_result,
                         int64_t* h_n_level, int32_t n_level_cap, int32_t* h_levels, void* stream) {
    ss_status rc = check_common(c, dt, d_data, n, k, h_result);
    if (rc) return rc;
    if (n_level_cap < 0 || (n_level_cap > 0 && !h_n_level))
        return fail(c, SS_ERR_INVALID_ARGUMENT, "ss_quickselect: bad n_level buffer");
    DevGuard g(c->device);
    try {
        return dispatch(dt, [&](auto* tag) {
            typedef std::remove_pointer_t<decltype(tag)> T;
            return op_quick(c, (const T*)d_data, (u64)n, (u64)k, h_result, h_n_level, n_level_cap, h_levels,
                                (cudaStream_t)stream);
        });
    } catch (...) {
        return fail(c, SS_ERR_INTERNAL, "exception in ss_quickselect");
    }
}

ss_status ss_select_multi(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, int32_t m,
                          const int64_t* h_ks, void* h_results, void* stream) {
    ss_status rc = check_common(c, dt, d_data, n, 0, h_results);
    if (rc) return rc;
    if (!h_ks || m < 1 || m > MULTI_MAX) return fail(c, SS_ERR_INVALID_ARGUMENT, "m must be in [1, 1024], ks non-NULL");
    for (int i = 0; i < m; ++i)
        if (h_ks[i] < 0 || h_ks[i] >= n) return fail(c, SS_ERR_INVALID_ARGUMENT, "rank outside [0, n)");
    if (((uintptr_t)d_data) % dt_size(dt)) return fail(c, SS_ERR_INVALID_ARGUMENT, "d_data misaligned for dtype");
    c->h2d = 0;
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    try {
        return dispatch(dt, [&](auto* tag) {
            typedef std::remove_pointer_t<decltype(tag)> T;
            return op_multi(c, dt, (const T*)d_data, (u64)n, m, h_ks, h_results, st);
        });
    } catch (...) {
        return fail(c, SS_ERR_INTERNAL, "exception in ss_select_multi");
    }
}

static ss_status approx_impl(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, int64_t k, int32_t b,
                             void* h_result, int64_t* h_rank, void* stream);

ss_status ss_approx_select(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, int64_t k, int32_t b,
                           void* h_result, int64_t* h_rank, void* stream) {
    if (c) c->h2d = 0;
    return approx_impl(c, dt, d_data, n, k, b, h_result, h_rank, stream);
}

static ss_status approx_impl(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, int64_t k, int32_t b,
                             void* h_result, int64_t* h_rank, void* stream) {
    ss_status rc = check_common(c, dt, d_data, n, k, h_result);
    if (rc) return rc;
    if (!pow2(b) || b < 4 || b > 1024) return fail(c, SS_ERR_INVALID_ARGUMENT, "b must be a power of two in [4, 1024]");
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    try {
        return dispatch(dt, [&](auto* tag) {
            typedef std::remove_pointer_t<decltype(tag)> T;
            return op_approx(c, (const T*)d_data, (u64)n, (u64)k, b, h_result, h_rank, st);
        });
    } catch (...) {
        return fail(c, SS_ERR_INTERNAL, "exception in ss_approx_select");
    }
}

ss_status ss_approx_select_host(ss_context* c, ss_dtype dt, const void* h_data, int64_t n, int64_t k,
                                int32_t b, void* h_result, int64_t* h_rank, void* stream) {
    ss_status rc = check_common(c, dt, h_data, n, k, h_result);
    if (rc) return rc;
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    if ((rc = stage_host(c, h_data, (size_t)n * dt_size(dt), st))) return rc;
    return approx_impl(c, dt, c->d_stage, n, k, b, h_result, h_rank, stream);
}

// ------------------------------------------------------------- steps ------
ss_status ss_step_sample(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, int32_t level,
                         int64_t slot_begin, int64_t count, void* d_sample_keys, void* stream) {
    if (!c || !dt_size(dt) || !d_data || !d_sample_keys || n < 1 || count < 0 || slot_begin < 0 || level < 0)
        return c ? fail(c, SS_ERR_INVALID_ARGUMENT, "ss_step_sample: bad argument") : SS_ERR_INVALID_ARGUMENT;
    if (count == 0) return SS_OK;
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    return dispatch(dt, [&](auto* tag) -> ss_status {
        typedef std::remove_pointer_t<decltype(tag)> T;
        return op_step_sample(c, (const T*)d_data, (u64)n, level, (u64)slot_begin, (u64)count, d_sample_keys, st);
    });
}

ss_status ss_step_tree(ss_context* c, ss_dtype dt, const void* d_sample_keys, int32_t s, int32_t b,
                       int32_t fixup, void* d_tree, void* d_splitters, uint8_t* d_eq, void* stream) {
    if (!c || !dt_size(dt) || !d_sample_keys || !d_tree || !pow2(s) || s > 16384 || !pow2(b) || b < 2 ||
        b > 1024 || s < b)
        return c ? fail(c, SS_ERR_INVALID_ARGUMENT, "ss_step_tree: bad argument") : SS_ERR_INVALID_ARGUMENT;
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    if (dt_size(dt) == 4) {
        tree_from_keys_kernel<u32><<<1, K1_THREADS, (size_t)s * 4, st>>>(
            (const u32*)d_sample_keys, s, b, fixup, (u32*)d_tree, (u32*)d_splitters, d_eq);
    } else {
        tree_from_keys_kernel<u64><<<1, K1_THREADS, (size_t)s * 8, st>>>(
            (const u64*)d_sample_keys, s, b, fixup, (u64*)d_tree, (u64*)d_splitters, d_eq);
    }
    CKLAUNCH("tree_from_keys_kernel");
    return SS_OK;
}

int64_t ss_oracle_offset(ss_dtype dt, const void* d_data, int64_t n) {
    const size_t S = dt_size(dt);
    if (!S || n < 0) return -1;
    const u64 mis = (u64)((uintptr_t)d_data & 15u);
    u64 head = mis ? (16 - mis) / S : 0;          // make_chunking's peeled head
    if (head > (u64)n) head = (u64)n;
    return (int64_t)oracle_pad(head);
}

ss_status ss_step_count(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, const void* d_tree,
                        int32_t b, uint64_t* d_totals, uint8_t* d_oracles, void* stream) {
    if (!c || !dt_size(dt) || !d_data || !d_tree || !d_totals || n < 1 || !pow2(b) || b < 4 || b > 1024 ||
        (d_oracles && b > 256) || ((uintptr_t)d_data) % dt_size(dt))
        return c ? fail(c, SS_ERR_INVALID_ARGUMENT, "ss_step_count: bad argument") : SS_ERR_INVALID_ARGUMENT;
    if (((uintptr_t)d_oracles) & 15u)
        return fail(c, SS_ERR_INVALID_ARGUMENT, "ss_step_count: d_oracles must be 16-byte aligned");
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    ss_status rc = ensure_small(c);
    if (rc) return rc;
    CK(cudaMemsetAsync(d_totals, 0, sizeof(u64) * b, st));
    return dispatch(dt, [&](auto* tag) -> ss_status {
        typedef std::remove_pointer_t<decltype(tag)> T;
        ss_status r2 = op_step_count(c, (const T*)d_data, (u64)n, d_tree, b, (u64*)d_totals, d_oracles, st);
        if (r2) return r2;
        c->step_ptr = d_data;
        c->step_n = (u64)n;
        c->step_b = b;
        c->step_dt = (int)dt;
        return SS_OK;
    });
}

ss_status ss_step_filter(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, const uint8_t* d_oracles,
                         int32_t bucket, void* d_out, uint64_t* d_count, void* stream) {
    if (!c || !dt_size(dt) || !d_data || !d_oracles || !d_out || !d_count || n < 1 || bucket < 0)
        return c ? fail(c, SS_ERR_INVALID_ARGUMENT, "ss_step_filter: bad argument") : SS_ERR_INVALID_ARGUMENT;
    if (((uintptr_t)d_oracles) & 15u)
        return fail(c, SS_ERR_INVALID_ARGUMENT, "ss_step_filter: d_oracles must be 16-byte aligned");
    if (c->step_ptr != d_data || c->step_n != (u64)n || c->step_dt != (int)dt || bucket >= c->step_b)
        return fail(c, SS_ERR_INVALID_ARGUMENT,
                    "ss_step_filter must follow ss_step_count on the same data (per-CTA counts)");
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    CK(cudaMemsetAsync(d_count, 0, sizeof(u64), st));
    return dispatch(dt, [&](auto* tag) -> ss_status {
        typedef std::remove_pointer_t<decltype(tag)> T;
        return op_step_filter(c, (const T*)d_data, (u64)n, d_oracles, bucket, (T*)d_out, (u64*)d_count, st);
    });
}

ss_status ss_step_count_ablation(ss_context* c, ss_dtype dt, const void* d_data, int64_t n, const void* d_tree,
                                 int32_t b, int32_t mode, uint64_t* d_totals, void* stream) {
    if (!c || !dt_size(dt) || !d_data || !d_tree || !d_totals || n < 1 || !pow2(b) || b < 2 || b > 1024 ||
        mode < 0 || mode >= ABL_MODES || ((uintptr_t)d_data) % dt_size(dt))
        return c ? fail(c, SS_ERR_INVALID_ARGUMENT, "ss_step_count_ablation: bad argument") : SS_ERR_INVALID_ARGUMENT;
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    CK(cudaMemsetAsync(d_totals, 0, sizeof(u64) * b, st));
    return dispatch(dt, [&](auto* tag) -> ss_status {
        typedef std::remove_pointer_t<decltype(tag)> T;
        return op_ablation(c, (const T*)d_data, (u64)n, d_tree, log2i(b), mode, (u64*)d_totals, st);
    });
}

ss_status ss_step_search(ss_context* c, const uint64_t* d_totals, int32_t b, int64_t k, const uint8_t* d_eq,
                         int64_t* d_out, void* stream) {
    if (!c || !d_totals || !d_out || b < 1 || b > 1024 || k < 0)
        return c ? fail(c, SS_ERR_INVALID_ARGUMENT, "ss_step_search: bad argument") : SS_ERR_INVALID_ARGUMENT;
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    search_kernel<<<1, 256, 0, st>>>((const u64*)d_totals, (u32)b, (u64)k, d_eq, (long long*)d_out);
    CKLAUNCH("search_kernel");
    return SS_OK;
}

ss_status ss_step_keys_to_values(ss_context* c, ss_dtype dt, const void* d_keys, int64_t count, void* d_values,
                                 void* stream) {
    if (!c || !dt_size(dt) || !d_keys || !d_values || count < 0)
        return c ? fail(c, SS_ERR_INVALID_ARGUMENT, "ss_step_keys_to_values: bad argument") : SS_ERR_INVALID_ARGUMENT;
    if (count == 0) return SS_OK;
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    return dispatch(dt, [&](auto* tag) -> ss_status {
        typedef std::remove_pointer_t<decltype(tag)> T;
        return op_keys_to_values(c, (const T*)nullptr, d_keys, (u64)count, d_values, st);
    });
}

// ------------------------------------------------------------ sharded ----
ss_status ss_nccl_unique_id(char out_id[128]) {
    if (!out_id) return SS_ERR_INVALID_ARGUMENT;
    std::string err;
    return ss_comm::nccl_unique_id(out_id, err);
}

ss_status ss_comm_init(ss_context* c, const char id[128], int nranks, int rank) {
    if (!c) return SS_ERR_INVALID_ARGUMENT;
    if (!id || nranks < 1 || nranks > DIST_MAX_RANKS || rank < 0 || rank >= nranks)
        return fail(c, SS_ERR_INVALID_ARGUMENT, "ss_comm_init: bad id, nranks (1..16) or rank");
    ss_status rc = SS_OK;
    std::string err;
    ss_comm::ShardComm* comm = ss_comm::make_nccl_comm(id, nranks, rank, c->device, &rc, err);
    if (!comm) return fail(c, rc, err);
    delete c->comm;
    c->comm = comm;
    c->dist_n_plan = 0;
    return SS_OK;
}

ss_status ss_local_group_create(int nranks, ss_local_group** out) { return ss_comm::local_group_create(nranks, out); }

void ss_local_group_destroy(ss_local_group* g) { ss_comm::local_group_destroy(g); }

ss_status ss_comm_init_local(ss_context* c, ss_local_group* g, int rank) {
    if (!c) return SS_ERR_INVALID_ARGUMENT;
    ss_status rc = SS_OK;
    std::string err;
    ss_comm::ShardComm* comm = ss_comm::make_local_comm(g, rank, c->device, &rc, err);
    if (!comm) return fail(c, rc, err);
    delete c->comm;
    c->comm = comm;
    c->dist_n_plan = 0;
    return SS_OK;
}

ss_status ss_select_sharded(ss_context* c, ss_dtype dt, const void* d_shard, int64_t n_local, int64_t k_global,
                            void* h_result, void* stream) {
    if (!c) return SS_ERR_INVALID_ARGUMENT;
    if (!dt_size(dt)) return fail(c, SS_ERR_INVALID_ARGUMENT, "unknown dtype");
    if (!h_result || (n_local > 0 && !d_shard)) return fail(c, SS_ERR_INVALID_ARGUMENT, "NULL pointer");
    if (n_local < 0 || k_global < 0) return fail(c, SS_ERR_INVALID_ARGUMENT, "n_local and k_global must be >= 0");
    if (((uintptr_t)d_shard) % dt_size(dt)) return fail(c, SS_ERR_INVALID_ARGUMENT, "data not naturally aligned");
    if (!c->comm) return fail(c, SS_ERR_INVALID_ARGUMENT, "ss_select_sharded: no communicator (ss_comm_init first)");
    c->h2d = 0;
    DevGuard g(c->device);
    cudaStream_t st = (cudaStream_t)stream;
    try {
        return dispatch(dt, [&](auto* tag) {
            typedef std::remove_pointer_t<decltype(tag)> T;
            return op_sharded(c, (const T*)d_shard, (u64)n_local, (u64)k_global, h_result, st);
        });
    } catch (...) {
        return fail(c, SS_ERR_INTERNAL, "exception in ss_select_sharded");
    }
}

// --------------------------------------------------------- convenience ----
}  // extern "C"

namespace {
// thread-local default contexts, one per device (destroyed with the thread)
struct DefaultContexts {
    ss_context* ctx[64] = {};
    ~DefaultContexts() {
        for (auto* c : ctx)
            if (c) ss_destroy(c);
    }
};
ss_status default_context(ss_context** out) {
    thread_local DefaultContexts dc;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) {
        (void)cudaGetLastError();
        return SS_ERR_CUDA;
    }
    if (dev < 0 || dev >= 64) return SS_ERR_INVALID_ARGUMENT;
    if (!dc.ctx[dev]) {
        const ss_status rc = ss_create(dev, &dc.ctx[dev]);
        if (rc) return rc;
    }
    *out = dc.ctx[dev];
    return SS_OK;
}
}  // namespace

extern "C" {

#define SS_CONVENIENCE(name, T, DT)                                                       \
    ss_status name(const T* d_data, int64_t n, int64_t k, T* h_result) {                  \
        ss_context* c = nullptr;                                                          \
        const ss_status rc = default_context(&c);                                         \
        if (rc) return rc;                                                                \
        return ss_select(c, DT, d_data, n, k, h_result, nullptr);                         \
    }
SS_CONVENIENCE(ss_select_f32, float, SS_FLOAT32)
SS_CONVENIENCE(ss_select_f64, double, SS_FLOAT64)
SS_CONVENIENCE(ss_select_i32, int32_t, SS_INT32)
SS_CONVENIENCE(ss_select_i64, int64_t, SS_INT64)
#undef SS_CONVENIENCE

ss_status ss_approx_select_f32(const float* d_data, int64_t n, int64_t k, int32_t b, float* h_result,
                               int64_t* h_rank) {
    ss_context* c = nullptr;
    const ss_status rc = default_context(&c);
    if (rc) return rc;
    return ss_approx_select(c, SS_FLOAT32, d_data, n, k, b, h_result, h_rank, nullptr);
}

}  // extern "C"
