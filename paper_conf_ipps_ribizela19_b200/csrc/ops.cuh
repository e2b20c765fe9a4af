// ops.cuh -- the per-dtype entry points of the driver (external linkage).
// inst_<dtype>.cu defines SS_INST_T and gets the definitions; abi.cu sees the
// declarations of all four dtypes and dispatches to them by overload.
#pragma once

#define SS_OPS_DECL(T)                                                                                        \
    ss_status op_set_attrs(ss_context* c, const T* tag);                                                      \
    ss_status op_exact(ss_context* c, const T* d, ss::u64 n, ss::u64 k, void* h_result, cudaStream_t st);     \
    ss_status op_approx(ss_context* c, const T* d, ss::u64 n, ss::u64 k, int b, void* h_result,               \
                        int64_t* h_rank, cudaStream_t st);                                                    \
    ss_status op_upper(ss_context* c, const T* d, ss::u64 n, ss::u64 k, T* d_out, void* h_result,             \
                       cudaStream_t st);                                                                      \
    ss_status op_multi(ss_context* c, ss_dtype dt, const T* d, ss::u64 n, int m, const int64_t* ks,           \
                       void* h_res, cudaStream_t st);                                                         \
    ss_status op_quick(ss_context* c, const T* d, ss::u64 n, ss::u64 k, void* h_result, int64_t* h_n_level,   \
                       int32_t cap, int32_t* h_levels, cudaStream_t st);                                      \
    ss_status op_ablation(ss_context* c, const T* d, ss::u64 n, const void* tree, int h, int mode,            \
                          ss::u64* totals, cudaStream_t st);                                                  \
    ss_status op_step_sample(ss_context* c, const T* d, ss::u64 n, int level, ss::u64 slot_begin,             \
                             ss::u64 count, void* keys, cudaStream_t st);                                     \
    ss_status op_step_count(ss_context* c, const T* d, ss::u64 n, const void* tree, int b, ss::u64* totals,   \
                            uint8_t* oracles, cudaStream_t st);                                               \
    ss_status op_step_filter(ss_context* c, const T* d, ss::u64 n, const uint8_t* oracles, int bucket,        \
                             T* out, ss::u64* count, cudaStream_t st);                                        \
    ss_status op_keys_to_values(ss_context* c, const T* tag, const void* keys, ss::u64 count, void* values,   \
                                cudaStream_t st);                                                             \
    ss_status op_sharded(ss_context* c, const T* d, ss::u64 n_local, ss::u64 k, void* h_result, cudaStream_t st);

SS_OPS_DECL(float)
SS_OPS_DECL(double)
SS_OPS_DECL(int)
SS_OPS_DECL(long long)

#ifdef SS_INST_T
namespace {
typedef SS_INST_T InstT;
}
ss_status op_set_attrs(ss_context* c, const InstT*) { return set_k1_attrs<InstT>(c); }

ss_status op_exact(ss_context* c, const InstT* d, u64 n, u64 k, void* h_result, cudaStream_t st) {
    return run_exact<InstT>(c, d, n, k, h_result, st);
}

ss_status op_approx(ss_context* c, const InstT* d, u64 n, u64 k, int b, void* h_result, int64_t* h_rank,
                    cudaStream_t st) {
    return run_approx<InstT>(c, d, n, k, b, h_result, h_rank, st);
}

ss_status op_upper(ss_context* c, const InstT* d, u64 n, u64 k, InstT* d_out, void* h_result, cudaStream_t st) {
    return run_upper<InstT>(c, d, n, k, d_out, h_result, st);
}

ss_status op_multi(ss_context* c, ss_dtype dt, const InstT* d, u64 n, int m, const int64_t* ks, void* h_res,
                   cudaStream_t st) {
    return run_multi<InstT>(c, dt, d, n, m, ks, h_res, st);
}

ss_status op_quick(ss_context* c, const InstT* d, u64 n, u64 k, void* h_result, int64_t* h_n_level, int32_t cap,
                   int32_t* h_levels, cudaStream_t st) {
    return run_quick<InstT>(c, d, n, k, h_result, h_n_level, cap, h_levels, st);
}

ss_status op_ablation(ss_context* c, const InstT* d, u64 n, const void* tree, int h, int mode, u64* totals,
                      cudaStream_t st) {
    return launch_ablation<InstT>(c, d, n, tree, h, mode, totals, st);
}

ss_status op_step_sample(ss_context* c, const InstT* d, u64 n, int level, u64 slot_begin, u64 count, void* keys,
                         cudaStream_t st) {
    typedef typename Traits<InstT>::Key K;
    const u32 blocks = (u32)std::min<u64>((count + 255) / 256, 1024);
    sample_keys_kernel<InstT><<<blocks, 256, 0, st>>>(d, n, level, slot_begin, count, c->cfg.seed, (K*)keys);
    CKLAUNCH("sample_keys_kernel");
    return SS_OK;
}

ss_status op_step_count(ss_context* c, const InstT* d, u64 n, const void* tree, int b, u64* totals,
                        uint8_t* oracles, cudaStream_t st) {
    CountArgs a{};
    a.tree = tree;
    a.oracles = oracles;
    a.cta_counts = c->d_cta_counts;
    a.totals = totals;
    a.lut = c->cfg.classify == 0;
    a.n = n;
    a.tail = TAIL_NONE;
    ss_status rc = launch_count<InstT>(c, log2i(b), d, a, st);
    if (rc) return rc;
    c->step_grid = a.grid;
    return SS_OK;
}

ss_status op_step_filter(ss_context* c, const InstT* d, u64 n, const uint8_t* oracles, int bucket, InstT* out,
                         u64* count, cudaStream_t st) {
    FilterArgs f{};
    f.oracles = oracles;
    f.cta_counts = c->d_cta_counts;
    f.b_count = (u32)c->step_b;
    f.count_out = count;
    f.n = n;
    f.bucket = (u32)bucket;
    f.grid = c->step_grid;
    filter_kernel<InstT><<<f.grid, K5_THREADS, FILTER_SMEM, st>>>(d, out, f);
    CKLAUNCH("filter_kernel");
    return SS_OK;
}

ss_status op_keys_to_values(ss_context* c, const InstT*, const void* keys, u64 count, void* values,
                            cudaStream_t st) {
    typedef typename Traits<InstT>::Key K;
    const u32 blocks = (u32)std::min<u64>((count + 255) / 256, 4096);
    keys_to_values_kernel<InstT><<<blocks, 256, 0, st>>>((const K*)keys, count, (K*)values);
    CKLAUNCH("keys_to_values_kernel");
    return SS_OK;
}
ss_status op_sharded(ss_context* c, const InstT* d, u64 n_local, u64 k, void* h_result, cudaStream_t st) {
    return run_sharded<InstT>(c, d, n_local, k, h_result, st);
}
#endif  // SS_INST_T
