/*
 * sampleselect.h -- C ABI of the B200 SampleSelect hot path.
 *
 * Method: Ribizel & Anzt, "Approximate and Exact Selection on GPUs",
 * IPDPS-W 2019 (/root/reference/PAPER.md, cited as L<line>).
 *
 * Problem (§II): for an input sequence x_0..x_{n-1}, return the element
 * at position k (0-based) of the sorted sequence; if a value occurs several
 * times it carries the smallest rank.  Floating-point values are ordered by
 * IEEE-754 totalOrder (-NaN < -inf < ... < -0 < +0 < ... < +inf < +NaN;
 * DESIGN.md reading R3), integers numerically, so the answer is unique
 * bit-for-bit.  The input is never modified (L237-245).
 *
 * Everything below runs in hand-written sm_100a kernels; there is no CPU
 * fallback.  If no CUDA device is usable every call returns SS_ERR_CUDA.
 *
 * Conventions shared by all calls
 *   - d_* pointers are DEVICE pointers on the context's device; h_* pointers
 *     are HOST pointers (pageable or pinned).  Device inputs must be
 *     naturally aligned for their dtype (4 or 8 bytes); any further alignment
 *     is handled (kernels peel unaligned heads).  Inputs are read-only.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *     stream).  Calls that return a host result synchronise that stream
 *     before returning; *_async calls only enqueue work.
 *   - The context owns all workspace (oracle bytes, survivor buffers, level
 *     state); it grows lazily and is freed by ss_destroy.  Outputs are
 *     written only on SS_OK; on error they are untouched and ss_last_error()
 *     describes the failure.  No C++ exception or abort crosses this ABI.
 *   - One context per host thread and stream; contexts are independent.
 */
#ifndef SAMPLESELECT_H
#define SAMPLESELECT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SS_ABI_VERSION 7
#define SS_MAX_LEVELS 32

typedef enum { SS_FLOAT32 = 0, SS_FLOAT64 = 1, SS_INT32 = 2, SS_INT64 = 3 } ss_dtype;

typedef enum {
    SS_OK = 0,
    SS_ERR_INVALID_ARGUMENT = 1, /* NULL pointer, n < 1, k not in [0,n), bad dtype/b/config */
    SS_ERR_CUDA = 2,             /* a CUDA runtime error (no device, launch failure, ...) */
    SS_ERR_OUT_OF_MEMORY = 3,    /* workspace allocation failed */
    SS_ERR_NCCL = 4,             /* NCCL unavailable or a NCCL call failed (sharded calls) */
    SS_ERR_INTERNAL = 5          /* recursion-depth guard tripped (should not happen) */
} ss_status;

typedef struct ss_context ss_context;
typedef struct ss_local_group ss_local_group;   /* in-process rank group (sharded calls, tests) */

/* Tuning knobs (§IV.H).  ss_create fills the defaults. */
typedef struct {
    int32_t b_exact;      /* buckets per exact level: power of two in [4, 256]
                             (oracle bytes cap b at 256, L272-276). default 256 */
    int32_t sample_size;  /* s: 0 = per-b default clamp(16 b, 4096, 16384) (L557-561);
                             else a power of two in [max(64, b_exact, b_deep), 16384] */
    int32_t base_case;    /* B: levels with n <= B finish in one CTA (L97, L579-583);
                             power of two in [256, 16384]. default 16384 */
    int32_t ctas_per_sm;  /* count/filter grid = ctas_per_sm * #SMs. default 4 */
    int32_t profile;      /* 1: record CUDA events around every kernel on the call's
                             stream and report per-kernel device times in ss_stats;
                             2: only around the dominant kernel (level-0 count);
                             3: in-kernel timeline stamps (ss_stats.tl_us) */
    int32_t b_deep;       /* buckets of the levels after the first: 0 = b_exact, else a
                             power of two in [4, 256] (each level is a full SampleSelect
                             level of Fig. 1; only its bucket count differs) */
    int32_t classify;     /* bucket classification in the count kernel: 0 = auto (cell
                             lookup table for 4-byte keys and b <= 256 where its
                             marker cells are light, else the Fig. 4 tree walk);
                             1 = always the tree walk.  Same buckets either way. default 0 */
    uint64_t seed;        /* sampling seed (reading R7). default 0x5A17 */
    int32_t fused_filter; /* exact levels: 1 = (default) fused levels where n_l >= spec_min_n:
                             the level's sample (16384 keys, or sample_size) gives a key
                             window around rank k (two order statistics, no sort) and one
                             pass counts the keys below it and copies the keys inside it to
                             the next level (reading R21: a SampleSelect level with two
                             splitters, no oracle bytes, no filter pass; a miss re-runs the
                             level with the paper's tree); 0 = always the paper's level:
                             b-bucket tree, oracle bytes, filter kernel (§IV.B).  Same answer. */
    float spec_z;         /* window half-width in standard deviations of the sample rank of k
                             (Binomial(s, k/n)); default 3 (miss probability ~3e-3 per level) */
    int64_t spec_min_n;   /* levels with at least this many elements (host estimate) are fused
                             levels. default 2^16 */
    float spec_max_frac;  /* speculate only if the window holds at most this fraction of the
                             sample. default 0.25 */
    int32_t shard_gather_log2; /* ss_select_sharded: survivors are gathered onto every rank once
                             the level holds at most 2^shard_gather_log2 elements (then the
                             single-GPU levels finish); 0 = default 20, else in [12, 28] */
    int32_t directed;     /* fused levels after the first: 1 = (default) the previous fused level
                             counts the keys it copies in 1024 equal key bins and the bin
                             holding the rank is this level's window (reading R28: exact, no
                             sample, cannot miss); 0 = every fused level draws a sample. */
    int32_t upper_onepass;/* ss_select_upper: 1 = (default) the top-k fusion of §IV.I in one pass:
                             a fused level 0 also copies every key above its window to d_out
                             while it copies the window, and after the select the window's
                             keys > result and the copies of result complete d_out (no second
                             read of the input), for outputs n - k <= n / 4; falls back to the
                             two-pass path when level 0 is not a fused hit.  0 = always two
                             passes (select, then one threshold pass over the input).  Same
                             multiset either way. */
} ss_config;

/* Per-call statistics of the last ss_select / ss_approx_select. */
typedef struct {
    int32_t levels;                    /* count passes executed (0 = base case only) */
    int32_t equality_exit;             /* 1 if the answer came from an equality bucket (§IV.C) */
    int64_t n_level[SS_MAX_LEVELS];    /* n_l entering level l (n_level[levels] = base-case size) */
    int32_t bucket[SS_MAX_LEVELS];     /* bucket chosen at level l */
    double bytes_algorithmic;          /* DESIGN.md §Roofline byte model for this call */
    int32_t launches;                  /* kernels this call launched */
    int64_t h2d_bytes;                 /* host->device bytes this call copied (host-input calls) */
    int64_t d2h_bytes;                 /* device->host bytes this call copied (result block) */
    float ms_kernel[SS_MAX_LEVELS][3]; /* profile=1: device ms of K1 (sample/tree or base
                                          case), K2 (count+tail), K5 (filter) per level;
                                          profile=3: last-CTA exit - first-CTA start */
    float tl_us[SS_MAX_LEVELS][3][2];  /* profile=3 (timeline): [start, end] of each kernel in
                                          us after the call's init kernel, from %globaltimer
                                          stamps taken inside the kernels (no events, so the
                                          PDL overlap of the chain is kept); -1 = not run */
    int32_t lut_ctas;                  /* level-0 count CTAs that classified with the cell
                                          lookup table (0 = all walked the tree) */
    int32_t lut_marker;                /* level 0: whole buckets inside the table's marker
                                          cells (the auto rule walks the tree when >= 2) */
    int32_t spec_levels;               /* bit l: level l ran the fused speculative filter */
    int32_t fused_levels;              /* bit l: ... and its window held bucket j (hit: the
                                          captured window is level l+1; else the fallback
                                          filter re-read level l) */
    int64_t upper_greater;             /* ss_select_upper: #{x > result} (the rest of the
                                          output is copies of result) */
    float ms_upper_gather;             /* ss_select_upper with profile != 0: device ms of the
                                          upper_gather_kernel pass (CUDA events) */
    float ms_quick;                    /* ss_quickselect with profile != 0: device ms from the
                                          init kernel to the last batch (CUDA events) */
    int32_t incomplete_rounds;         /* ss_select: times the planned levels ended with more than
                                          base_case elements left and the host enqueued one more
                                          level (an unlucky sample; 0 almost always) */
    int32_t shard_levels;              /* ss_select_sharded: sharded levels run before the gather
                                          (n_level[l] for l < shard_levels are global sizes,
                                          n_level[shard_levels] the gathered size) */
    int32_t shard_ranks;               /* ss_select_sharded: ranks of the communicator */
    int64_t workspace_bytes;           /* ss_select: device bytes the context owns after the call
                                          (level buffers sized for the planned survivors; they
                                          grow only when a level would not fit) */
    int32_t upper_onepass;             /* ss_select_upper: 1 if the one-pass top-k path produced
                                          d_out (see ss_config.upper_onepass), 0 if two passes ran */
    int32_t pad_;
} ss_stats;

/* ---- context --------------------------------------------------------- */
/* Create a context bound to CUDA device `device` (>= 0). */
ss_status ss_create(int device, ss_context** out);
void      ss_destroy(ss_context* ctx);
ss_status ss_get_config(const ss_context* ctx, ss_config* out);
ss_status ss_set_config(ss_context* ctx, const ss_config* cfg);
ss_status ss_last_stats(const ss_context* ctx, ss_stats* out);
const char* ss_last_error(const ss_context* ctx);
/* Totals accumulated over all calls since the last reset: per (level, kernel)
 * device ms summed from the profile events (ms_sum[SS_MAX_LEVELS*3], index
 * level*3 + kernel, kernel 0 = K1, 1 = K2, 2 = K5) and how many launches each
 * sum covers (count[SS_MAX_LEVELS*3]); total kernel launches and calls.  Any
 * output pointer may be NULL.  reset != 0 zeroes the totals after reading. */
ss_status ss_profile_totals(ss_context* ctx, double* ms_sum, int64_t* count, int64_t* launches,
                            int64_t* calls, int32_t reset);
const char* ss_status_string(ss_status s);
int       ss_abi_version(void);

/* ---- exact selection (§II; Fig. 1 L95-127; §IV.B-E) --------------
 * Writes the element of rank k of d_data[0..n) (4 or 8 bytes, the dtype's
 * bits) to *h_result.  Device input, host result; synchronises `stream`. */
ss_status ss_select(ss_context* ctx, ss_dtype dt, const void* d_data, int64_t n, int64_t k,
                    void* h_result, void* stream);

/* Same, input in HOST memory: the call copies it to device workspace on
 * `stream` (pinned memory makes that copy asynchronous and fast). */
ss_status ss_select_host(ss_context* ctx, ss_dtype dt, const void* h_data, int64_t n, int64_t k,
                         void* h_result, void* stream);

/* ---- approximate selection (§II.C; §V.G) ---------------
 * One level with b buckets (power of two in [4, 1024]): sample, count, and
 * return the splitter s_i whose rank r_i is closest to k (ties: smaller i),
 * with its exact rank *h_rank = #{x < s_i} (reading R11). */
ss_status ss_approx_select(ss_context* ctx, ss_dtype dt, const void* d_data, int64_t n, int64_t k,
                           int32_t b, void* h_result, int64_t* h_rank, void* stream);
ss_status ss_approx_select_host(ss_context* ctx, ss_dtype dt, const void* h_data, int64_t n,
                                int64_t k, int32_t b, void* h_result, int64_t* h_rank, void* stream);

/* ---- selection with all larger elements: top-k fusion (§IV.I) ----
 * "not only the kth-smallest element is required, but also all larger
 * elements": writes the element of rank k to *h_result (as ss_select) and the
 * n-k elements of ranks k..n-1 (IEEE totalOrder / numeric order, reading R3)
 * to d_out[0..n-k), a caller-owned DEVICE buffer of at least n-k elements of
 * dtype dt that must not overlap d_data.  The output is a multiset: its order
 * is unspecified (elements > result first, then n-k-#{x > result} copies of
 * result; reading R22).  Errors as ss_select; d_out == NULL is
 * SS_ERR_INVALID_ARGUMENT.  Synchronises `stream`. */
ss_status ss_select_upper(ss_context* ctx, ss_dtype dt, const void* d_data, int64_t n, int64_t k,
                          void* d_out, void* h_result, void* stream);

/* ---- multi-rank selection (§VI; reading R23) ------
 * Writes the element of rank h_ks[i] to h_results[i] (m elements of dtype dt,
 * host memory) for i < m, 1 <= m <= 1024, every h_ks[i] in [0, n) (any order,
 * repeats allowed).  For n >= 2^20 and m >= 4 the ranks share one sample, one splitter
 * tree and one count pass; each distinct bucket holding a rank is extracted
 * once and finished by the single-rank path.  Results are bit-identical to m
 * calls of ss_select.  d_data: device, naturally aligned.  Synchronises. */
ss_status ss_select_multi(ss_context* ctx, ss_dtype dt, const void* d_data, int64_t n, int32_t m,
                          const int64_t* h_ks, void* h_results, void* stream);

/* ---- single steps of one level (per-kernel parity tests, sharded driver) --
 * All are asynchronous on `stream` and touch only the buffers passed in.  Keys
 * are the order-preserving unsigned images of the values (u32 for 4-byte,
 * u64 for 8-byte dtypes; reading R3), so tree/splitter buffers hold keys.     */

/* K1a (§IV.B-a; reading R7): draw sample slots [slot_begin,
 * slot_begin+count) of level `level` uniformly with replacement from
 * d_data[0..n); writes `count` KEYS to d_sample_keys. */
ss_status ss_step_sample(ss_context* ctx, ss_dtype dt, const void* d_data, int64_t n, int32_t level,
                         int64_t slot_begin, int64_t count, void* d_sample_keys, void* stream);

/* K1b (§IV.B-a, §IV.C, Fig. 3): sort s sample keys in one
 * CTA (bitonic, §IV.D), pick splitters s_i = sorted[floor(i s / b)], apply
 * the equality fix-up if `fixup` != 0, write the heap-ordered tree
 * d_tree[b-1], the sorted (fixed) splitters d_splitters[b-1] and the
 * equality flags d_eq[b] (uint8).  s: power of two <= 16384. */
ss_status ss_step_tree(ss_context* ctx, ss_dtype dt, const void* d_sample_keys, int32_t s, int32_t b,
                       int32_t fixup, void* d_tree, void* d_splitters, uint8_t* d_eq, void* stream);

/* Oracle-byte layout (§IV.B-b: one bucket byte per element).  The
 * count kernel stores the bytes of 16-byte input vectors as aligned words, so
 * the byte of element i lives at d_oracles[ss_oracle_offset(dt, d_data, n) + i],
 * with the offset in [0, 16) chosen so that the bytes of the input's first
 * 16-byte-aligned element are 16-byte aligned.  An oracle buffer therefore
 * needs n + 16 bytes and a 16-byte-aligned base.  Pure host arithmetic (no
 * device access); returns -1 for an unknown dtype. */
int64_t ss_oracle_offset(ss_dtype dt, const void* d_data, int64_t n);

/* K2 (§IV.B-b, Fig. 4, §IV.G): classify d_data[0..n) against the tree (keys),
 * write per-bucket totals d_totals[b] (uint64, overwritten) and, if
 * d_oracles != NULL (requires b <= 256), the bucket byte of element i to
 * d_oracles[ss_oracle_offset(dt, d_data, n) + i] (see above: >= n + 16 bytes,
 * 16-byte-aligned base, else SS_ERR_INVALID_ARGUMENT).  Also records the
 * per-CTA counts the next ss_step_filter on the same data needs. */
ss_status ss_step_count(ss_context* ctx, ss_dtype dt, const void* d_data, int64_t n, const void* d_tree,
                        int32_t b, uint64_t* d_totals, uint8_t* d_oracles, void* stream);

/* K5 (§IV.B-c): stable compaction of the elements i with oracle
 * byte == bucket (layout of ss_oracle_offset; the buffer ss_step_count wrote,
 * 16-byte-aligned base) into d_out (values, input order).  Must follow
 * ss_step_count on the same d_data and n (it uses that pass's per-CTA
 * counts).  Writes the number of elements copied to *d_count (uint64). */
ss_status ss_step_filter(ss_context* ctx, ss_dtype dt, const void* d_data, int64_t n,
                         const uint8_t* d_oracles, int32_t bucket, void* d_out, uint64_t* d_count,
                         void* stream);

/* Atomics ablation (§V.E, Fig. 6, Fig. 8
 * right L1093-1120): the same per-bucket totals as ss_step_count (d_totals[b]
 * uint64, overwritten; no oracle bytes) from a plain Fig. 4 count kernel whose
 * bucket increments are applied by `mode`:
 *   0 SS_ABL_SHARED      shared-memory atomics
 *   1 SS_ABL_SHARED_WA   shared, warp-aggregated (__match_any_sync)
 *   2 SS_ABL_SHARED_FIG6 shared, warp-aggregated by Fig. 6's per-bit ballots (reading R13)
 *   3 SS_ABL_GLOBAL      global atomics on d_totals
 *   4 SS_ABL_GLOBAL_WA   global, warp-aggregated
 * b: power of two in [2, 1024]; tree as for ss_step_count.  Not used by
 * ss_select (the product's count kernel has its own histogram);
 * it exists to measure the paper's design space on B200. */
enum { SS_ABL_SHARED = 0, SS_ABL_SHARED_WA = 1, SS_ABL_SHARED_FIG6 = 2, SS_ABL_GLOBAL = 3,
       SS_ABL_GLOBAL_WA = 4 };
ss_status ss_step_count_ablation(ss_context* ctx, ss_dtype dt, const void* d_data, int64_t n,
                                 const void* d_tree, int32_t b, int32_t mode, uint64_t* d_totals,
                                 void* stream);

/* QuickSelect, the paper's own GPU comparison baseline (
 * §IV.F, Fig. 5, §V.D).  Same result as
 * ss_select (the element of rank k under totalOrder, 0-based) by a single
 * pivot per level: the pivot is the median of a 1024-key sample, one pass
 * splits the level three ways (< pivot to the left of the next buffer,
 * > pivot to the right, == pivot only counted: reading R24), and the level
 * recurses into the part holding k or returns the pivot; levels with
 * n_l <= base_case finish in one CTA.  d_data: caller-owned device array,
 * read only; n in [1, 2^32).  The context owns two n-element level buffers
 * (allocated on first use, grown on demand).  Optional outputs:
 * h_n_level[0..n_level_cap) receives n_l per level (0 past the last one),
 * *h_levels the number of partition passes.  Synchronises `stream`.
 * Errors: SS_ERR_INVALID_ARGUMENT for the ss_select conditions, n >= 2^32,
 * n_level_cap < 0 or a positive cap with NULL h_n_level. */
ss_status ss_quickselect(ss_context* ctx, ss_dtype dt, const void* d_data, int64_t n, int64_t k,
                         void* h_result, int64_t* h_n_level, int32_t n_level_cap, int32_t* h_levels,
                         void* stream);

/* ---- sharded (multi-GPU) selection support -------------------
 * The sharded driver (paper_conf_ipps_ribizela19_b200/sharded.py) runs one
 * process per GPU, exchanges the sample keys (allgather) and bucket totals
 * (allreduce) with NCCL through torch.distributed, and calls these steps. */

/* K3/K4 (§IV.G; Fig. 1 lines 11-16; reading R6): given GLOBAL bucket
 * totals d_totals[b] (uint64) and rank k, find the unique j with
 * r_j <= k < r_{j+1}; write d_out[0]=j, d_out[1]=k-r_j, d_out[2]=totals[j],
 * d_out[3]=eq[j] (int64[4]); reads the equality flags d_eq[b]. */
ss_status ss_step_search(ss_context* ctx, const uint64_t* d_totals, int32_t b, int64_t k,
                         const uint8_t* d_eq, int64_t* d_out, void* stream);

/* Inverse key map: turn `count` keys into values of dtype dt (in place OK). */
ss_status ss_step_keys_to_values(ss_context* ctx, ss_dtype dt, const void* d_keys, int64_t count,
                                 void* d_values, void* stream);

/* ---- sharded (multi-GPU) exact selection --------------------
 * One process (or, with a local group, one host thread) per rank, one context
 * per rank.  Every rank holds a contiguous shard d_shard[0..n_local) (device,
 * naturally aligned, read only; n_local >= 0, shards may be empty or of
 * different sizes) and calls ss_select_sharded with the SAME k_global; every
 * rank receives the element of rank k_global (0-based, reading R3) of the
 * union of all shards in *h_result.  Per level every rank draws its share of
 * the level's sample (proportional to its share of the level), the sample keys
 * are exchanged so every rank sorts the identical sample and derives the
 * identical window (reading R21), each rank streams its own shard through the
 * fused count+filter kernel, and the per-rank counts {below, window} -- the
 * level's bucket counts -- are exchanged so every rank takes the identical
 * decision on the device.  Once the level holds at most
 * 2^shard_gather_log2 elements the survivors are gathered onto every rank and
 * the single-GPU levels finish.  Exchanges are sum-allreduces over buffers in
 * which each rank fills disjoint slots.  No host round trip until the result.
 * Synchronises `stream`.  Errors: SS_ERR_INVALID_ARGUMENT (no communicator,
 * NULL pointers, k_global outside [0, sum of n_local)), SS_ERR_NCCL, as
 * ss_select otherwise.  Every rank must make the same sequence of sharded
 * calls (the exchanges are collective). */

/* NCCL unique id (128 bytes) for ss_comm_init; rank 0 creates it and the
 * caller broadcasts it (e.g. torch.distributed).  NCCL is loaded at run time
 * (libnccl.so.2, or $SS_NCCL_LIB); SS_ERR_NCCL if unavailable. */
ss_status ss_nccl_unique_id(char out_id[128]);

/* Bind a NCCL communicator of `nranks` ranks to the context (collective over
 * all ranks, each on its context's device).  Replaces a previous one. */
ss_status ss_comm_init(ss_context* ctx, const char id[128], int nranks, int rank);

/* In-process group of `nranks` (<= 16) ranks: contexts in different host
 * threads of one process (same device, or peer-accessible devices) exchange
 * through device-to-device reads with host barriers.  For tests of the
 * sharded path on one GPU ("virtual ranks"); not graph-capturable. */
ss_status ss_local_group_create(int nranks, ss_local_group** out);
void      ss_local_group_destroy(ss_local_group* group);
ss_status ss_comm_init_local(ss_context* ctx, ss_local_group* group, int rank);

ss_status ss_select_sharded(ss_context* ctx, ss_dtype dt, const void* d_shard, int64_t n_local,
                            int64_t k_global, void* h_result, void* stream);

/* ---- convenience calls mirroring north_star's select(data, n, k) ---------
 * A thread-local default context per current CUDA device (created on first
 * use), the current device's legacy default stream, device input, host
 * result.  Same semantics and errors as ss_select / ss_approx_select. */
ss_status ss_select_f32(const float* d_data, int64_t n, int64_t k, float* h_result);
ss_status ss_select_f64(const double* d_data, int64_t n, int64_t k, double* h_result);
ss_status ss_select_i32(const int32_t* d_data, int64_t n, int64_t k, int32_t* h_result);
ss_status ss_select_i64(const int64_t* d_data, int64_t n, int64_t k, int64_t* h_result);
ss_status ss_approx_select_f32(const float* d_data, int64_t n, int64_t k, int32_t b, float* h_result,
                               int64_t* h_rank);

#ifdef __cplusplus
}
#endif
#endif /* SAMPLESELECT_H */
