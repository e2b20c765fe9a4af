// quickselect.cuh -- GPU QuickSelect, the paper's own comparison baseline
// (§IV.F, Fig. 5, §V.D).
//
// "QUICKSELECT only chooses a single so-called pivot element based on which
// the input data is bipartitioned" (L405-408); the bipartition grows the
// elements smaller than the pivot from the left of the output and the larger
// ones from the right (Fig. 5: o = smaller ? l++ : r--).  Built on the same
// infrastructure as SampleSelect (L399-401): order-preserving keys, the
// counter-based sample (reading R7), the one-CTA base case (Fig. 1 l.2-5).
//
// Reading R24: Fig. 5 is a two-way split (< pivot | >= pivot),
// which never shrinks when the pivot is the minimum of an all-equal run.  The
// kernel splits three ways in the same pass -- keys < p go left, keys > p go
// right, keys == p are only counted (n_l - L - G of them) -- so rank k is
// either in the left part, equal to the pivot (early exit, like the equality
// buckets of §IV.C) or in the right part, and every level strictly shrinks.
// The pivot is the median of a 256-key sample of the level (the paper does
// not say how it picks the pivot).
//
// GPU shape per level l (input n_l, output buffer l & 1):
//   qs_pivot_kernel     1 CTA: base case if n_l <= B, else sample, sort, median
//   qs_partition_kernel one wave: per 4096-key tile a CTA scan of the per-thread
//                       < / > counts, ONE 64-bit global atomic per tile reserves
//                       both output ranges (low word: left, high word: right),
//                       the keys are staged in shared memory in rank order and
//                       copied out as two contiguous runs (the paper's quick-s uses
//                       shared atomics in the block + a global offset, L411-414)
//   qs_decide_kernel    1 thread: next range, rank, or the pivot as the answer
// The host enqueues levels in batches and checks the done flag between them.
#pragma once
#include "common.cuh"

namespace ss {

constexpr int QS_MAX_LEVELS = 128;
constexpr int QS_SAMPLE = 256;  // pivot = sample median (R24)
constexpr u32 QP_THREADS = 256;
#ifndef SS_QP_MINB
#define SS_QP_MINB 6
#endif
#ifndef SS_QP_IPT
#define SS_QP_IPT 16
#endif
// CTAs per SM: 4-byte keys 6 (<= 40 registers; measured 1.14 vs 1.19 ms at
// 2^28 with 4), 8-byte keys 4 (<= 64 registers: 6 spills, 2.70 vs 1.78 ms)
constexpr int QP_MINB = SS_QP_MINB;
template <typename T> constexpr int qp_minb() { return sizeof(T) == 4 ? QP_MINB : 4; }
constexpr int QP_IPT = SS_QP_IPT;     // default 16 keys per thread: 4096-key tiles

struct QsCtl {
    u64 n, k, off;               // level input: n_l elements at buffer + off, rank k_l
    unsigned long long lg;       // packed #{key < p} (low 32 bits) | #{key > p} (high 32 bits)
    u64 pivot;                   // pivot key
    u64 bits;                    // answer (raw bits of T)
    u32 done, levels, eq_exit, pad_;
    u64 n_level[QS_MAX_LEVELS];  // n_l entering level l
    u64 n_out[QS_MAX_LEVELS];    // L + G written by level l's partition
};

static __global__ void qs_init_kernel(QsCtl* c, u64 n, u64 k) {
    c->n = n;
    c->k = k;
    c->off = 0;
    c->lg = 0;
    c->pivot = 0;
    c->bits = 0;
    c->done = 0;
    c->levels = 0;
    c->eq_exit = 0;
}

template <typename T>
__device__ __forceinline__ const T* qs_input(const T* in0, const T* buf_in, const QsCtl* c, int level) {
    return (level == 0 ? in0 : buf_in) + c->off;
}

template <typename T>
__global__ void __launch_bounds__(1024)
qs_pivot_kernel(const T* __restrict__ in0, const T* __restrict__ buf_in, QsCtl* __restrict__ c, u32 B, u64 seed,
                int level) {
    typedef typename Traits<T>::Key K;
    __shared__ __align__(16) K keys[QS_SAMPLE];
    __shared__ __align__(16) u32 hist[32 * 256];
    __shared__ u32 misc[16];
    __shared__ K red[66];
    __shared__ u32 misc_rank[QS_SAMPLE];
    extern __shared__ __align__(16) unsigned char qs_smem[];   // the base case's keys (B of them)
    if (c->done) return;
    const u64 n = c->n;
    const T* in = qs_input(in0, buf_in, c, level);
    if (n <= B) {                                 // Fig. 1 lines 2-5: base case
        K r = block_select_base<T>(in, (u32)n, (u32)c->k, reinterpret_cast<K*>(qs_smem), hist, misc, red);
        if (threadIdx.x == 0) {
            c->n_level[level] = n;
            c->n_out[level] = 0;
            c->bits = Traits<T>::from_key(r);
            c->done = 1;
        }
        return;
    }
    // the median by stable rank: thread t ranks sample key t & 255 against
    // the quarter t >> 8 of the sample, the four partial ranks are summed in
    // shared memory; the key of stable rank QS_SAMPLE / 2 is sorted[QS_SAMPLE / 2]
    const u64 base = level_base(seed, level);    // reading R7
    u32* rank = misc_rank;
    const u32 t = threadIdx.x & (QS_SAMPLE - 1), part = threadIdx.x / QS_SAMPLE;
    if (threadIdx.x < QS_SAMPLE) {
        keys[t] = load_key(in + sample_index(base, t, n));
        rank[t] = 0;
    }
    __syncthreads();
    if (part < 1024 / QS_SAMPLE) {
        const K me = keys[t];
        u32 r = 0;
        constexpr u32 Q = QS_SAMPLE / (1024 / QS_SAMPLE);
        for (u32 j = part * Q; j < (part + 1) * Q; ++j) {
            const K o = keys[j];
            r += (o < me) | ((o == me) & (j < t));
        }
        atomicAdd(&rank[t], r);
    }
    __syncthreads();
    if (threadIdx.x < QS_SAMPLE && rank[t] == QS_SAMPLE / 2) {
        c->n_level[level] = n;
        c->pivot = (u64)keys[t];
        c->lg = 0;
    }
}

// One pass over the level: tile = QP_THREADS * IPT keys, thread t holds keys
// t, t + 256, ... (coalesced 4/8-byte loads).  Each thread counts its own
// < / > keys; a warp scan and a CTA scan of the packed counts (left in the
// low 16 bits, right in the high 16 bits: a tile holds <= 4096 keys) give
// every thread its slots in the tile, one packed 64-bit atomic reserves the
// tile's left and right output ranges, the keys are staged in shared memory
// (left run upwards from 0, right run downwards from TILE - 1) and both runs
// are copied out with consecutive threads on consecutive addresses.  Order
// inside a level is unspecified (reading R24).  Padding (i >= n) is neither.
template <typename T, int IPT>
__global__ void __launch_bounds__(QP_THREADS, qp_minb<T>())
qs_partition_kernel(const T* __restrict__ in0, const T* __restrict__ buf_in, T* __restrict__ out,
                    QsCtl* __restrict__ c, int level) {
    typedef typename Traits<T>::Key K;
    constexpr u32 NW = QP_THREADS / 32;
    constexpr u32 TILE = QP_THREADS * IPT;
    static_assert(TILE < 65536, "packed 16-bit tile counts");
    __shared__ u32 wtot[NW];
    __shared__ unsigned long long base_s;
    __shared__ u32 tot_s;
    __shared__ K stage[TILE];
    if (c->done) return;
    const u64 n = c->n;
    const K pk = (K)c->pivot;
    const K* in = reinterpret_cast<const K*>(qs_input(in0, buf_in, c, level));
    K* o = reinterpret_cast<K*>(out);
    const u32 lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (u64 t0 = (u64)blockIdx.x * TILE; t0 < n; t0 += (u64)gridDim.x * TILE) {
        const u64 rem = n - t0;
        const K* p = in + t0 + threadIdx.x;
        K x[IPT];
        u32 lt = 0, gt = 0;                      // bit j: key j goes left / right
        if (rem >= TILE) {
#pragma unroll
            for (int j = 0; j < IPT; ++j) x[j] = __ldcs(p + j * QP_THREADS);
#pragma unroll
            for (int j = 0; j < IPT; ++j) {
                const K key = Traits<T>::to_key(x[j]);
                lt |= (u32)(key < pk) << j;
                gt |= (u32)(key > pk) << j;
            }
        } else {
#pragma unroll
            for (int j = 0; j < IPT; ++j) {
                const bool v = (u64)(j * QP_THREADS + threadIdx.x) < rem;
                x[j] = v ? __ldcs(p + j * QP_THREADS) : (K)0;
                const K key = Traits<T>::to_key(x[j]);
                lt |= (u32)(v && key < pk) << j;
                gt |= (u32)(v && key > pk) << j;
            }
        }
        const u32 mine = (u32)__popc(lt) | ((u32)__popc(gt) << 16);
        u32 incl = mine;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const u32 y = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= (u32)d) incl += y;
        }
        if (lane == 31) wtot[warp] = incl;
        __syncthreads();
        unsigned long long old = 0;              // thread 0: the tile's reservation (used after staging)
        if (threadIdx.x == 0) {
            u32 sum = 0;
#pragma unroll
            for (u32 w = 0; w < NW; ++w) {
                const u32 t = wtot[w];
                wtot[w] = sum;
                sum += t;
            }
            tot_s = sum;
            const u32 sl = sum & 0xffffu, sg = sum >> 16;
            if (sum) old = atomicAdd(&c->lg, (unsigned long long)sl | ((unsigned long long)sg << 32));
        }
        __syncthreads();
        const u32 off = wtot[warp] + incl - mine;
        u32 ql = off & 0xffffu, qg = off >> 16;
#pragma unroll
        for (int j = 0; j < IPT; ++j) {
            if ((lt >> j) & 1) stage[ql++] = x[j];
            if ((gt >> j) & 1) stage[TILE - 1 - qg++] = x[j];
        }
        if (threadIdx.x == 0) base_s = old;      // the atomic's latency overlapped the staging
        __syncthreads();
        const unsigned long long bs = base_s;
        const u32 tl = tot_s & 0xffffu, tg = tot_s >> 16;
        const u64 bl = bs & 0xffffffffull, bg = bs >> 32;
        for (u32 i = threadIdx.x; i < tl; i += QP_THREADS) o[bl + i] = stage[i];
        for (u32 i = threadIdx.x; i < tg; i += QP_THREADS) o[n - 1 - (bg + i)] = stage[TILE - 1 - i];
        __syncthreads();                                   // wtot/tot_s/base_s/stage reused by the next tile
    }
}

template <typename T>
__global__ void qs_decide_kernel(QsCtl* c, int level) {
    if (c->done) return;
    const u64 n = c->n, k = c->k, lg = c->lg;
    const u64 L = lg & 0xffffffffull, G = lg >> 32, E = n - L - G;
    c->levels = (u32)level + 1;
    c->n_out[level] = L + G;
    if (k < L) {                                  // rank k among the smaller keys (left part)
        c->n = L;
        c->off = 0;
    } else if (k < L + E) {                       // rank k is a copy of the pivot
        c->bits = Traits<T>::from_key((typename Traits<T>::Key)c->pivot);
        c->eq_exit = 1;
        c->done = 1;
    } else {                                      // right part: the last G slots of the output
        c->n = G;
        c->off = n - G;
        c->k = k - L - E;
    }
}

}  // namespace ss
