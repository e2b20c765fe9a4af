// dist_kernels.cuh -- the per-rank kernels of the sharded (multi-GPU) level
// (driver: sharded.cuh).  Every rank holds a contiguous shard; the
// global rank k and the level's global size N are the same on every rank.
// One sharded level is one SampleSelect level with the fused window (reading
// R21) distributed over the ranks:
//
//   dsample  this rank draws its share of the level's s sample slots
//            (proportional to its share of N, reading R7 per rank) into its
//            slots of the sample buffer             -> exchange 1 (sample keys)
//   K1       every rank ranks the identical sample (sample_rank_kernel)
//   K2'      window_kernel: counts #{x < klo}, copies the window [klo, khi) of
//            the shard to the next level's buffer, writes this rank's row
//            {below, window, cap, n}                -> exchange 2 (the counts)
//   decide   every rank sums the rows -- the identical global decision: k in
//            the window (the window is the next level, rank k - below), an
//            equality window holding k (done, §IV.C), or a miss (the next
//            level is the side of the window holding k, a "directed" window)
//   dcopy    a miss or a pass-through level copies the shard unchanged
//
// Once the level is small (N <= G) the ranks' survivors are gathered into one
// G-element buffer on every rank (exchange 3) and every rank finishes the
// selection with the single-GPU levels (identical on every rank).
// The exchanges are integer sum-allreduces over buffers in which every rank
// writes disjoint slots (comm.cuh).
#pragma once
#include "common.cuh"

namespace ss {

constexpr int DIST_MAX_RANKS = 16;
constexpr int DIST_REC = 4;   // row: below, window elements, window elements + chunk padding (cap), n

// Per call: rank r's slot of the level-0 sizes exchange.
static __global__ void dist_sizes_kernel(u64* __restrict__ send, int P, int rank, u64 n_local) {
    pdl_wait();
    pdl_trigger();
    for (int q = threadIdx.x; q < P; q += blockDim.x) send[q] = q == rank ? n_local : 0ull;
}

// After the sizes exchange: k must be a rank of the union.
static __global__ void dist_check_kernel(const u64* __restrict__ sizes, int P, u64 k, SelectResult* res) {
    pdl_wait();
    pdl_trigger();
    if (threadIdx.x != 0) return;
    u64 N = 0;
    for (int q = 0; q < P; ++q) N += sizes[q];
    res->dist_n = N;
    if (k >= N) {
        res->dist_halt = 2;
        res->done = 1;
    }
}

// Sample slots owned by `rank`: [floor(s P_r / N), floor(s P_{r+1} / N)),
// P_r = sum of the sizes of ranks < r (each rank draws in proportion to its
// share of the level, so the union's sample is uniform over the union).
__host__ __device__ __forceinline__ void dist_slot_range(const u64* sizes, int P, int rank, u64 s, u64* lo,
                                                         u64* hi) {
    u64 N = 0, pre = 0;
    for (int q = 0; q < P; ++q) {
        if (q < rank) pre += sizes[q];
        N += sizes[q];
    }
    if (N == 0) {
        *lo = *hi = 0;
        return;
    }
    // s <= 2^14 and N < 2^49: the products fit in 64 bits
    *lo = s * pre / N;
    *hi = s * (pre + sizes[rank]) / N;
}

template <typename T>
__global__ void dist_sample_kernel(const T* __restrict__ in, LevelCtl* __restrict__ ctl,
                                   SelectResult* __restrict__ res, const u64* __restrict__ sizes, int P, int rank,
                                   int s, u64 seed, int level, u64 G, typename Traits<T>::Key* __restrict__ ksend,
                                   u64* __restrict__ rsend) {
    typedef typename Traits<T>::Key K;
    pdl_wait();
    pdl_trigger();
    const u64 n = ctl->n;
    const u32 gid = blockIdx.x * blockDim.x + threadIdx.x, gsz = gridDim.x * blockDim.x;
    for (u32 i = gid; i < (u32)(P * DIST_REC); i += gsz) rsend[i] = i == (u32)(rank * DIST_REC + 3) ? n : 0ull;
    if (res->done) return;
    u64 N = 0;
    for (int q = 0; q < P; ++q) N += sizes[q];
    if (gid == 0) {
        ctl->gn = N;
        ctl->pass = N <= G;
        ctl->pre = 1;
    }
    u64 lo, hi;
    dist_slot_range(sizes, P, rank, (u64)s, &lo, &hi);
    const u64 base = level_base(seed, level);   // reading R7, slot j of the level's sample
    for (u32 j = gid; j < (u32)s; j += gsz)
        ksend[j] = (j >= lo && j < hi) ? load_key(in + sample_index(base, j, n)) : (K)0;
}

// Every rank sums the rows of the counts exchange and takes the same decision.
template <typename T>
__global__ void dist_decide_kernel(LevelCtl* __restrict__ ctl, LevelCtl* __restrict__ ctl_next,
                                   SelectResult* __restrict__ res, const u64* __restrict__ rows, int P, int rank,
                                   u64* __restrict__ sizes_next, int level) {
    typedef typename Traits<T>::Key K;
    pdl_wait();
    pdl_trigger();
    if (threadIdx.x != 0 || res->done) return;
    const u64 N = ctl->gn, k = ctl->k;
    u64 below = 0, W = 0, C = 0;
    for (int q = 0; q < P; ++q) {
        below += rows[q * DIST_REC + 0];
        W += rows[q * DIST_REC + 1];
        C += rows[q * DIST_REC + 2];
    }
    if (level < 32) {
        res->n_level[level] = (long long)N;
        res->bucket[level] = -1;
    }
    ctl_next->k = k;
    ctl_next->gn = N;
    ctl_next->n = ctl->n;
    ctl->hit = 0;
    if (ctl->pass) {                                 // pass-through: the shard is copied unchanged
        for (int q = 0; q < P; ++q) sizes_next[q] = rows[q * DIST_REC + 3];
        return;
    }
    res->levels = level + 1;
    res->spec_levels |= 1u << level;
    const bool inwin = below <= k && k < below + W;
    const K klo = (K)ctl->klo, kspan = (K)ctl->kspan;
    if (inwin && ctl->spec_eq) {                     // §IV.C: the window is one value
        res->bits = Traits<T>::from_key(klo);
        res->eq_exit = 1;
        res->done = 1;
        return;
    }
    if (inwin) {                                     // the (padded) windows are the next level
        ctl->hit = 1;
        res->fused_levels |= 1u << level;
        ctl_next->n = rows[rank * DIST_REC + 2];
        ctl_next->gn = C;
        ctl_next->k = k - below + (pad_low(klo, kspan) ? C - W : 0ull);   // (padding below the window)
        for (int q = 0; q < P; ++q) sizes_next[q] = rows[q * DIST_REC + 2];
        return;
    }
    // miss: the next level is the side of the window that holds k, streamed
    // from a copy of this level (no sample needed, and it always shrinks:
    // the window held at least one element of the level)
    for (int q = 0; q < P; ++q) sizes_next[q] = rows[q * DIST_REC + 3];
    ctl_next->directed = 1;
    if (k < below) {                                 // [min, klo)
        ctl_next->klo = 0;
        ctl_next->kspan = (u64)klo;
        ctl_next->dfrac = N ? (float)((double)below / (double)N) : 1.0f;
    } else {                                         // [klo + kspan, max]
        const K khi = (K)(klo + kspan);
        ctl_next->klo = (u64)khi;
        ctl_next->kspan = (u64)(K)((K)0 - khi);
        ctl_next->dfrac = N ? (float)((double)(N - below - W) / (double)N) : 1.0f;
    }
}

// A miss or a pass-through level: the next level is this shard unchanged.
template <typename T>
__global__ void dist_copy_kernel(const T* __restrict__ in, T* __restrict__ out, const LevelCtl* __restrict__ ctl,
                                 const SelectResult* __restrict__ res) {
    pdl_wait();
    pdl_trigger();
    if (res->done || ctl->hit) return;
    const u64 n = ctl->n;
    for (u64 i = blockIdx.x * (u64)blockDim.x + threadIdx.x; i < n; i += (u64)gridDim.x * blockDim.x) out[i] = in[i];
}

// Gather: rank r writes its survivors at positions [off_r, off_r + n_r) of a
// G-element buffer (zeros elsewhere; exchange 3 sums the buffers), and the
// single-GPU tail's first level gets n = N, rank k.  If the survivors do not
// fit, the call halts (res->done) and the host enqueues more sharded levels.
template <typename T>
__global__ void dist_gather_kernel(const T* __restrict__ in, const LevelCtl* __restrict__ ctl,
                                   LevelCtl* __restrict__ ctl_tail, SelectResult* __restrict__ res,
                                   const u64* __restrict__ sizes, int P, int rank, u64 G, T* __restrict__ gsend,
                                   int level) {
    typedef typename Bits<T>::type RawT;
    pdl_wait();
    pdl_trigger();
    if (res->done) return;
    u64 N = 0, off = 0;
    for (int q = 0; q < P; ++q) {
        if (q < rank) off += sizes[q];
        N += sizes[q];
    }
    if (N > G) {
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            res->dist_halt = 1;
            res->done = 1;
        }
        return;
    }
    const u64 n = ctl->n;
    const RawT* src = reinterpret_cast<const RawT*>(in);
    RawT* dst = reinterpret_cast<RawT*>(gsend);
    for (u64 i = blockIdx.x * (u64)blockDim.x + threadIdx.x; i < G; i += (u64)gridDim.x * blockDim.x)
        dst[i] = (i >= off && i < off + n) ? src[i - off] : (RawT)0;
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        ctl_tail->n = N;
        ctl_tail->k = ctl->k;
        if (level < 32) res->n_level[level] = (long long)N;
    }
}

}  // namespace ss
