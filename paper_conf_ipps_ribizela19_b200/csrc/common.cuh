// common.cuh -- device-side building blocks of the B200 SampleSelect path.
//
// Order-preserving keys (reading R3): every value is
// mapped to an unsigned integer whose numeric order is IEEE totalOrder (floats)
// or numeric order (ints).  All comparisons in the path (Fig. 4 L335 walk,
// sample sort, base case) are integer compares on these keys, so -0/+0 and
// NaNs are ordered bit-exactly; the key successor (+1) is the "s_e + eps" of
// §IV.C L350-354.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace ss {

typedef unsigned long long u64;
typedef unsigned int u32;

// ---------------------------------------------------------------- keys ----
template <typename T> struct Traits;
template <> struct Traits<float> {
    typedef u32 Key;
    static __host__ __device__ __forceinline__ Key to_key(u32 u) {
        return u ^ ((u32)((int)u >> 31) | 0x80000000u);
    }
    static __host__ __device__ __forceinline__ u32 from_key(Key k) {
        return (k & 0x80000000u) ? (k ^ 0x80000000u) : ~k;
    }
};
template <> struct Traits<double> {
    typedef u64 Key;
    static __host__ __device__ __forceinline__ Key to_key(u64 u) {
        return u ^ ((u64)((long long)u >> 63) | 0x8000000000000000ull);
    }
    static __host__ __device__ __forceinline__ u64 from_key(Key k) {
        return (k & 0x8000000000000000ull) ? (k ^ 0x8000000000000000ull) : ~k;
    }
};
template <> struct Traits<int> {
    typedef u32 Key;
    static __host__ __device__ __forceinline__ Key to_key(u32 u) { return u ^ 0x80000000u; }
    static __host__ __device__ __forceinline__ u32 from_key(Key k) { return k ^ 0x80000000u; }
};
template <> struct Traits<long long> {
    typedef u64 Key;
    static __host__ __device__ __forceinline__ Key to_key(u64 u) { return u ^ 0x8000000000000000ull; }
    static __host__ __device__ __forceinline__ u64 from_key(Key k) { return k ^ 0x8000000000000000ull; }
};

// Raw bits type of T (same width as the key).
template <typename T> struct Bits { typedef typename Traits<T>::Key type; };

template <typename T>
__device__ __forceinline__ typename Traits<T>::Key load_key(const T* p) {
    typedef typename Traits<T>::Key K;
    K raw = __ldg(reinterpret_cast<const K*>(p));
    return Traits<T>::to_key(raw);
}

// --------------------------------------------------------- level state ----
// Device-resident control block, one per recursion level (§IV.E:
// control stays on the GPU; the paper used CDP, we pre-enqueue early-exiting
// kernels).  Zeroed by the init kernel at the start of each call.
struct LevelCtl {
    u64 n;          // n_l: elements entering level l
    u64 k;          // k_l: rank within level l
    u32 ticket;     // count-kernel CTA completion ticket (last CTA runs the tail)
    u32 bucket;     // bucket j chosen at level l
    u32 ncta;       // active CTAs of the count/filter grid
    u32 marker;     // whole buckets inside the cell LUT's marker cells (tree_image_kernel)
    // fused speculative filter (window_kernel): spec is set when
    // the level streams once against the sample-predicted key window
    // [klo, klo + kspan), copying it to the next level's buffer (cap counts
    // it); hit = rank k fell inside the window
    u32 spec;
    u32 hit;
    u64 cap;
    u64 klo, kspan; // the window as a key range: klo <= key < klo + kspan (mod 2^bits)
    u64 below;      // elements with key < klo (count kernel CTAs add theirs)
    u64 wtot;       // elements inside the window (cap also counts the chunk padding)
    u32 nospec;     // set by a miss: this level re-runs the paper's filter on the same data
    u32 spec_eq;    // the window is one equality bucket (§IV.C): a hit returns its value
    u32 pre;        // this level's sample keys were gathered ahead (init / previous level's tail)
    u32 pad2_;
    // sharded driver (sharded.cuh): n above is this rank's share
    // of the level, gn the level's size over all ranks (0 = one GPU)
    u64 gn;
    u32 pass;       // the level is a pass-through (the global level is already small)
    u32 directed;   // the window is [klo, klo + kspan) from the previous level's miss, not the sample
    float dfrac;    // directed window: expected fraction of the level inside it
    u32 pad3_;
    const void* src;// level 0: the call's input (written by the init kernel, whose argument is patched
                    // per call in a cached CUDA graph); NULL on deeper levels
    void* up_out;   // level 0 of a top-k call (§IV.I): the caller's output of the n - k largest
                    // elements (written by the init kernel, patched like src); NULL otherwise
    u64 ucnt;       // top-k: elements written to up_out so far (the keys above the answer)
    u64 hlo, hspan; // fused level whose window runs to the top / bottom of the key range: its
                    // histogram bins [hlo, hlo + hspan) (the sample's keys), the first bin also
                    // taking the window's keys below hlo, the last those above; hspan 0 = the window
};

struct SelectResult {
    u64 bits;                 // answer (raw bits of T)
    long long rank;           // approximate: exact rank #{x < answer}
    int done;                 // 1 once bits is valid
    int levels;               // count passes executed
    int eq_exit;              // answer from an equality bucket (§IV.C)
    int incomplete;           // final K1 saw n_l > B: host must enqueue more levels
    long long n_level[32];
    int bucket[32];
    long long split_index;    // approximate: 1-based splitter index returned
    unsigned int lut_stats[2];// level 0: CTAs that used the cell LUT, marker-cell buckets
    unsigned int fused_levels;// bit l: level l's survivors came from the fused filter (window hit)
    unsigned int spec_levels; // bit l: level l ran the fused filter (hit or miss)
    unsigned int spec_err;    // captured count != window total (internal consistency check)
    int dist_halt;            // sharded: 1 = survivors exceed the gather buffer (host adds levels), 2 = k >= N
    unsigned int seq;         // host mirror only: publish sequence number, written last
    int halt;                 // level + 1 of a fused level whose window missed rank k (or could not
                              // shrink the level): the chain stopped (done), the host re-runs it
    unsigned long long dist_n;// sharded: the size of the union of the shards (the host plans the next call with it)
    unsigned long long upper_cnt;// top-k call: #{x > answer} written to the output by the fused path
    int tl_on;                // timeline mode (profile = 3): kernels stamp tl[]
    int pad_;
    u64 t_init;               // %globaltimer at the init kernel (timeline origin)
    // timeline: per (level, kernel) slot, [0] = ~(earliest CTA start after
    // pdl_wait) and [1] = latest CTA exit, %globaltimer ns (atomicMax both)
    u64 tl[32 * 3][2];
};

__device__ __forceinline__ u64 gtimer() {
    u64 t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

// Scope guard stamping a kernel's device-side interval into the timeline
// (one atomic per CTA on entry and exit; inert unless res->tl_on).
struct TimelineScope {
    u64* slot;
    __device__ __forceinline__ TimelineScope(SelectResult* r, int level, int kernel) : slot(nullptr) {
        if (r && level < 32 && r->tl_on) {
            slot = r->tl[level * 3 + kernel];
            if (threadIdx.x == 0) atomicMax(reinterpret_cast<unsigned long long*>(slot), ~gtimer());
        }
    }
    __device__ __forceinline__ ~TimelineScope() {
        if (slot && threadIdx.x == 0) atomicMax(reinterpret_cast<unsigned long long*>(slot + 1), gtimer());
    }
};

// Phase stamp of a kernel (profile = 3 diagnostics, compiled in only with
// -DSS_PHASE_STAMPS=1: a stamp costs the stamping warp a global round trip):
// slot [0] = ~earliest, [1] = latest %globaltimer over the CTAs that pass it
// (slots 80.. are free: levels >= 27 never run).
#ifndef SS_PHASE_STAMPS
#define SS_PHASE_STAMPS 0
#endif
__device__ __forceinline__ void tl_phase(SelectResult* r, int slot) {
    if (SS_PHASE_STAMPS && r && r->tl_on && threadIdx.x == 0) {
        const u64 t = gtimer();
        atomicMax(reinterpret_cast<unsigned long long*>(r->tl[slot]), ~t);
        atomicMax(reinterpret_cast<unsigned long long*>(r->tl[slot] + 1), t);
    }
}

// ------------------------------------------------------------ chunking ----
// Element -> CTA mapping shared by the count (K2) and filter (K5) kernels;
// the filter must see exactly the count's partition so that the K3 offsets
// apply (§IV.G).  The body is cut into 16-element groups (16 oracle
// bytes = one 128-bit load); CTA g owns the contiguous groups
// [g*gpc, (g+1)*gpc).  Elements [0, head) are peeled so the body starts
// 16-byte aligned (CTA 0 owns them); [tail_begin, n) (< 16 elements) belongs
// to the last active CTA.  Inside its chunk K2 gives each warp a contiguous
// run of groups (any order counts the same); K5 walks the chunk in slices so
// that its output is in input order (reading R15).
constexpr u64 MIN_GROUPS_PER_CTA = 32;  // 512 elements: small levels still spread over many CTAs

struct Chunking {
    u64 head, ngroups, tail_begin, gpc;
    u32 ncta;
};

template <typename T>
__host__ __device__ __forceinline__ Chunking make_chunking(const T* p, u64 n, u32 grid) {
    Chunking c;
    u64 mis = (u64)((uintptr_t)p & 15u);
    u64 head = mis ? (16 - mis) / sizeof(T) : 0;
    if (head > n) head = n;
    c.head = head;
    c.ngroups = (n - head) / 16;
    c.tail_begin = head + c.ngroups * 16;
    u64 gpc = (c.ngroups + grid - 1) / grid;
    if (gpc < MIN_GROUPS_PER_CTA) gpc = MIN_GROUPS_PER_CTA;
    c.gpc = gpc;
    u64 nc = (c.ngroups + gpc - 1) / gpc;
    if (nc == 0) nc = 1;
    if (nc > grid) nc = grid;
    c.ncta = (u32)nc;
    return c;
}

// Oracle byte of element i lives at oracle_base + i, with the base shifted so
// that the body's bytes start 16-byte aligned.
__host__ __device__ __forceinline__ u64 oracle_pad(u64 head) { return (16 - (head & 15)) & 15; }

// ------------------------------------------------------------ sampling ----
// Reading R7: SplitMix64 finaliser (Steele/Lea/Flood 2014), counter based.
__host__ __device__ __forceinline__ u64 splitmix64(u64 x) {
    u64 z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
__host__ __device__ __forceinline__ u64 level_base(u64 seed, int level) {
    return splitmix64(seed + (u64)level * 0xD1B54A32D192ED03ull);
}
__device__ __forceinline__ u64 sample_index(u64 base, u64 slot, u64 n) {
    return __umul64hi(splitmix64(base + slot), n);
}

}  // namespace ss
