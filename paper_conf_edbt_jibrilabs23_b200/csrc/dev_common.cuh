// dev_common.cuh - device building blocks shared by the h2tap kernels (sm_100a).
//
//  * block-wide exclusive scans over per-thread item counts (warp shuffles + smem)
//  * decoupled look-back (Merrill & Garland single-pass scan): each tile publishes
//    its aggregate, then one warp inspects 128 predecessors at a time until it
//    meets an inclusive prefix.  Status word: 2-bit flag | 62-bit value.
//    Tiles take their index from an atomic counter, so every predecessor of a
//    spinning tile has already been scheduled (forward progress).
//  * lower_bound searches over sorted device arrays.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace h2tap {

constexpr int kWarp = 32;
constexpr uint64_t kFlagAgg = 1ull << 62;
constexpr uint64_t kFlagPrefix = 2ull << 62;
constexpr uint64_t kValMask = (1ull << 62) - 1;
constexpr uint32_t kNone32 = 0xFFFFFFFFu;

__device__ __forceinline__ uint64_t sm64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

template <typename T>
__device__ __forceinline__ T warp_inclusive_scan(T v) {
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T n = __shfl_up_sync(0xffffffffu, v, o);
        if ((int)lane_id() >= o) v += n;
    }
    return v;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// Block-wide exclusive scan of one value per thread.  smem: >= NT/32 + 1 slots.
// Returns the exclusive prefix; *total gets the block total (all threads).
template <int NT, typename T>
__device__ __forceinline__ T block_exclusive_scan(T v, T* smem, T* total) {
    const int w = threadIdx.x >> 5;
    T inc = warp_inclusive_scan(v);
    if (lane_id() == 31) smem[w] = inc;
    __syncthreads();
    if (w == 0) {
        T s = (lane_id() < NT / 32) ? smem[lane_id()] : T(0);
        T si = warp_inclusive_scan(s);
        if (lane_id() < NT / 32) smem[lane_id()] = si - s;
        if (lane_id() == NT / 32 - 1) smem[NT / 32] = si;
    }
    __syncthreads();
    T r = smem[w] + inc - v;
    *total = smem[NT / 32];
    __syncthreads();
    return r;
}

// ---------------------------------------------------------------- look-back
__device__ __forceinline__ uint64_t ld_volatile(const uint64_t* p) {
    return *reinterpret_cast<const volatile uint64_t*>(p);
}
__device__ __forceinline__ void st_volatile(uint64_t* p, uint64_t v) {
    *reinterpret_cast<volatile uint64_t*>(p) = v;
}

// Called by ONE full warp of the tile.  Publishes `aggregate` for `tile`, looks
// back over predecessors, publishes the inclusive prefix, returns the exclusive
// prefix (identical in all lanes).  Each step reads 32 * kLookQ predecessors
// (kLookQ per lane, nearest first).  Measured on B200 (round 2): 4 or 8 per lane made
// the 1M-item select / classify kernels slower (more L2 traffic while spinning on
// predecessors that have not published yet), so the default stays at 1.
#ifndef H2TAP_LOOKQ
#define H2TAP_LOOKQ 1
#endif
constexpr int kLookQ = H2TAP_LOOKQ;
#ifndef H2TAP_LOOK_BACKOFF
#define H2TAP_LOOK_BACKOFF 32
#endif
constexpr unsigned kLookBackoffNs = H2TAP_LOOK_BACKOFF;  // look-back re-poll delay (ns)
__device__ __forceinline__ uint64_t lookback_warp(uint64_t* status, uint32_t tile, uint64_t aggregate) {
    if (tile == 0) {
        if (lane_id() == 0) st_volatile(&status[0], kFlagPrefix | aggregate);
        return 0;
    }
    if (lane_id() == 0) st_volatile(&status[tile], kFlagAgg | aggregate);
    uint64_t excl = 0;
    int64_t t = (int64_t)tile - 1;
    while (true) {
        uint64_t s[kLookQ];
        bool not_ready = false;
#pragma unroll
        for (int q = 0; q < kLookQ; ++q) {
            const int64_t idx = t - (int64_t)(lane_id() * kLookQ + q);   // lane 0, q 0 = nearest
            s[q] = (idx >= 0) ? ld_volatile(&status[idx]) : kFlagPrefix;  // virtual prefix 0 before tile 0
            not_ready |= (s[q] >> 62) == 0;
        }
        if (__any_sync(0xffffffffu, not_ready)) {  // spin until all are visible (predecessors are scheduled),
            __nanosleep(kLookBackoffNs);             // backing off so the polls leave L2 bandwidth to them
            continue;
        }
        int fq = kLookQ;  // this lane's nearest prefix
#pragma unroll
        for (int q = kLookQ - 1; q >= 0; --q)
            if ((s[q] >> 62) == 2) fq = q;
        const uint32_t has = __ballot_sync(0xffffffffu, fq < kLookQ);
        const int first = has ? (__ffs(has) - 1) : 32;  // lane holding the nearest prefix
        uint64_t v = 0;
#pragma unroll
        for (int q = 0; q < kLookQ; ++q)
            if ((int)lane_id() < first || ((int)lane_id() == first && q <= fq)) v += s[q] & kValMask;
        excl += warp_sum(v);
        if (has) break;
        t -= 32 * kLookQ;
    }
    if (lane_id() == 0) st_volatile(&status[tile], kFlagPrefix | (excl + aggregate));
    return excl;
}

// ------------------------------------------------------------------ search
// first index i in [lo, hi) with a[i] >= key (returns hi if none)
template <typename T, typename K>
__device__ __forceinline__ uint64_t lower_bound_dev(const T* a, uint64_t lo, uint64_t hi, K key) {
    while (lo < hi) {
        uint64_t mid = lo + ((hi - lo) >> 1);
        if (a[mid] < key) lo = mid + 1; else hi = mid;
    }
    return lo;
}
// first index i in [lo, hi) with a[i] > key
template <typename T, typename K>
__device__ __forceinline__ uint64_t upper_bound_dev(const T* a, uint64_t lo, uint64_t hi, K key) {
    while (lo < hi) {
        uint64_t mid = lo + ((hi - lo) >> 1);
        if (!(key < a[mid])) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// lower_bound over a sorted u64 array: a few interpolation steps between the
// known key bounds (external IDs are near-arithmetic runs), then bisection
__device__ __forceinline__ uint64_t interp_lower_bound(const uint64_t* a, uint64_t lo, uint64_t hi, uint64_t key) {
    if (lo >= hi) return lo;
    uint64_t vlo = a[lo], vhi = a[hi - 1];
    if (key <= vlo) return lo;
    if (key > vhi) return hi;
    // invariant: a[lo] < key <= a[hi-1] (so lo < hi - 1 here)
    for (int step = 0; step < 6 && hi - lo > 16; ++step) {
        const double f = (double)(key - vlo) / (double)(vhi - vlo);
        uint64_t mid = lo + 1 + (uint64_t)(f * (double)(hi - lo - 2));
        if (mid >= hi - 1) mid = hi - 2;
        const uint64_t v = a[mid];
        if (v < key) { lo = mid; vlo = v; } else { hi = mid + 1; vhi = v; }
    }
    return lower_bound_dev(a, lo + 1, hi, key);
}

// Stable compaction of a tile of kThreads x ITEMS items in STRIPED order (item k of
// thread t is tile item k*NT + t, so global loads coalesce): flag[k] -> pos[k] =
// rank of the item among flagged items of the tile.  smem: ITEMS*NT/32 + 1 words.
// Returns the tile total.  Requires ITEMS * NT/32 <= 64.
template <int NT, int ITEMS>
__device__ __forceinline__ uint32_t striped_compact(const bool (&flag)[ITEMS], uint32_t (&pos)[ITEMS], uint32_t* s) {
    constexpr int NW = NT / 32;
    static_assert(ITEMS * NW <= 64, "striped_compact: too many (item, warp) cells");
    const int w = threadIdx.x >> 5;
    const uint32_t lane = lane_id(), lt = lanemask_lt();
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
        uint32_t m = __ballot_sync(0xffffffffu, flag[k]);
        pos[k] = __popc(m & lt);
        if (lane == 0) s[k * NW + w] = __popc(m);
    }
    __syncthreads();
    if (w == 0) {
        constexpr int C = ITEMS * NW;
        uint32_t a = (2 * lane < C) ? s[2 * lane] : 0, b = (2 * lane + 1 < C) ? s[2 * lane + 1] : 0;
        uint32_t inc = warp_inclusive_scan(a + b);
        uint32_t ex = inc - a - b;
        if (2 * lane < C) s[2 * lane] = ex;
        if (2 * lane + 1 < C) s[2 * lane + 1] = ex + a;
        if (lane == 31) s[C] = inc;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) pos[k] += s[k * NW + w];
    uint32_t tot = s[ITEMS * NW];
    __syncthreads();
    return tot;
}

// (ts, seq) commit point, lexicographic (reading A5)
struct Point {
    uint64_t ts, seq;
};
__device__ __forceinline__ bool pt_less(uint64_t ts_a, uint64_t seq_a, uint64_t ts_b, uint64_t seq_b) {
    return ts_a < ts_b || (ts_a == ts_b && seq_a < seq_b);
}

}  // namespace h2tap
