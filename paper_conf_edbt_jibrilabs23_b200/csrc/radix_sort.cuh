// radix_sort.cuh - stable LSD radix sort of (uint64 key, uint32 value) pairs for
// sm_100a, onesweep style (one kernel per 8-bit digit pass, 3072-key tiles):
//   1. one histogram kernel counts the digits of every pass in a single read;
//   2. a tiny kernel turns them into per-pass digit bases;
//   3. per pass, each 3072-key tile ranks its keys stably with warp match_any,
//      publishes per-digit counts and resolves its global digit offsets with a
//      per-digit decoupled look-back (256 threads, one digit each, 8 predecessor
//      tiles per step), stages the
//      keys digit-sorted in shared memory and writes them out in contiguous runs.
// Only the significant key bits are sorted (2*ceil(log2 V') for packed
// (src', dst') edge keys).
#pragma once
#include "dev_common.cuh"

namespace h2tap {

#ifndef H2TAP_RS_ITEMS
#define H2TAP_RS_ITEMS 12
#endif
#ifndef H2TAP_RS_LOOK
#define H2TAP_RS_LOOK 8
#endif
#ifndef H2TAP_RS_BALLOT
#define H2TAP_RS_BALLOT 0
#endif
constexpr int kRsThreads = 256;
constexpr int kRsItems = H2TAP_RS_ITEMS;
constexpr int kRsTile = kRsThreads * kRsItems;  // 3072 keys per tile
constexpr int kRsSmem = kRsTile * 12;           // dynamic smem: staged keys + values
constexpr int kRsWarps = kRsThreads / 32;
constexpr int kRsMaxPasses = 8;
constexpr int kRsLook = H2TAP_RS_LOOK;  // look-back: predecessor tiles read per step
#ifndef H2TAP_RS_DIRECT
#define H2TAP_RS_DIRECT 128
#endif
constexpr uint32_t kRsDirectTiles = H2TAP_RS_DIRECT;  // rs_coop: tiles up to which every CTA sums the count columns itself

// n_dev (nullable): the key count lives in device memory (no host sync before the
// sort); `n` is then an upper bound that only sizes the grids
__device__ __forceinline__ uint64_t rs_count(uint64_t n, const unsigned long long* n_dev) {
    return n_dev ? min(n, (uint64_t)*n_dev) : n;
}

__global__ void __launch_bounds__(256) rs_histogram(const uint64_t* __restrict__ keys, uint64_t n,
                                                    const unsigned long long* __restrict__ n_dev,
                                                    int passes, uint32_t* __restrict__ hist) {
    __shared__ uint32_t s[kRsMaxPasses][256];
    n = rs_count(n, n_dev);
    for (int i = threadIdx.x; i < kRsMaxPasses * 256; i += blockDim.x) (&s[0][0])[i] = 0;
    __syncthreads();
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t k = keys[i];
        for (int p = 0; p < passes; ++p) atomicAdd(&s[p][(k >> (8 * p)) & 255], 1u);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < passes * 256; i += blockDim.x) {
        uint32_t v = (&s[0][0])[i];
        if (v) atomicAdd(&hist[i], v);
    }
}

// one block per pass: exclusive scan of the 256 digit counts; skip[p] = 1 when every key
// has the same digit in pass p (the pass is the identity permutation: a plain copy)
__global__ void __launch_bounds__(256) rs_digit_base(const uint32_t* __restrict__ hist,
                                                     uint64_t* __restrict__ base, uint64_t n,
                                                     const unsigned long long* __restrict__ n_dev,
                                                     uint32_t* __restrict__ skip) {
    __shared__ uint64_t sm[9];
    const int p = blockIdx.x;
    n = rs_count(n, n_dev);
    uint64_t v = hist[p * 256 + threadIdx.x], tot;
    uint64_t e = block_exclusive_scan<256>(v, sm, &tot);
    base[p * 256 + threadIdx.x] = e;
    if (threadIdx.x == 0) skip[p] = 0;
    __syncthreads();
    if (v == n) skip[p] = 1;
}

__global__ void __launch_bounds__(kRsThreads) rs_onesweep(
    const uint64_t* __restrict__ kin, const uint32_t* __restrict__ vin, uint64_t* __restrict__ kout,
    uint32_t* __restrict__ vout, uint64_t n, const unsigned long long* __restrict__ n_dev, int shift,
    const uint64_t* __restrict__ digit_base, uint64_t* __restrict__ status /* [ntiles][256] */,
    uint32_t* __restrict__ tile_ctr, const uint32_t* __restrict__ skip) {
    __shared__ uint32_t s_tile;
    __shared__ uint32_t s_wcnt[kRsWarps][256];
    __shared__ uint32_t s_dstart[256];
    __shared__ uint64_t s_gpre[256];
    extern __shared__ __align__(16) uint8_t rs_dsm[];  // kRsSmem bytes
    uint64_t* s_keys = reinterpret_cast<uint64_t*>(rs_dsm);
    uint32_t* s_vals = reinterpret_cast<uint32_t*>(rs_dsm + kRsTile * 8);
    __shared__ uint32_t s_scan[kRsThreads / 32 + 1];

    const int tid = threadIdx.x, w = tid >> 5, l = lane_id();
    n = rs_count(n, n_dev);
    if (*skip) {  // constant digit: stable order unchanged, copy this CTA's tile
        for (uint64_t i = (uint64_t)blockIdx.x * kRsTile + tid; i < min(n, (uint64_t)(blockIdx.x + 1) * kRsTile);
             i += kRsThreads) {
            kout[i] = kin[i];
            vout[i] = vin[i];
        }
        return;
    }
    if (tid == 0) s_tile = atomicAdd(tile_ctr, 1u);
    for (int i = tid; i < kRsWarps * 256; i += kRsThreads) (&s_wcnt[0][0])[i] = 0;
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t base = (uint64_t)tile * kRsTile;
    if (base >= n) return;  // grid sized by an upper bound: no later tile depends on this one
    const uint64_t tile_n = (n - base < (uint64_t)kRsTile) ? (n - base) : (uint64_t)kRsTile;

    uint64_t k[kRsItems];
    uint32_t v[kRsItems];
    uint32_t rank[kRsItems];
#pragma unroll
    for (int i = 0; i < kRsItems; ++i) {
        uint64_t idx = base + (uint64_t)w * 32 * kRsItems + i * 32 + l;
        bool ok = idx < n;
        k[i] = ok ? kin[idx] : 0;
        v[i] = ok ? vin[idx] : 0;
    }
    // stable in-warp ranking, iteration-major then lane order == tile index order
#pragma unroll
    for (int i = 0; i < kRsItems; ++i) {
        uint64_t idx = base + (uint64_t)w * 32 * kRsItems + i * 32 + l;
        bool ok = idx < n;
        uint32_t valid = __ballot_sync(0xffffffffu, ok);
        rank[i] = 0;
        if (ok) {
            uint32_t d = (uint32_t)(k[i] >> shift) & 255u;
#if H2TAP_RS_BALLOT
            // peers with the same digit from 8 ballots (no MATCH instruction)
            uint32_t peers = valid;
#pragma unroll
            for (int b = 0; b < 8; ++b) {
                const uint32_t m = __ballot_sync(valid, (d >> b) & 1u);
                peers &= ((d >> b) & 1u) ? m : ~m;
            }
#else
            uint32_t peers = __match_any_sync(valid, d);
#endif
            uint32_t before = s_wcnt[w][d];
            __syncwarp(valid);
            if (l == (uint32_t)(__ffs(peers) - 1)) s_wcnt[w][d] = before + __popc(peers);
            __syncwarp(valid);
            rank[i] = before + __popc(peers & lanemask_lt());
        }
    }
    __syncthreads();
    // per digit: exclusive over warps, tile count
    uint32_t c = 0;
    if (tid < 256) {
        const int d = tid;  // threads 0..255 own one digit each
        for (int ww = 0; ww < kRsWarps; ++ww) {
            uint32_t t = s_wcnt[ww][d];
            s_wcnt[ww][d] = c;
            c += t;
        }
    }
    uint32_t tot;
    uint32_t ds = block_exclusive_scan<kRsThreads>(c, s_scan, &tot);
    if (tid < 256) s_dstart[tid] = ds;
    // per-digit decoupled look-back: thread d walks back over the tiles for digit d,
    // kRsLook predecessors per step (independent loads, one L2 round trip per step)
    if (tid < 256) {
        const int d = tid;
        uint64_t* st = status + (uint64_t)tile * 256 + d;
        uint64_t excl = 0;
        if (tile == 0) {
            st_volatile(st, kFlagPrefix | c);
        } else {
            st_volatile(st, kFlagAgg | c);
            int64_t t = (int64_t)tile - 1;
            while (t >= 0) {
                uint64_t s[kRsLook];
#pragma unroll
                for (int q = 0; q < kRsLook; ++q)
                    s[q] = (t - q >= 0) ? ld_volatile(status + (uint64_t)(t - q) * 256 + d) : kFlagPrefix;
                // consume the ready run up to (and including) the nearest prefix
                int q = 0;
                bool done = false;
#pragma unroll
                for (int j = 0; j < kRsLook; ++j) {
                    if (done || q != j) continue;
                    const uint64_t f = s[j] >> 62;
                    if (f == 0) continue;  // not published yet: re-poll from here
                    excl += s[j] & kValMask;
                    ++q;
                    if (f == 2) done = true;
                }
                if (done) break;
                if (q == 0) __nanosleep(kLookBackoffNs);  // nearest predecessor not published yet
                t -= q;
            }
            st_volatile(st, kFlagPrefix | (excl + c));
        }
        s_gpre[d] = digit_base[d] + excl;
    }
    __syncthreads();
#pragma unroll
    for (int i = 0; i < kRsItems; ++i) {
        uint64_t idx = base + (uint64_t)w * 32 * kRsItems + i * 32 + l;
        if (idx < n) {
            uint32_t d = (uint32_t)(k[i] >> shift) & 255u;
            uint32_t pos = s_dstart[d] + s_wcnt[w][d] + rank[i];
            s_keys[pos] = k[i];
            s_vals[pos] = v[i];
        }
    }
    __syncthreads();
    for (uint32_t p = tid; p < tile_n; p += kRsThreads) {
        uint64_t key = s_keys[p];
        uint32_t d = (uint32_t)(key >> shift) & 255u;
        uint64_t o = s_gpre[d] + (p - s_dstart[d]);
        kout[o] = key;
        vout[o] = s_vals[p];
    }
}

// ------------------------------------------------------------ cooperative ----
// All passes in ONE launch for key counts whose tiles are co-resident (launched with
// cudaLaunchCooperativeKernel, one tile per CTA).  A pass: every CTA ranks its tile
// (warp match_any, stable) and publishes its 256 digit counts; grid barrier; the CTAs
// scan the count matrix column-wise (digit d by CTA d mod grid: exclusive over tiles,
// plus the digit total); grid barrier; every CTA turns the 256 totals into digit bases
// (block scan), adds its tile's column prefix and scatters through shared memory in
// contiguous runs; grid barrier before the next pass reads the output.  This replaces
// the per-digit decoupled look-back of rs_onesweep, whose chain of 8-tile steps is the
// critical path when every tile publishes at the same moment (all tiles resident), by
// two barriers and a parallel scan, and the per-pass launches by one.
__device__ __forceinline__ void rs_grid_sync(unsigned int* bar, unsigned int& target) {
    __syncthreads();
    if (threadIdx.x == 0) {
        target += gridDim.x;
        __threadfence();
        atomicAdd(bar, 1u);
        while (*reinterpret_cast<volatile unsigned int*>(bar) < target) __nanosleep(32);
        __threadfence();
    }
    __syncthreads();
}

template <int ITEMS>
__global__ void __launch_bounds__(kRsThreads, ITEMS >= 12 ? 3 : 4) rs_coop(
    uint64_t* __restrict__ k0, uint32_t* __restrict__ v0, uint64_t* __restrict__ k1, uint32_t* __restrict__ v1,
    uint64_t n, const unsigned long long* __restrict__ n_dev, int passes,
    uint32_t* __restrict__ cnt /* [grid][256] */, uint32_t* __restrict__ tot /* [256] */, unsigned int* __restrict__ bar) {
    constexpr int TILE = kRsThreads * ITEMS;
    __shared__ uint32_t s_wcnt[kRsWarps][256];
    __shared__ uint32_t s_dstart[256];
    __shared__ uint32_t s_gpre[256];
    __shared__ uint32_t s_scan[kRsThreads / 32 + 1];
    extern __shared__ __align__(16) uint8_t rs_dsm[];  // TILE * 12 bytes
    uint64_t* s_keys = reinterpret_cast<uint64_t*>(rs_dsm);
    uint32_t* s_vals = reinterpret_cast<uint32_t*>(rs_dsm + TILE * 8);
    const int tid = threadIdx.x, w = tid >> 5, l = lane_id();
    const uint32_t T = gridDim.x, b = blockIdx.x;
    n = rs_count(n, n_dev);
    const uint64_t base = (uint64_t)b * TILE;
    const uint32_t tile_n = base >= n ? 0u : (uint32_t)(n - base < (uint64_t)TILE ? n - base : (uint64_t)TILE);
    unsigned int target = 0;
    for (int p = 0; p < passes; ++p) {
        const int shift = 8 * p;
        const uint64_t* kin = (p & 1) ? k1 : k0;
        const uint32_t* vin = (p & 1) ? v1 : v0;
        uint64_t* kout = (p & 1) ? k0 : k1;
        uint32_t* vout = (p & 1) ? v0 : v1;
        for (int i = tid; i < kRsWarps * 256; i += kRsThreads) (&s_wcnt[0][0])[i] = 0;
        __syncthreads();
        uint64_t k[ITEMS];
        uint32_t v[ITEMS], rank[ITEMS];
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) {
            const uint32_t j = (uint32_t)w * 32 * ITEMS + i * 32 + l;
            const bool ok = j < tile_n;
            k[i] = ok ? kin[base + j] : 0;
            v[i] = ok ? vin[base + j] : 0;
        }
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) {
            const uint32_t j = (uint32_t)w * 32 * ITEMS + i * 32 + l;
            const bool ok = j < tile_n;
            const uint32_t valid = __ballot_sync(0xffffffffu, ok);
            rank[i] = 0;
            if (ok) {
                const uint32_t d = (uint32_t)(k[i] >> shift) & 255u;
                const uint32_t peers = __match_any_sync(valid, d);
                const uint32_t before = s_wcnt[w][d];
                __syncwarp(valid);
                if (l == (uint32_t)(__ffs(peers) - 1)) s_wcnt[w][d] = before + __popc(peers);
                __syncwarp(valid);
                rank[i] = before + __popc(peers & lanemask_lt());
            }
        }
        __syncthreads();
        uint32_t c = 0;
        {   // thread d: exclusive over warps for digit d, tile count of d
            const int d = tid;
            for (int ww = 0; ww < kRsWarps; ++ww) {
                const uint32_t t = s_wcnt[ww][d];
                s_wcnt[ww][d] = c;
                c += t;
            }
        }
        uint32_t tt;
        const uint32_t ds = block_exclusive_scan<kRsThreads>(c, s_scan, &tt);
        s_dstart[tid] = ds;
        cnt[(uint64_t)b * 256 + tid] = c;
        rs_grid_sync(bar, target);
        if (T <= kRsDirectTiles) {
            // few tiles: thread d of every CTA sums column d itself (T coalesced 1 KB rows):
            // its tile's prefix and the digit total, no second barrier
            uint32_t pre = 0, all = 0;
            for (uint32_t t = 0; t < T; ++t) {
                const uint32_t x = cnt[(uint64_t)t * 256 + tid];
                pre += t < b ? x : 0u;
                all += x;
            }
            uint32_t sum;
            const uint32_t db = block_exclusive_scan<kRsThreads>(all, s_scan, &sum);
            s_gpre[tid] = db + pre;
        } else {
            // column scans: digit d by CTA d mod T (exclusive over tiles, in place), total -> tot[d]
            for (uint32_t d = b; d < 256; d += T) {
                uint32_t carry = 0;
                for (uint32_t t0 = 0; t0 < T; t0 += kRsThreads) {
                    const uint32_t t = t0 + tid;
                    const uint32_t x = t < T ? cnt[(uint64_t)t * 256 + d] : 0u;
                    uint32_t sum;
                    const uint32_t e = block_exclusive_scan<kRsThreads>(x, s_scan, &sum);
                    if (t < T) cnt[(uint64_t)t * 256 + d] = carry + e;
                    carry += sum;
                }
                if (tid == 0) tot[d] = carry;
            }
            rs_grid_sync(bar, target);
            uint32_t sum;
            const uint32_t db = block_exclusive_scan<kRsThreads>(tot[tid], s_scan, &sum);
            s_gpre[tid] = db + cnt[(uint64_t)b * 256 + tid];
        }
        __syncthreads();
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) {
            const uint32_t j = (uint32_t)w * 32 * ITEMS + i * 32 + l;
            if (j < tile_n) {
                const uint32_t d = (uint32_t)(k[i] >> shift) & 255u;
                const uint32_t pos = s_dstart[d] + s_wcnt[w][d] + rank[i];
                s_keys[pos] = k[i];
                s_vals[pos] = v[i];
            }
        }
        __syncthreads();
        for (uint32_t q = tid; q < tile_n; q += kRsThreads) {
            const uint64_t key = s_keys[q];
            const uint32_t d = (uint32_t)(key >> shift) & 255u;
            const uint32_t o = s_gpre[d] + (q - s_dstart[d]);
            kout[o] = key;
            vout[o] = s_vals[q];
        }
        if (p + 1 < passes) rs_grid_sync(bar, target);
    }
}

}  // namespace h2tap
