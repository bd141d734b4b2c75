// kernels.cuh - the propagation kernels.
//
// Notation follows the paper: a batch of deltas (ops) with commit timestamps is
// scanned (§5.2), checked for visibility against the propagation snapshot
// (§5.3), combined per (source, destination) key (§5.2 "combines such deltas
// into a single delta") and merged into the old CSR (§5.4, Algorithm 2 and
// merge()).  The B200 design replaces the per-node sequential merge with one
// global merge path over (kept old elements) x (inserted records).
#pragma once
#include "dev_common.cuh"

namespace h2tap {

constexpr int kThreads = 256;
constexpr int kItems = 8;
constexpr int kTile = kThreads * kItems;  // 2048 items per tile for select-style kernels

enum : uint8_t { NODE_INSERT = 0, NODE_DELETE = 1, EDGE_INSERT = 2, EDGE_DELETE = 3, EDGE_WEIGHT = 4 };
enum : uint64_t { ST_BAD_KIND = 1, ST_STALE = 2, ST_CREATE_ENDPOINT = 4, ST_NOT_OWNED = 8 };

// work ops: pending (older seq) ++ batch, SoA, in ascending seq order
struct Ops {
    const uint8_t* kind;
    const uint64_t* src;
    const uint64_t* dst;
    const float* w;
    const uint64_t* ts;
    const uint64_t* seq;
};

// device counters, zeroed at the start of every apply and read back at sync points
struct Counters {
    unsigned long long status;
    unsigned long long n_pend, n_node, n_edge;
    unsigned long long ts_min, ts_max, v_min, v_max;
    unsigned long long n_unique, n_dropped, n_inserted, n_hd;
    unsigned long long n_valid, n_gated;
    unsigned long long n_ins, n_del, n_upd;
    unsigned long long n_casc;
    unsigned long long row_lo_new, row_hi_new;  // sharded: the shard's row range in the new ID map
    unsigned long long Vn, Vr_new, En, new_identity;  // written by k_finish
    unsigned long long n_killed;  // vertices live before the cycle and dead after it (stats)
    unsigned long long first_pend;  // delta-store scan: first record left valid (k_rec_consume)
    unsigned long long idmap_lo;    // node mode: ids below it keep their id and external id
    unsigned long long idmap_keep;  // node mode: ID-map prefix the survivor pass did not rewrite
    unsigned int tiles[16];
};

__global__ void k_store_counters(const Counters* __restrict__ c, Counters* host_mapped) {
    constexpr int nw = sizeof(Counters) / 8;
    for (int i = threadIdx.x; i < nw; i += blockDim.x)
        reinterpret_cast<volatile unsigned long long*>(host_mapped)[i] = reinterpret_cast<const unsigned long long*>(c)[i];
}
__global__ void k_store_words(const unsigned long long* __restrict__ src, int n, unsigned long long* host_mapped) {
    for (int i = threadIdx.x; i < n; i += blockDim.x) reinterpret_cast<volatile unsigned long long*>(host_mapped)[i] = src[i];
}
__global__ void k_init_counters(Counters* c) {  // zero, with the two minima at their identity
    constexpr int nw = sizeof(Counters) / 8;
    static_assert(sizeof(Counters) % 8 == 0, "Counters is zeroed in 8-byte words");
    for (int i = threadIdx.x; i < nw; i += blockDim.x) reinterpret_cast<unsigned long long*>(c)[i] = 0;
    __syncwarp();
    if (threadIdx.x == 0) { c->ts_min = ~0ull; c->v_min = ~0ull; c->first_pend = ~0ull; }
}

// owned external-ID range of a shard: [lo, hi), hi == ~0 means "through UINT64_MAX"
struct OwnRange {
    uint64_t lo, hi;
    __device__ __forceinline__ bool owns(uint64_t x) const { return x >= lo && (hi == ~0ull || x < hi); }
};

// per unique vertex touched by visible node ops (a2)
struct NodeVtx {
    uint64_t tD_ts, tD_seq;  // latest NODE_DELETE point (valid if flags & NV_HASD)
    uint32_t start, end;     // segment in the (v, ts, seq)-sorted node-op list
    uint32_t oldpos;         // old dense index if old-present, else insertion rank
    uint32_t newid;          // new dense id if finally live
    uint32_t flags;
    uint32_t pad;
};
// NV_OLD: present in the old ID map; NV_LIVE0: live before the cycle (= NV_OLD unless
// the replica keeps tombstones, reading A23)
enum : uint32_t { NV_FINAL = 1, NV_HASD = 2, NV_OLD = 4, NV_LIVE0 = 8 };

// ID-map compaction (reading A9), evaluated on the fly: new dense id of old vertex k
// = k - (#dropped ids < k) + (#inserted ids placed at old positions <= k).
//   shift[k >> 16]: constant shift of a 64K-id block without dropped ids or insertion
//                   points strictly inside, else kRemapMixed
//   g32[k >> 5]  : {new id of the group's first id | exact << 31, dropped bitmask};
//                   exact groups (an insertion point strictly inside) add the insertion
//                   ranks.  Dense ids stay below 2^31 (checked on the host).
constexpr int kRemapBlockShift = 16;
constexpr int32_t kRemapMixed = INT32_MIN;
struct RemapView {
    const int32_t* shift;  // nullptr: identity
    const uint2* g32;
    const uint32_t* ins_oldpos;
    const unsigned long long* n_vins;  // device count of inserted vertices
    const int32_t* lohi;   // {lo, hi, shift, mlo, mhi, msh}: ids < lo unchanged, ids >= hi shifted by
                           // `shift`, ids in [mlo, mhi) shifted by `msh`
};
__device__ __forceinline__ uint32_t remap_of(const RemapView& R, uint32_t k) {
    if (!R.shift) return k;
    const int32_t shf = R.shift[k >> kRemapBlockShift];
    if (shf != kRemapMixed) return (uint32_t)((int64_t)k + shf);
    const uint2 g = R.g32[k >> 5];
    const uint32_t r = k & 31;
    if (g.y >> r & 1) return kNone32;  // dropped
    uint32_t v = (g.x & 0x7FFFFFFFu) + r - (r ? __popc(g.y & (0xFFFFFFFFu >> (32 - r))) : 0u);
    if (g.x >> 31) {
        const uint64_t nv = *R.n_vins;
        v += (uint32_t)(upper_bound_dev(R.ins_oldpos, 0, nv, k) - upper_bound_dev(R.ins_oldpos, 0, nv, k - r));
    }
    return v;
}

// out-of-line exact path (fields by value: no stack copy of the view in the caller)
__device__ __noinline__ uint32_t remap_of_slow(const int32_t* shift, const uint2* g32, const uint32_t* ins_oldpos,
                                               const unsigned long long* n_vins, uint32_t k) {
    RemapView R{shift, g32, ins_oldpos, n_vins, nullptr};
    return remap_of(R, k);
}

// ===================================================================== a1 ====
// Validate + number + split: pending (ts > S) / visible node ops / visible edge
// ops, each stable (ascending seq) via a 3-way decoupled look-back compaction.
__global__ void __launch_bounds__(kThreads) k_partition(
    Ops ops, uint64_t m, uint64_t n_pend_old, uint64_t snap_old, uint64_t S, int check_stale,
    uint32_t* __restrict__ pend_idx, uint32_t* __restrict__ node_idx, uint32_t* __restrict__ edge_idx,
    uint64_t* __restrict__ status3, uint64_t n_tiles, Counters* __restrict__ c) {
    __shared__ uint32_t s_tile;
    __shared__ uint64_t s_scan[kThreads / 32 + 1];
    __shared__ uint64_t s_base[3];
    if (threadIdx.x == 0) s_tile = atomicAdd(&c->tiles[0], 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t i0 = (uint64_t)tile * kTile + (uint64_t)threadIdx.x * kItems;
    uint8_t cat[kItems];
    uint64_t cnt[3] = {0, 0, 0};
    uint64_t bad = 0, tmin = ~0ull, tmax = 0, vmin = ~0ull, vmax = 0;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        uint64_t i = i0 + j;
        cat[j] = 3;
        if (i < m) {
            uint8_t k = ops.kind[i];
            uint64_t t = ops.ts[i];
            if (i >= n_pend_old) {
                if (k > EDGE_WEIGHT) bad |= ST_BAD_KIND;
                if (check_stale && t <= snap_old) bad |= ST_STALE;
            }
            if (t > S) cat[j] = 0;
            else if (k <= NODE_DELETE) {
                cat[j] = 1;
                uint64_t v = ops.src[i];
                tmin = min(tmin, t); tmax = max(tmax, t);
                vmin = min(vmin, v); vmax = max(vmax, v);
            } else cat[j] = 2;
            cnt[0] += cat[j] == 0; cnt[1] += cat[j] == 1; cnt[2] += cat[j] == 2;  // no dynamic index
        }
    }
    if (bad) atomicOr(&c->status, (unsigned long long)bad);
    // node-op ranges: reduced per warp first (one atomic per warp, not per thread: a node-heavy
    // batch would otherwise serialise thousands of atomics on four addresses)
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        tmin = min(tmin, (uint64_t)__shfl_xor_sync(0xffffffffu, tmin, o));
        tmax = max(tmax, (uint64_t)__shfl_xor_sync(0xffffffffu, tmax, o));
        vmin = min(vmin, (uint64_t)__shfl_xor_sync(0xffffffffu, vmin, o));
        vmax = max(vmax, (uint64_t)__shfl_xor_sync(0xffffffffu, vmax, o));
    }
    if (lane_id() == 0 && tmin != ~0ull) {
        atomicMin(&c->ts_min, tmin); atomicMax(&c->ts_max, tmax);
        atomicMin(&c->v_min, vmin); atomicMax(&c->v_max, vmax);
    }
    uint64_t excl[3], tot[3];
#pragma unroll
    for (int q = 0; q < 3; ++q) excl[q] = block_exclusive_scan<kThreads>(cnt[q], s_scan, &tot[q]);
    const int wid = threadIdx.x >> 5;
    if (wid < 3) {
        const uint64_t tw = wid == 0 ? tot[0] : (wid == 1 ? tot[1] : tot[2]);  // register select
        uint64_t b = lookback_warp(status3 + (uint64_t)wid * n_tiles, tile, tw);
        if (lane_id() == 0) {
            s_base[wid] = b;
            if (tile == n_tiles - 1) {
                unsigned long long* dst = wid == 0 ? &c->n_pend : (wid == 1 ? &c->n_node : &c->n_edge);
                *dst = b + tw;
            }
        }
    }
    __syncthreads();
    // three running output positions in registers (no dynamically indexed local arrays)
    uint64_t o0 = s_base[0] + excl[0], o1 = s_base[1] + excl[1], o2 = s_base[2] + excl[2];
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        const uint32_t x = (uint32_t)(i0 + j);
        if (cat[j] == 0) pend_idx[o0++] = x;
        else if (cat[j] == 1) node_idx[o1++] = x;
        else if (cat[j] == 2) edge_idx[o2++] = x;
    }
}

__global__ void k_fill_seq(uint64_t* seq, uint64_t first, uint64_t n, uint64_t seq0) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) seq[first + i] = seq0 + i;
}

__global__ void k_gather_ops(Ops ops, const uint32_t* __restrict__ idx, uint64_t n, uint8_t* kind,
                             uint64_t* src, uint64_t* dst, float* w, uint64_t* ts, uint64_t* seq) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    uint32_t o = idx[i];
    kind[i] = ops.kind[o]; src[i] = ops.src[o]; dst[i] = ops.dst[o];
    w[i] = ops.w[o]; ts[i] = ops.ts[o]; seq[i] = ops.seq[o];
}

// keys[i] = field[idx[i]] - sub ; vals[i] = idx[i]
__global__ void k_keys_from(const uint32_t* __restrict__ idx, uint64_t n, const uint64_t* __restrict__ field,
                            uint64_t sub, uint64_t* __restrict__ keys, uint32_t* __restrict__ vals) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    uint32_t o = idx[i];
    keys[i] = field[o] - sub;
    vals[i] = o;
}

// keys[i] = (src[o] - v0) << tb | (ts[o] - t0) ; vals[i] = o = idx[i]  (node ops: (v, ts) key)
__global__ void k_node_keys(const uint32_t* __restrict__ idx, uint64_t n, const uint64_t* __restrict__ src, uint64_t v0,
                            const uint64_t* __restrict__ ts, uint64_t t0, int tb, uint64_t* __restrict__ keys,
                            uint32_t* __restrict__ vals) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    uint32_t o = idx[i];
    const uint64_t hi = src[o] - v0;
    keys[i] = (tb >= 64 ? 0ull : hi << tb) | (ts[o] - t0);
    vals[i] = o;
}

// Old dense index of external id x.  Identity fast path, else a two-level search:
// fence[i] = ext[i << 8] (V/32 bytes, L2-resident) picks a 256-id block, then a
// binary search inside the block (2 KB) -- one DRAM-latency chain of ~8 probes
// instead of ~25 over the whole 8V-byte array.
constexpr int kFenceShift = 8;
struct ExtIndex {
    const uint64_t* ext;
    const uint64_t* fence;
    uint64_t V, nf;
    int identity;
    const uint8_t* live;  // tombstone mode: liveness per old dense id (nullptr: all live)
};
__device__ __forceinline__ uint64_t old_lookup(const ExtIndex& X, uint64_t x, bool* present) {
    if (X.identity) { *present = x < X.V; return x < X.V ? x : X.V; }
    uint64_t i = upper_bound_dev(X.fence, 0, X.nf, x);
    if (i == 0) { *present = false; return 0; }
    uint64_t lo = (i - 1) << kFenceShift, hi = min(lo + (uint64_t)(1u << kFenceShift), (uint64_t)X.V);
    // a dense run of ids (ext[lo + d] = ext[lo] + d) answers with one probe
    const uint64_t d = x - X.fence[i - 1];
    if (d < hi - lo && X.ext[lo + d] == x) { *present = true; return lo + d; }
    uint64_t k = lower_bound_dev(X.ext, lo, hi, x);
    *present = (k < X.V && X.ext[k] == x);
    return k;
}
__global__ void k_build_fence(const uint64_t* __restrict__ ext, uint64_t V, uint64_t* __restrict__ fence) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if ((i << kFenceShift) < V) fence[i] = ext[i << kFenceShift];
}

// ============================================================ a8 exchange ====
// 40-byte route record (layout of h2tap_route_rec)
struct RouteRec {
    uint64_t src, dst, ts, seq;
    float w;
    uint8_t kind;
    uint8_t pad[3];
};
static_assert(sizeof(RouteRec) == 40, "route record layout");

__global__ void k_validate(const uint8_t* __restrict__ kind, const uint64_t* __restrict__ ts, uint64_t n,
                           uint64_t snap, unsigned long long* __restrict__ status) {
    uint64_t bad = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        if (kind[i] > EDGE_WEIGHT) bad |= ST_BAD_KIND;
        if (ts[i] <= snap) bad |= ST_STALE;
    }
    if (bad) atomicOr(status, (unsigned long long)bad);
}

// owner shard of external id x: number of interior split points <= x
__device__ __forceinline__ int owner_of(const uint64_t* __restrict__ bounds, int P, uint64_t x) {
    int lo = 1, hi = P;  // interior bounds[1..P-1]
    while (lo < hi) { int mid = (lo + hi) >> 1; if (bounds[mid] <= x) lo = mid + 1; else hi = mid; }
    return lo - 1;
}

__global__ void k_route_count(const uint8_t* __restrict__ kind, const uint64_t* __restrict__ src, uint64_t n,
                              const uint64_t* __restrict__ bounds, int P, unsigned long long* __restrict__ counts) {
    extern __shared__ unsigned int s_cnt[];  // P + 1 block-local counters (slot P = node ops)
    for (int d = threadIdx.x; d <= P; d += blockDim.x) s_cnt[d] = 0;
    __syncthreads();
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        atomicAdd(&s_cnt[kind[i] <= NODE_DELETE ? P : owner_of(bounds, P, src[i])], 1u);
    __syncthreads();
    for (int d = threadIdx.x; d < P; d += blockDim.x)
        if (s_cnt[d] + s_cnt[P]) atomicAdd(&counts[d], (unsigned long long)(s_cnt[d] + s_cnt[P]));
}

// stable selection of the ops bound for shard d (node ops go everywhere) into its segment
__global__ void __launch_bounds__(kThreads) k_route_pack(
    const uint8_t* __restrict__ kind, const uint64_t* __restrict__ src, const uint64_t* __restrict__ dst,
    const float* __restrict__ w, const uint64_t* __restrict__ ts, uint64_t n, uint64_t seq0,
    const uint64_t* __restrict__ bounds, int P, int d, RouteRec* __restrict__ out,
    uint64_t* __restrict__ status, unsigned int* __restrict__ ctr) {
    __shared__ uint32_t s_tile;
    __shared__ uint32_t s_cmp[kItems * kThreads / 32 + 1];
    __shared__ uint64_t s_base;
    if (threadIdx.x == 0) s_tile = atomicAdd(ctr, 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t i0 = (uint64_t)tile * kTile + threadIdx.x;
    bool f[kItems];
    uint32_t pos[kItems];
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        const uint64_t i = i0 + (uint64_t)j * kThreads;
        f[j] = i < n && (kind[i] <= NODE_DELETE || owner_of(bounds, P, src[i]) == d);
    }
    const uint32_t tot = striped_compact<kThreads, kItems>(f, pos, s_cmp);
    if (threadIdx.x < 32) {
        const uint64_t b = lookback_warp(status, tile, tot);
        if (lane_id() == 0) s_base = b;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        if (!f[j]) continue;
        const uint64_t i = i0 + (uint64_t)j * kThreads;
        RouteRec r;
        r.src = src[i]; r.dst = dst ? dst[i] : 0; r.ts = ts[i]; r.seq = seq0 + i;
        r.w = w ? w[i] : 0.f; r.kind = kind[i]; r.pad[0] = r.pad[1] = r.pad[2] = 0;
        out[s_base + pos[j]] = r;
    }
}

// Fused pack + exchange ("a fused pack-and-store kernel writing into
// peers' windows"): one pass over the rank's batch slice compacts, per destination shard
// d, the ops bound for d (node ops go to every shard) in arrival order and stores each
// 40-byte route record straight into d's receive buffer — a peer-mapped (CUDA IPC)
// pointer, so the stores travel over NVLink / NVSwitch — at d's offset for this rank
// (the records of lower ranks come first: the global rank-major order, reading A5).
constexpr int kMaxP2P = 16;
struct PeerOut {
    RouteRec* out[kMaxP2P];   // destination d's receive buffer (peer-mapped device pointer)
    uint64_t off[kMaxP2P];    // this rank's first record slot in it
};
__global__ void __launch_bounds__(kThreads) k_route_pack_p2p(
    const uint8_t* __restrict__ kind, const uint64_t* __restrict__ src, const uint64_t* __restrict__ dst,
    const float* __restrict__ w, const uint64_t* __restrict__ ts, uint64_t n, uint64_t seq0,
    const uint64_t* __restrict__ bounds, int P, PeerOut po, uint64_t* __restrict__ status, uint64_t nt,
    unsigned int* __restrict__ ctr) {
    __shared__ uint32_t s_tile;
    __shared__ uint32_t s_cmp[kItems * kThreads / 32 + 1];
    __shared__ uint64_t s_base;
    if (threadIdx.x == 0) s_tile = atomicAdd(ctr, 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t i0 = (uint64_t)tile * kTile + threadIdx.x;
    int own[kItems];  // destination shard, -1 = every shard (node op), -2 = no item
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        const uint64_t i = i0 + (uint64_t)j * kThreads;
        own[j] = i >= n ? -2 : (kind[i] <= NODE_DELETE ? -1 : (int)owner_of(bounds, P, src[i]));
    }
    for (int d = 0; d < P; ++d) {
        bool f[kItems];
        uint32_t pos[kItems];
#pragma unroll
        for (int j = 0; j < kItems; ++j) f[j] = own[j] == -1 || own[j] == d;
        const uint32_t tot = striped_compact<kThreads, kItems>(f, pos, s_cmp);
        if (threadIdx.x < 32) {
            const uint64_t b = lookback_warp(status + (uint64_t)d * nt, tile, tot);
            if (lane_id() == 0) s_base = b;
        }
        __syncthreads();
        RouteRec* out = po.out[d] + po.off[d] + s_base;
#pragma unroll
        for (int j = 0; j < kItems; ++j) {
            if (!f[j]) continue;
            const uint64_t i = i0 + (uint64_t)j * kThreads;
            RouteRec r;
            r.src = src[i]; r.dst = dst ? dst[i] : 0; r.ts = ts[i]; r.seq = seq0 + i;
            r.w = w ? w[i] : 0.f; r.kind = kind[i]; r.pad[0] = r.pad[1] = r.pad[2] = 0;
            out[pos[j]] = r;
        }
        __syncthreads();  // s_base is rewritten by the next destination's look-back
    }
}

__global__ void k_unpack_recs(const RouteRec* __restrict__ recs, uint64_t n, uint8_t* kind, uint64_t* src,
                              uint64_t* dst, float* w, uint64_t* ts, uint64_t* seq) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const RouteRec r = recs[i];
    kind[i] = r.kind; src[i] = r.src; dst[i] = r.dst; w[i] = r.w; ts[i] = r.ts; seq[i] = r.seq;
}

// ============================================================ a1 records ====
// Delta-store scan of the paper's delta-record layout (§5.1-§5.2, P:L604-661,
// P:L702-725): each valid record expands, in the order of reading
// A22, into [NODE_INSERT] EDGE_DELETE* EDGE_INSERT* [NODE_DELETE] at the record's
// transaction timestamp.  Pass 1 counts (and validates) the ops of every record,
// an exclusive scan places them, pass 2 writes them into the work-op SoA.
struct DeltaRec {  // layout of h2tap_delta_record
    uint64_t ts, node, ins_off, del_off;
    uint32_t ins_cnt, del_cnt;
    uint8_t valid, deleted, inserted, pad[5];
};
static_assert(sizeof(DeltaRec) == 48, "delta record layout");
enum : uint32_t { REC_BAD_SLICE = 1, REC_BAD_FLAG = 2 };
// vis_ts: only records with ts <= vis_ts expand (the delta-store scan's visibility check,
// §5.3; UINT64_MAX for a caller-supplied batch); ins_base / del_base: absolute
// array position of element 0 of ins / del (a store's device mirror holds a window)
__global__ void k_rec_count(const DeltaRec* __restrict__ rec, uint64_t n, uint64_t n_ins, uint64_t n_del,
                            uint64_t* __restrict__ cnt, unsigned long long* __restrict__ tot_bad,
                            uint64_t vis_ts = ~0ull, uint64_t ins_base = 0, uint64_t del_base = 0) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    uint64_t c = 0;
    uint32_t bad = 0;
    if (i < n) {
        const DeltaRec r = rec[i];
        if (r.valid > 1 || r.deleted > 1 || r.inserted > 1) bad |= REC_BAD_FLAG;
        if (r.valid) {   // an empty slice's offset is never read
            if ((r.ins_cnt && (r.ins_off < ins_base || r.ins_off - ins_base > n_ins ||
                               r.ins_cnt > n_ins - (r.ins_off - ins_base))) ||
                (r.del_cnt && (r.del_off < del_base || r.del_off - del_base > n_del ||
                               r.del_cnt > n_del - (r.del_off - del_base))))
                bad |= REC_BAD_SLICE;
            if (r.ts <= vis_ts) c = (uint64_t)r.inserted + r.del_cnt + r.ins_cnt + r.deleted;
        }
        cnt[i] = c;
    }
    const unsigned long long s = warp_sum<unsigned long long>(c);
    const uint32_t b = __reduce_or_sync(0xffffffffu, bad);
    if (lane_id() == 0) {
        if (s) atomicAdd(&tot_bad[0], s);
        if (b) atomicOr(&tot_bad[1], (unsigned long long)b);
    }
}
// Expansion: pass 0 (BIG = 0) one thread per record for records of <= kRecSmall ops (most
// deltas are one transaction's change to one node); larger records are queued and pass 1
// (BIG = 1) gives each one warp (a hub's record may carry thousands of inserts).  Weights: f32
// (wts) or the paper's 8-byte weights (wts64) narrowed to the replica's f32 by
// round-to-nearest-even (reading A15).
constexpr uint32_t kRecSmall = 8;
template <int BIG>
__global__ void k_rec_expand(const DeltaRec* __restrict__ rec, uint64_t n, const uint64_t* __restrict__ off,
                             const uint64_t* __restrict__ ins, const float* __restrict__ wts,
                             const uint64_t* __restrict__ del, uint8_t* __restrict__ kind, uint64_t* __restrict__ src,
                             uint64_t* __restrict__ dst, float* __restrict__ w, uint64_t* __restrict__ ts,
                             const double* __restrict__ wts64, uint64_t vis_ts, uint64_t ins_base, uint64_t del_base,
                             uint32_t* __restrict__ big, unsigned long long* __restrict__ n_big) {
    if (!BIG) {
        const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
        if (i >= n) return;
        const DeltaRec r = rec[i];
        if (!r.valid || r.ts > vis_ts) return;
        const uint32_t a = r.inserted, b = a + r.del_cnt, c = b + r.ins_cnt, e = c + r.deleted;
        if (e > kRecSmall) { big[atomicAdd(n_big, 1ull)] = (uint32_t)i; return; }
        const uint64_t o = off[i], io = r.ins_off - ins_base, dq = r.del_off - del_base;
        for (uint32_t j = 0; j < e; ++j) {
            uint8_t k;
            uint64_t d = 0;
            float x = 0.f;
            if (j < a) k = NODE_INSERT;
            else if (j < b) { k = EDGE_DELETE; d = del[dq + (j - a)]; }
            else if (j < c) {
                k = EDGE_INSERT;
                d = ins[io + (j - b)];
                x = wts64 ? __double2float_rn(wts64[io + (j - b)]) : wts[io + (j - b)];
            } else k = NODE_DELETE;
            kind[o + j] = k; src[o + j] = r.node; dst[o + j] = d; w[o + j] = x; ts[o + j] = r.ts;
        }
        return;
    }
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t nb = *n_big;
    for (uint64_t q = warp; q < nb; q += nwarps) {
        const uint64_t i = big[q];
        const DeltaRec r = rec[i];
        if (!r.valid || r.ts > vis_ts) continue;
        const uint64_t o = off[i], io = r.ins_off - ins_base, dq = r.del_off - del_base;
        const uint32_t a = r.inserted, b = a + r.del_cnt, c = b + r.ins_cnt, e = c + r.deleted;
        for (uint32_t j = lane_id(); j < e; j += 32) {
            uint8_t k;
            uint64_t d = 0;
            float x = 0.f;
            if (j < a) k = NODE_INSERT;
            else if (j < b) { k = EDGE_DELETE; d = del[dq + (j - a)]; }
            else if (j < c) {
                k = EDGE_INSERT;
                d = ins[io + (j - b)];
                x = wts64 ? __double2float_rn(wts64[io + (j - b)]) : wts[io + (j - b)];
            } else k = NODE_DELETE;
            kind[o + j] = k; src[o + j] = r.node; dst[o + j] = d; w[o + j] = x; ts[o + j] = r.ts;
        }
    }
}
// after a successful cycle from a delta store: every record the scan used is marked
// invalid ("by the end of the delta store scan"; each delta is used once,
// P:L615-619); first_pending = lowest index of a still-valid (not yet visible) record
__global__ void k_rec_consume(DeltaRec* __restrict__ rec, uint64_t n, uint64_t vis_ts, Counters* __restrict__ c,
                              unsigned long long fail_mask) {
    // runs behind the cycle's last kernel, before its read-back: a cycle whose status carries
    // an error bit marks nothing (the host then reports the error and keeps every delta)
    if (c->status & fail_mask) return;
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    bool pend = false;
    if (i < n && rec[i].valid) {
        if (rec[i].ts <= vis_ts) rec[i].valid = 0;
        else pend = true;
    }
    const uint32_t m = __ballot_sync(0xffffffffu, pend);   // the warp's lowest pending index
    if (m && lane_id() == (uint32_t)(__ffs(m) - 1)) atomicMin(&c->first_pend, (unsigned long long)i);
}

// ===================================================================== a2 ====
// Unique vertices of the (v, ts, seq)-sorted visible node ops: final liveness
// (last op), latest delete point tD, old presence.  Compaction via look-back.
// One op per thread: a segment head walks its segment and then searches the old
// ID map (a chain of dependent loads), so heads must not queue behind each other.
constexpr int kSegTile = kThreads;
__global__ void __launch_bounds__(kThreads) k_node_segments(
    Ops ops, const uint32_t* __restrict__ sidx, uint64_t n, ExtIndex X, NodeVtx* __restrict__ nv,
    uint64_t* __restrict__ nv_ext, uint64_t* __restrict__ status, uint64_t n_tiles, Counters* __restrict__ c) {
    __shared__ uint32_t s_tile;
    __shared__ uint32_t s_cmp[kThreads / 32 + 1];
    __shared__ uint64_t s_base;
    if (threadIdx.x == 0) s_tile = atomicAdd(&c->tiles[1], 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t i = (uint64_t)tile * kSegTile + threadIdx.x;
    const uint64_t v = i < n ? ops.src[sidx[i]] : 0;
    bool head[1] = {i < n && (i == 0 || v != ops.src[sidx[i - 1]])};
    // head work before the compaction so its loads overlap the look-back
    NodeVtx r{};
    if (head[0]) {
        uint64_t e = i;
        r.flags = 0; r.tD_ts = 0; r.tD_seq = 0;
        uint8_t last = NODE_INSERT;
        while (e < n && ops.src[sidx[e]] == v) {
            uint32_t o = sidx[e];
            last = ops.kind[o];
            if (last == NODE_DELETE) { r.tD_ts = ops.ts[o]; r.tD_seq = ops.seq[o]; r.flags |= NV_HASD; }
            ++e;
        }
        if (last == NODE_INSERT) r.flags |= NV_FINAL;
        bool present;
        uint64_t k = old_lookup(X, v, &present);
        if (present) r.flags |= NV_OLD;
        if (present && (!X.live || X.live[k])) r.flags |= NV_LIVE0;
        r.oldpos = (uint32_t)k;
        r.start = (uint32_t)i;
        r.end = (uint32_t)e;
        r.newid = kNone32;
        r.pad = 0;
    }
    uint32_t pos[1];
    uint32_t tot = striped_compact<kThreads, 1>(head, pos, s_cmp);
    if (threadIdx.x < 32) {
        uint64_t b = lookback_warp(status, tile, tot);
        if (lane_id() == 0) { s_base = b; if (tile == n_tiles - 1) c->n_unique = b + tot; }
    }
    __syncthreads();
    if (head[0]) {
        uint64_t q = s_base + pos[0];
        nv[q] = r;
        nv_ext[q] = v;
    }
}

// dropped (old-live -> dead), inserted (new & finally live), hd (old-present with a delete)
__global__ void __launch_bounds__(kThreads) k_node_lists(
    const NodeVtx* __restrict__ nv, uint32_t* __restrict__ dropped,
    uint32_t* __restrict__ ins_q, uint32_t* __restrict__ ins_oldpos, uint32_t* __restrict__ hd_rows,
    uint32_t* __restrict__ hd_bits, uint64_t* __restrict__ status3, uint64_t n_tiles_ub, Counters* __restrict__ c,
    int tomb) {
    __shared__ uint32_t s_tile;
    __shared__ uint64_t s_scan[kThreads / 32 + 1];
    __shared__ uint64_t s_base[3];
    if (threadIdx.x == 0) s_tile = atomicAdd(&c->tiles[2], 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t U = c->n_unique, n_tiles = (U + kTile - 1) / kTile;  // grid: upper bound
    if (tile >= n_tiles) return;
    const uint64_t i0 = (uint64_t)tile * kTile + (uint64_t)threadIdx.x * kItems;
    uint64_t cnt[3] = {0, 0, 0}, killed = 0;
    uint32_t fl[kItems];
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        uint64_t i = i0 + j;
        fl[j] = 0;
        if (i < U) {
            uint32_t f = nv[i].flags;
            bool old = f & NV_OLD, live0 = f & NV_LIVE0, fin = f & NV_FINAL, hd = f & NV_HASD;
            if (live0 && !fin && !tomb) { fl[j] |= 1; cnt[0]++; }  // tombstone mode keeps the slot (A23)
            if (live0 && !fin) killed++;
            if (!old && fin) { fl[j] |= 2; cnt[1]++; }
            if (live0 && hd) { fl[j] |= 4; cnt[2]++; }             // its old edges cascade
        }
    }
    {
        const unsigned long long ks = warp_sum<unsigned long long>(killed);
        if (lane_id() == 0 && ks) atomicAdd(&c->n_killed, ks);
    }
    uint64_t excl[3], tot[3];
#pragma unroll
    for (int q = 0; q < 3; ++q) excl[q] = block_exclusive_scan<kThreads>(cnt[q], s_scan, &tot[q]);
    const int wid = threadIdx.x >> 5;
    if (wid < 3) {
        const uint64_t tw = wid == 0 ? tot[0] : (wid == 1 ? tot[1] : tot[2]);  // register select
        uint64_t b = lookback_warp(status3 + (uint64_t)wid * n_tiles_ub, tile, tw);
        if (lane_id() == 0) {
            s_base[wid] = b;
            if (tile == n_tiles - 1) {
                unsigned long long* d = wid == 0 ? &c->n_dropped : (wid == 1 ? &c->n_inserted : &c->n_hd);
                *d = b + tw;
            }
        }
    }
    __syncthreads();
    uint64_t o0 = s_base[0] + excl[0], o1 = s_base[1] + excl[1], o2 = s_base[2] + excl[2];
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        uint64_t i = i0 + j;
        if (fl[j] & 1) dropped[o0++] = nv[i].oldpos;
        if (fl[j] & 2) { ins_q[o1] = (uint32_t)i; ins_oldpos[o1] = nv[i].oldpos; ++o1; }
        if (fl[j] & 4) {  // + its bit in the deleted-vertex bitmap of the cascade pass
            const uint32_t v = nv[i].oldpos;
            hd_rows[o2++] = v;
            atomicOr(&hd_bits[v >> 5], 1u << (v & 31));
        }
    }
}

// galloping lower bound from a known lower position (keys increase slowly)
template <typename T, typename K>
__device__ __forceinline__ uint64_t gallop_lb(const T* a, uint64_t lo, uint64_t hi, K key) {
    uint64_t step = 1, p = lo;
    while (p < hi && a[p] < key) { lo = p + 1; p = lo + step; step <<= 1; }
    if (p > hi) p = hi;
    return lower_bound_dev(a, lo, p, key);
}
template <typename T, typename K>
__device__ __forceinline__ uint64_t gallop_ub(const T* a, uint64_t lo, uint64_t hi, K key) {
    uint64_t step = 1, p = lo;
    while (p < hi && !(key < a[p])) { lo = p + 1; p = lo + step; step <<= 1; }
    if (p > hi) p = hi;
    return upper_bound_dev(a, lo, p, key);
}

// inserted vertex i lands at oldpos_i - (#dropped before oldpos_i) + i

// new ids of surviving old vertices that have node ops

// tombstone mode: final liveness of the vertices with node ops in the new slots (after
// k_rows_fused copied the old flags): present vertices keep their slot (remapped only by
// insertions), inserted ones take their placed id
// After the node-op lists and the remap tables (a2), one launch, thread i: the ID-map entry
// and new id of the i-th inserted vertex (insertion point minus the dropped ids before it,
// plus the inserted ones before it) and the new id of the i-th unique node-op vertex that
// existed and survives
__global__ void k_node_place(NodeVtx* __restrict__ nv, const uint64_t* __restrict__ nv_ext,
                             const uint32_t* __restrict__ ins_q, const uint32_t* __restrict__ ins_oldpos,
                             const uint32_t* __restrict__ dropped, const Counters* __restrict__ c,
                             uint64_t* __restrict__ new_ext, RemapView R) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < c->n_inserted) {
        const uint32_t op = ins_oldpos[i];
        const uint64_t pos = op - lower_bound_dev(dropped, 0, c->n_dropped, op) + i;
        new_ext[pos] = nv_ext[ins_q[i]];
        nv[ins_q[i]].newid = (uint32_t)pos;
    }
    if (i < c->n_unique) {  // existed and survives (never an inserted vertex: no race with the above)
        const uint32_t f = nv[i].flags;
        if ((f & NV_OLD) && (f & NV_FINAL)) nv[i].newid = remap_of(R, nv[i].oldpos);
    }
}
__global__ void k_nv_live(const NodeVtx* __restrict__ nv, const Counters* __restrict__ c, RemapView R,
                          uint8_t* __restrict__ new_live) {
    const uint64_t q = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (q >= c->n_unique) return;
    const NodeVtx r = nv[q];
    const uint32_t u = (r.flags & NV_OLD) ? remap_of(R, r.oldpos) : r.newid;
    if (u != kNone32) new_live[u] = (r.flags & NV_FINAL) ? 1 : 0;
}

// ===================================================================== a3 ====
struct Lookup {
    int64_t q;        // index in the node-vertex list or -1
    uint32_t oldpos;  // old dense index (present) or insertion rank
    uint32_t newid;
    bool old_present, final_live, hasD, live0;
    uint64_t tD_ts, tD_seq;
};

// Everything the segmented reduce needs about one surviving edge op, in one 32-byte
// sector (the sort carries only the record index; the SoA op arrays would cost
// ~7 scattered sectors per op once the sort passes have evicted them from L2).
struct __align__(32) EdgeRec {
    uint64_t ts, seq;         // commit point (reading A5)
    float w;
    uint32_t opos_u, opos_w;  // old dense index (present) or insertion rank of src / dst
    uint8_t kind;
    uint8_t flags;            // bit0 src old-present, bit1 dst old-present, bit2 key had a node delete
    uint16_t pad;
};

struct PrepArgs {
    Ops ops;
    const uint32_t* edge_idx;
    uint64_t n_edge;
    ExtIndex X;
    RemapView R;            // identity when R.shift == nullptr
    const NodeVtx* nv;
    const uint64_t* nv_ext;
    uint64_t U;                   // node mode: read from c->n_unique at kernel start
    const uint32_t* node_sorted;  // (v, ts, seq)-sorted node op indices
    int bits;                     // bits of a dense id in the packed key
    int create;                   // create_from_edges: endpoints must exist
    OwnRange own;                 // sharded: every edge op's source must be owned here
    uint64_t* keys;
    uint32_t* vals;
    struct EdgeRec* recs;         // one compact record per surviving edge op, indexed by op
    uint64_t* status;
    uint64_t n_tiles;
    Counters* c;
    int count_dev;                // 1: n_edge is an upper bound, the count is c->n_edge (speculative launch)
    const uint32_t* epre;         // node mode: old-map lookups of the endpoints of edge op i at
                                  // [2i], [2i+1] (k_edge_oldpos: old dense id | present << 31)
};

__device__ __forceinline__ Lookup do_lookup(const PrepArgs& a, uint64_t U, uint64_t x, uint32_t pre = kNone32) {
    Lookup L;
    L.q = -1;
    L.hasD = false;
    L.tD_ts = 0; L.tD_seq = 0;
    if (U) {
        uint64_t q = lower_bound_dev(a.nv_ext, 0, U, x);
        if (q < U && a.nv_ext[q] == x) {
            const NodeVtx& r = a.nv[q];
            L.q = (int64_t)q;
            L.oldpos = r.oldpos;
            L.newid = r.newid;
            L.old_present = r.flags & NV_OLD;
            L.live0 = r.flags & NV_LIVE0;
            L.final_live = r.flags & NV_FINAL;
            L.hasD = r.flags & NV_HASD;
            L.tD_ts = r.tD_ts; L.tD_seq = r.tD_seq;
            return L;
        }
    }
    bool present;
    uint64_t k;
    if (pre != kNone32) { k = pre & 0x7FFFFFFFu; present = pre >> 31; }  // looked up earlier
    else k = old_lookup(a.X, x, &present);
    L.oldpos = (uint32_t)k;
    L.old_present = present;
    L.final_live = L.live0 = present && (!a.X.live || a.X.live[k]);
    L.newid = present ? remap_of(a.R, (uint32_t)k) : kNone32;
    return L;
}

// Node mode: the old-map lookups of every visible edge op's endpoints (old dense id | present
// << 31), done on the side stream while the node-op phase runs - before the cascade pass
// saturates HBM, which would multiply the latency of these random ID-map reads inside
// k_edge_prep
__global__ void k_edge_oldpos(Ops ops, const uint32_t* __restrict__ edge_idx, const Counters* __restrict__ c,
                              ExtIndex X, uint32_t* __restrict__ epre) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= c->n_edge) return;
    const uint32_t o = edge_idx[i];
    bool p0, p1;
    const uint64_t k0 = old_lookup(X, ops.src[o], &p0), k1 = old_lookup(X, ops.dst[o], &p1);
    epre[2 * i] = (uint32_t)k0 | (p0 ? 0x80000000u : 0u);
    epre[2 * i + 1] = (uint32_t)k1 | (p1 ? 0x80000000u : 0u);
}

// liveness of a vertex with node ops just before point (ts, seq) (reading A13)
__device__ __forceinline__ bool live_at(const PrepArgs& a, const Lookup& L, uint64_t ts, uint64_t seq) {
    if (L.q < 0) return L.live0;
    const NodeVtx& r = a.nv[L.q];
    uint64_t lo = r.start, hi = r.end;  // first node op with point >= p
    while (lo < hi) {
        uint64_t mid = (lo + hi) >> 1;
        uint32_t o = a.node_sorted[mid];
        if (pt_less(a.ops.ts[o], a.ops.seq[o], ts, seq)) lo = mid + 1; else hi = mid;
    }
    if (lo == r.start) return L.live0;
    return a.ops.kind[a.node_sorted[lo - 1]] == NODE_INSERT;
}

// Per visible edge op: endpoint lookups, liveness gating and node-delete
// supersession (order-free form of the replay), packed key
// (src' << bits | dst'), compaction of surviving ops via look-back.
// EI ops per thread: 1 when ID lookups are searches (latency-bound chains need
// parallelism), 8 for the identity ID map
template <int EI>
__global__ void __launch_bounds__(kThreads) k_edge_prep(PrepArgs a) {
    constexpr int kEItems = EI, kETile = kThreads * EI;
    __shared__ uint32_t s_tile;
    __shared__ uint32_t s_cmp[kEItems * kThreads / 32 + 1];
    __shared__ uint64_t s_base;
    if (threadIdx.x == 0) s_tile = atomicAdd(&a.c->tiles[3], 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    if (a.count_dev) {   // launched before the host knew the count: the partition wrote it
        a.n_edge = min(a.n_edge, (uint64_t)a.c->n_edge);
        a.n_tiles = (a.n_edge + kETile - 1) / kETile;
        if (tile >= a.n_tiles) return;   // beyond the last tile: no later tile depends on it
    }
    const uint64_t i0 = (uint64_t)tile * kETile + threadIdx.x;
    const uint64_t U = a.nv ? a.c->n_unique : 0;
    uint64_t key[kEItems];
    bool valid[kEItems];
    uint32_t pos[kEItems];
    uint64_t ngated = 0, nbad = 0;
    // the op fields of all items are loaded before any record is stored (the stores
    // would otherwise order every later item's loads behind them: possible aliasing)
    uint32_t oj[kEItems];
    uint64_t sj[kEItems], dj[kEItems];
#pragma unroll
    for (int j = 0; j < kEItems; ++j) {
        const uint64_t i = i0 + (uint64_t)j * kThreads;
        oj[j] = i < a.n_edge ? a.edge_idx[i] : 0u;
    }
#pragma unroll
    for (int j = 0; j < kEItems; ++j) {
        const bool in = i0 + (uint64_t)j * kThreads < a.n_edge;
        sj[j] = in ? a.ops.src[oj[j]] : 0;
        dj[j] = in ? a.ops.dst[oj[j]] : 0;
    }
#pragma unroll
    for (int j = 0; j < kEItems; ++j) {
        uint64_t i = i0 + (uint64_t)j * kThreads;
        key[j] = 0;
        valid[j] = false;
        if (i >= a.n_edge) continue;
        uint32_t o = oj[j];
        uint8_t kind = a.ops.kind[o];
        uint64_t ts = a.ops.ts[o], seq = a.ops.seq[o];
        Lookup Lu = do_lookup(a, U, sj[j], a.epre ? a.epre[2 * i] : kNone32);
        Lookup Lw = do_lookup(a, U, dj[j], a.epre ? a.epre[2 * i + 1] : kNone32);
        bool ok = Lu.final_live && Lw.final_live;
        if (a.create && !(Lu.old_present && Lw.old_present)) nbad++;
        // routed to the wrong shard: flagged (the apply fails) and dropped here, so the
        // rest of the cycle never indexes rows this shard does not hold
        if (!a.own.owns(sj[j])) { nbad |= 1ull << 40; ok = false; }
        if (ok && (Lu.hasD || Lw.hasD)) {
            // superseded by a later node delete of an endpoint (A8)
            if (Lu.hasD && pt_less(ts, seq, Lu.tD_ts, Lu.tD_seq)) ok = false;
            if (Lw.hasD && pt_less(ts, seq, Lw.tD_ts, Lw.tD_seq)) ok = false;
        }
        if (ok && kind != EDGE_DELETE && (Lu.q >= 0 || Lw.q >= 0)) {
            if (!live_at(a, Lu, ts, seq) || !live_at(a, Lw, ts, seq)) ok = false;
        }
        if (ok) {
            valid[j] = true;
            key[j] = ((uint64_t)Lu.newid << a.bits) | (uint64_t)Lw.newid;
            EdgeRec rc;
            rc.ts = ts;
            rc.seq = seq;
            rc.w = a.ops.w[o];
            rc.opos_u = Lu.oldpos;
            rc.opos_w = Lw.oldpos;
            rc.kind = kind;
            rc.flags = (uint8_t)((Lu.old_present ? 1 : 0) | (Lw.old_present ? 2 : 0) | ((Lu.hasD || Lw.hasD) ? 4 : 0));
            rc.pad = 0;
            a.recs[o] = rc;  // indexed by op; the sort payload is the op index
        } else {
            ngated++;
        }
    }
    uint64_t gsum = warp_sum(ngated);
    if (lane_id() == 0 && gsum) atomicAdd(&a.c->n_gated, (unsigned long long)gsum);
    uint64_t bsum = warp_sum(nbad & 0xFFFFFFFFFFull), osum = warp_sum(nbad >> 40);
    if (lane_id() == 0 && bsum) atomicOr(&a.c->status, (unsigned long long)ST_CREATE_ENDPOINT);
    if (lane_id() == 0 && osum) atomicOr(&a.c->status, (unsigned long long)ST_NOT_OWNED);
    uint32_t tot = striped_compact<kThreads, kEItems>(valid, pos, s_cmp);
    if (threadIdx.x < 32) {
        uint64_t b = lookback_warp(a.status, tile, tot);
        if (lane_id() == 0) { s_base = b; if (tile == a.n_tiles - 1) a.c->n_valid = b + tot; }
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < kEItems; ++j) {
        if (valid[j]) {
            uint64_t p = s_base + pos[j];
            a.keys[p] = key[j];
            a.vals[p] = a.edge_idx[i0 + (uint64_t)j * kThreads];
        }
    }
}

// ===================================================================== a3' ===
// Segmented arg-max reduce of the key-sorted edge ops (latest-commit-wins,
// insert/delete cancellation) and classification against the old CSR:
//   lastNW = arg-max point over {INSERT, DELETE}; lastW = over {INSERT, WEIGHT}
//   INSERT last  -> upsert(lastW.w)     DELETE last -> delete
//   only WEIGHTs -> update-if-present(lastW.w) (absent if a node delete cleared the key)
// Outcome lists (each sorted by old position): ins (absent keys), del (present
// edges removed), upd (present edges with a new weight).
struct ClassArgs {
    Ops ops;
    const uint64_t* keys;
    const uint32_t* vals;
    uint64_t n;
    int bits;
    const EdgeRec* recs;
    const int64_t* old_off;
    const uint32_t* old_cols;
    uint64_t V_old;
    int direct;                // identity ID map, no node ops: key row == old row
    uint64_t* ins_pos;
    uint32_t* ins_row;
    uint32_t* ins_col;
    float* ins_w;
    uint64_t* del_pos;
    uint32_t* del_row;
    uint64_t* upd_pos;
    float* upd_w;
    uint64_t* status3;
    uint64_t n_tiles;
    Counters* c;
    uint8_t* kcat;    // split mode: per sorted item, 0 none / 1 insert / 2 delete / 3 weight update
    uint64_t* kpos;   //             its old position (lower bound of the key in its old row)
    float* kw;        //             its weight
};

#ifndef H2TAP_CITEMS
#define H2TAP_CITEMS 1
#endif
constexpr int kCItems = H2TAP_CITEMS;  // classify: items per thread (occupancy over ILP)
constexpr int kCTile = kThreads * kCItems;
// SPLIT = 1: the classification alone (no compaction, no look-back), one item per thread in
// launch order: its outcome goes to kcat / kpos / kw and k_classify_compact builds the three
// lists.  The fused form (SPLIT = 0) compacts in the same kernel; there a tile holding a slow
// dependent chain (gather -> row bounds -> probes) delays every later tile's look-back.
template <int SPLIT>
__global__ void __launch_bounds__(kThreads) k_reduce_classify(ClassArgs a) {
    __shared__ uint32_t s_tile;
    __shared__ uint32_t s_cmp[3][kCItems * kThreads / 32 + 1];
    __shared__ uint64_t s_base[3];
    if (!SPLIT && threadIdx.x == 0) s_tile = atomicAdd(&a.c->tiles[4], 1u);
    if (!SPLIT) __syncthreads();
    const uint32_t tile = SPLIT ? blockIdx.x : s_tile;
    const uint64_t n = min(a.n, (uint64_t)a.c->n_valid);  // a.n: the grid's upper bound
    const uint64_t n_tiles = (n + kCTile - 1) / kCTile;
    if (tile >= n_tiles) return;
    const uint64_t i0 = (uint64_t)tile * kCTile + threadIdx.x;
    // Identity ID map (no node ops): the key's row IS the old row, so its bounds are
    // fetched together with the key, off the record-gather chain.
    const bool direct = a.direct;
    uint64_t key[kCItems], lo[kCItems], hi[kCItems];
    uint32_t rec_i[kCItems];
    bool head[kCItems];
#pragma unroll
    for (int j = 0; j < kCItems; ++j) {
        const uint64_t i = i0 + (uint64_t)j * kThreads;
        key[j] = i < n ? a.keys[i] : 0;
        head[j] = i < n && (i == 0 || a.keys[i - 1] != key[j]);
        rec_i[j] = head[j] ? a.vals[i] : 0u;
        lo[j] = hi[j] = 0;
        if (direct && head[j]) {
            const uint64_t u = key[j] >> a.bits;
            lo[j] = (uint64_t)a.old_off[u];
            hi[j] = (uint64_t)a.old_off[u + 1];
        }
    }
    // segmented arg-max over (ts, seq): the first record of every segment is gathered
    // for all items at once; longer segments (repeated keys) continue serially
    EdgeRec r0[kCItems];
#pragma unroll
    for (int j = 0; j < kCItems; ++j)
        if (head[j]) r0[j] = a.recs[rec_i[j]];
    uint8_t cat[kCItems], meta[kCItems];
    uint32_t colq[kCItems];
    float wv[kCItems];
#pragma unroll
    for (int j = 0; j < kCItems; ++j) {
        cat[j] = 0; meta[j] = 0; colq[j] = 0; wv[j] = 0.f;
        if (!head[j]) continue;
        uint64_t nw_ts = 0, nw_seq = 0, w_ts = 0, w_seq = 0;
        bool has_nw = false, has_w = false;
        uint8_t nw_kind = 0;
        float w_val = 0.f;
        EdgeRec re = r0[j];
        for (uint64_t e = i0 + (uint64_t)j * kThreads;;) {
            const uint8_t k = re.kind;
            if (k == EDGE_INSERT || k == EDGE_DELETE) {
                if (!has_nw || pt_less(nw_ts, nw_seq, re.ts, re.seq)) { has_nw = true; nw_ts = re.ts; nw_seq = re.seq; nw_kind = k; }
            }
            if (k == EDGE_INSERT || k == EDGE_WEIGHT) {
                if (!has_w || pt_less(w_ts, w_seq, re.ts, re.seq)) { has_w = true; w_ts = re.ts; w_seq = re.seq; w_val = re.w; }
            }
            if (++e >= n || a.keys[e] != key[j]) break;
            re = a.recs[a.vals[e]];
        }
        const uint8_t fl = r0[j].flags;
        // outcome category before the old-row lookup: 1 insert-like, 2 delete, 3 weight-only
        cat[j] = (has_nw && nw_kind == EDGE_INSERT) ? 1 : (has_nw ? 2 : (has_w ? 3 : 0));
        meta[j] = fl;
        colq[j] = r0[j].opos_w;
        wv[j] = w_val;
        if (!direct) {
            const uint32_t ou = r0[j].opos_u;
            if (fl & 1) { lo[j] = (uint64_t)a.old_off[ou]; hi[j] = (uint64_t)a.old_off[ou + 1]; }
            else { lo[j] = hi[j] = (uint64_t)a.old_off[ou]; }
        }
    }
    uint64_t end[kCItems];
#pragma unroll
    for (int j = 0; j < kCItems; ++j) end[j] = hi[j];
    // lock-step searches of every item's column in its old row.  The first probes
    // interpolate between the known value bounds (columns of a row spread over
    // [0, V)), then plain bisection; cuts DRAM probes per lookup to ~2-3.
    uint32_t vlo[kCItems], vhi[kCItems];
#pragma unroll
    for (int j = 0; j < kCItems; ++j) { vlo[j] = 0; vhi[j] = (uint32_t)a.V_old; }
    // Every probe reads the whole aligned 32-byte sector (8 columns) around the probe
    // point — DRAM moves the sector anyway — and resolves the search if the boundary
    // falls inside it, else narrows past the sector's ends.
    for (int step = 0; step < 48; ++step) {
        bool any = false;
#pragma unroll
        for (int j = 0; j < kCItems; ++j) {
            if (lo[j] < hi[j]) {
                const uint64_t len = hi[j] - lo[j];
                uint64_t mid;
                if (step < 4 && len > 8 && colq[j] >= vlo[j] && vhi[j] > vlo[j]) {
                    mid = lo[j] + (uint64_t)(((float)(colq[j] - vlo[j]) / (float)(vhi[j] - vlo[j])) * (float)len);
                    if (mid >= hi[j]) mid = hi[j] - 1;
                } else {
                    mid = (lo[j] + hi[j]) >> 1;
                }
                const uint64_t base = mid & ~7ull;
                const uint4* q = reinterpret_cast<const uint4*>(a.old_cols + base);
                const uint4 x0 = q[0], x1 = q[1];  // 16 elements of slack past E (over-read)
                const uint32_t x[8] = {x0.x, x0.y, x0.z, x0.w, x1.x, x1.y, x1.z, x1.w};
                const uint32_t s0 = (uint32_t)((lo[j] > base ? lo[j] : base) - base);
                const uint32_t e0 = (uint32_t)((hi[j] < base + 8 ? hi[j] : base + 8) - base);
                uint32_t p = e0, xs = 0, xe = 0;  // first t in [s0, e0) with x[t] >= colq; x[s0], x[e0-1]
#pragma unroll
                for (int t = 7; t >= 0; --t) {
                    if ((uint32_t)t >= s0 && (uint32_t)t < e0 && x[t] >= colq[j]) p = (uint32_t)t;
                    if ((uint32_t)t == s0) xs = x[t];
                    if ((uint32_t)t + 1 == e0) xe = x[t];
                }
                if (p > s0 && p < e0) { lo[j] = hi[j] = base + p; }                       // boundary inside
                else if (p == s0) { hi[j] = base + s0; vhi[j] = xs; }                     // all >= colq
                else { lo[j] = base + e0; vlo[j] = xe + 1; }                              // all < colq
                any = true;
            }
        }
        if (!any) break;
    }
    bool f0[kCItems], f1[kCItems], f2[kCItems];
#pragma unroll
    for (int j = 0; j < kCItems; ++j) {
        uint8_t ct = 0;
        if (cat[j]) {
            const uint64_t p = lo[j];
            const bool found = (meta[j] & 1) && (meta[j] & 2) && p < end[j] && a.old_cols[p] == colq[j];
            const bool present = found && !(meta[j] & 4);  // a node delete of an endpoint cleared the old edge
            if (cat[j] == 1) ct = present ? 3 : 1;
            else if (cat[j] == 2) ct = present ? 2 : 0;
            else ct = present ? 3 : 0;
        }
        cat[j] = ct;
        f0[j] = ct == 1; f1[j] = ct == 2; f2[j] = ct == 3;
    }
    if (SPLIT) {
#pragma unroll
        for (int j = 0; j < kCItems; ++j) {
            const uint64_t i = i0 + (uint64_t)j * kThreads;
            if (i < n) {
                a.kcat[i] = cat[j];
                a.kpos[i] = lo[j];
                a.kw[i] = wv[j];
            }
        }
        return;
    }
    uint32_t rk0[kCItems], rk1[kCItems], rk2[kCItems];
    const uint32_t t0 = striped_compact<kThreads, kCItems>(f0, rk0, s_cmp[0]);
    const uint32_t t1 = striped_compact<kThreads, kCItems>(f1, rk1, s_cmp[1]);
    const uint32_t t2 = striped_compact<kThreads, kCItems>(f2, rk2, s_cmp[2]);
    const int wid = threadIdx.x >> 5;
    if (wid < 3) {
        const uint32_t tw = wid == 0 ? t0 : (wid == 1 ? t1 : t2);
        uint64_t b = lookback_warp(a.status3 + (uint64_t)wid * a.n_tiles, tile, tw);
        if (lane_id() == 0) {
            s_base[wid] = b;
            if (tile == n_tiles - 1) {
                unsigned long long* d = wid == 0 ? &a.c->n_ins : (wid == 1 ? &a.c->n_del : &a.c->n_upd);
                *d = b + tw;
            }
        }
    }
    __syncthreads();
    const uint64_t mask = (1ull << a.bits) - 1;
#pragma unroll
    for (int j = 0; j < kCItems; ++j) {
        if (cat[j] == 1) {
            const uint64_t oi = s_base[0] + rk0[j];
            a.ins_pos[oi] = lo[j];
            a.ins_row[oi] = (uint32_t)(key[j] >> a.bits);
            a.ins_col[oi] = (uint32_t)(key[j] & mask);
            a.ins_w[oi] = wv[j];
        } else if (cat[j] == 2) {
            const uint64_t od = s_base[1] + rk1[j];
            a.del_pos[od] = lo[j];
            a.del_row[od] = (uint32_t)(key[j] >> a.bits);
        } else if (cat[j] == 3) {
            const uint64_t ou = s_base[2] + rk2[j];
            a.upd_pos[ou] = lo[j];
            a.upd_w[ou] = wv[j];
        }
    }
}

// the three outcome lists from the split classification: stable 3-way compaction of the
// classified items (key order), decoupled look-back; the item fields are read only for
// items that go to a list
__global__ void __launch_bounds__(kThreads) k_classify_compact(ClassArgs a) {
    __shared__ uint32_t s_tile;
    __shared__ uint32_t s_cmp[3][kItems * kThreads / 32 + 1];
    __shared__ uint64_t s_base[3];
    if (threadIdx.x == 0) s_tile = atomicAdd(&a.c->tiles[4], 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t n = min(a.n, (uint64_t)a.c->n_valid);
    const uint64_t n_tiles = (n + kTile - 1) / kTile;
    if (tile >= n_tiles) return;
    const uint64_t i0 = (uint64_t)tile * kTile + threadIdx.x;
    uint8_t cat[kItems];
    bool f0[kItems], f1[kItems], f2[kItems];
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        const uint64_t i = i0 + (uint64_t)j * kThreads;
        cat[j] = i < n ? a.kcat[i] : 0;
        f0[j] = cat[j] == 1; f1[j] = cat[j] == 2; f2[j] = cat[j] == 3;
    }
    uint32_t rk0[kItems], rk1[kItems], rk2[kItems];
    const uint32_t t0 = striped_compact<kThreads, kItems>(f0, rk0, s_cmp[0]);
    const uint32_t t1 = striped_compact<kThreads, kItems>(f1, rk1, s_cmp[1]);
    const uint32_t t2 = striped_compact<kThreads, kItems>(f2, rk2, s_cmp[2]);
    const int wid = threadIdx.x >> 5;
    if (wid < 3) {
        const uint32_t tw = wid == 0 ? t0 : (wid == 1 ? t1 : t2);
        uint64_t b = lookback_warp(a.status3 + (uint64_t)wid * a.n_tiles, tile, tw);
        if (lane_id() == 0) {
            s_base[wid] = b;
            if (tile == n_tiles - 1) {
                unsigned long long* d = wid == 0 ? &a.c->n_ins : (wid == 1 ? &a.c->n_del : &a.c->n_upd);
                *d = b + tw;
            }
        }
    }
    __syncthreads();
    const uint64_t mask = (1ull << a.bits) - 1;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        if (!cat[j]) continue;
        const uint64_t i = i0 + (uint64_t)j * kThreads;
        const uint64_t key = a.keys[i], pos = a.kpos[i];
        if (cat[j] == 1) {
            const uint64_t oi = s_base[0] + rk0[j];
            a.ins_pos[oi] = pos;
            a.ins_row[oi] = (uint32_t)(key >> a.bits);
            a.ins_col[oi] = (uint32_t)(key & mask);
            a.ins_w[oi] = a.kw[i];
        } else if (cat[j] == 2) {
            const uint64_t od = s_base[1] + rk1[j];
            a.del_pos[od] = pos;
            a.del_row[od] = (uint32_t)(key >> a.bits);
        } else {
            const uint64_t ou = s_base[2] + rk2[j];
            a.upd_pos[ou] = pos;
            a.upd_w[ou] = a.kw[i];
        }
    }
}

// ===================================================================== a6 ====
// Global merge path: the new column/weight arrays are the merge of the kept old
// elements (old order) with the inserted records (key order); an inserted record
// at old position p precedes old element p, so its merged index is p + r.  Each
// CTA takes a fixed-length diagonal range of the merged sequence (load balanced
// for giant rows and insert bursts), stages its old elements in shared memory,
// drops deleted / cascaded elements, overrides weights, remaps column IDs and
// writes its contiguous output chunk with coalesced 128-bit stores.
constexpr int kMergeTile = 2048;             // merged items per tile
constexpr int kCascBlock = 2048;             // cascade mask: elements per counted block (64 words)
constexpr int kMergeBuf = kMergeTile + 8;     // staged old elements (+ 16 B alignment slack)

struct MergeArgs {
    const uint32_t* old_cols;
    const float* old_w;
    uint64_t E_old;
    const uint64_t* ins_pos;
    const uint32_t* ins_col;
    const float* ins_w;
    uint64_t n_ins;
    const uint64_t* del_pos;
    uint64_t n_del;
    const uint64_t* upd_pos;
    const float* upd_w;
    uint64_t n_upd;
    RemapView R;
    uint32_t* new_cols;
    float* new_w;
    const uint32_t* casc_mask;  // CASC: 1 bit per old element (removed by a node delete)
    const uint64_t* casc_pre;   // CASC: cascaded elements before each 2048-element block
    uint64_t n_tiles;           // host: upper bound (grid / partition size); device: actual
    Counters* c;
};
// the outcome-list sizes live in device memory (no host sync between classify and merge)
__device__ __forceinline__ MergeArgs merge_counts(MergeArgs a) {
    a.n_ins = a.c->n_ins;
    a.n_del = a.c->n_del;
    a.n_upd = a.c->n_upd;
    a.n_tiles = (a.E_old + a.n_ins + kMergeTile - 1) / kMergeTile;
    return a;
}

// Merge-path split of tile boundary t: r = inserted records among the first d
// merged items (smallest r with ins_pos[r] + r >= d), j = d - r old elements,
// and the ranks of j in the sorted delete / update / cascade-row lists.
struct TilePart {
    uint64_t r, dl, ul;
    uint64_t cb;  // cascade mode: cascaded old elements before j
};
static_assert(sizeof(TilePart) == 32, "TilePart is prefetched as 16-byte chunks");

__device__ __forceinline__ uint64_t ins_split(const uint64_t* ins_pos, uint64_t n_ins, uint64_t d) {
    uint64_t lo = 0, hi = n_ins;
    while (lo < hi) {
        uint64_t mid = (lo + hi) >> 1;
        if (ins_pos[mid] + mid < d) lo = mid + 1; else hi = mid;
    }
    return lo;
}

__global__ void k_merge_partition(MergeArgs a_, TilePart* __restrict__ part) {
    const MergeArgs a = merge_counts(a_);
    uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (t > a.n_tiles) return;
    const uint64_t Dtot = a.E_old + a.n_ins;
    const uint64_t d = min(t * kMergeTile, Dtot);
    TilePart p;
    p.r = (d == Dtot) ? a.n_ins : ins_split(a.ins_pos, a.n_ins, d);
    const uint64_t j = d - p.r;
    p.dl = lower_bound_dev(a.del_pos, 0, a.n_del, j);
    p.ul = lower_bound_dev(a.upd_pos, 0, a.n_upd, j);
    p.cb = 0;
    if (a.casc_mask) {  // cascaded elements before j: block prefix + popcount of the partial block
        const uint64_t blk = j / kCascBlock;
        uint64_t c = a.casc_pre[blk];
        for (uint64_t q = blk * (kCascBlock / 32); q < (j >> 5); ++q) c += __popc(a.casc_mask[q]);
        if (j & 31) c += __popc(a.casc_mask[j >> 5] & (0xFFFFFFFFu >> (32 - (j & 31))));
        p.cb = c;
    }
    part[t] = p;
}

// ---- TMA 1-D bulk copy + mbarrier helpers (sm_90+ async proxy; SASS UBLKCP)
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)), "r"(phase) : "memory");
}

// Cascade mode (a4 cascade pass): one bit per old element, set when a node delete
// removes it (its row's vertex or its column's vertex had a visible delete, A8),
// plus per-2048-element block counts.  Runs on a side stream, overlapped with the
// edge-op sort/classify phase, so the merge never touches the cascade bitmap.

// columns pointing at deleted vertices -> mask words (pure stores, every element's
// loads independent).  Persistent: each CTA strides over 4096-element blocks, so the
// prologue (device count + id range of the deleted vertices) is paid once per CTA.
__global__ void __launch_bounds__(kThreads) k_casc_cols(const uint32_t* __restrict__ old_cols, uint64_t E,
        const uint32_t* __restrict__ hd_bits, const uint32_t* __restrict__ hd_rows, const Counters* __restrict__ cn,
        uint32_t* __restrict__ mask) {
    const uint64_t n_hd = cn->n_hd;
    // sorted: id range [hd_lo, hd_lo + span] of deleted vertices (none: empty range)
    const uint32_t hd_lo = n_hd ? hd_rows[0] : 1u;
    const uint32_t span = n_hd ? hd_rows[n_hd - 1] - hd_lo : 0u;
    const bool none = n_hd == 0;
    // each lane owns 4 consecutive elements per step (128-bit loads), a warp step covers
    // 128 elements = 4 mask words; 16 columns in flight per lane
    constexpr int STEPS = 4;
    constexpr uint64_t BLK = 2 * kCascBlock;
    const int w = threadIdx.x >> 5;
    const uint64_t nb = (E + BLK - 1) / BLK;
    const uint64_t wend = ((E + 31) & ~31ull) + 2 * kCascBlock;  // mask words past E are written as 0
    for (uint64_t blk = blockIdx.x; blk < nb; blk += gridDim.x) {
        const uint64_t b0 = blk * BLK;
        const bool full = b0 + BLK <= E;
        uint4 c[STEPS];
#pragma unroll
        for (int j = 0; j < STEPS; ++j) {
            const uint64_t x = b0 + ((uint64_t)(j * (kThreads / 32) + w) * 128) + lane_id() * 4;
            if (none) c[j] = make_uint4(0u, 0u, 0u, 0u);
            else if (full || x + 3 < E) c[j] = __ldcs(reinterpret_cast<const uint4*>(old_cols + x));
            else c[j] = make_uint4(x < E ? old_cols[x] : 0u, x + 1 < E ? old_cols[x + 1] : 0u,
                                   x + 2 < E ? old_cols[x + 2] : 0u, 0u);
        }
        uint32_t bits[STEPS];
#pragma unroll
        for (int j = 0; j < STEPS; ++j) {
            const uint32_t v[4] = {c[j].x, c[j].y, c[j].z, c[j].w};
            uint32_t m = 0;
#pragma unroll
            for (int e = 0; e < 4; ++e) {
                const uint32_t d = v[e] - hd_lo;  // unsigned: one compare for the id range
                if (d <= span && !none) m |= (hd_bits[v[e] >> 5] >> (v[e] & 31) & 1u) << e;
            }
            if (!full) {  // elements past E
                const uint64_t x = b0 + ((uint64_t)(j * (kThreads / 32) + w) * 128) + lane_id() * 4;
                m &= x >= E ? 0u : (x + 4 <= E ? 0xFu : (0xFu >> (4 - (E - x))));
            }
            bits[j] = m;  // 4 bits for this lane's elements
        }
#pragma unroll
        for (int j = 0; j < STEPS; ++j) {
            // lane L holds bits of elements 4L..4L+3 of the 128-element step: word q = L / 8
            uint32_t word = bits[j] << ((lane_id() & 7) * 4);
            word |= __shfl_xor_sync(0xffffffffu, word, 1);
            word |= __shfl_xor_sync(0xffffffffu, word, 2);
            word |= __shfl_xor_sync(0xffffffffu, word, 4);
            const uint64_t x = b0 + ((uint64_t)(j * (kThreads / 32) + w) * 128);
            if ((lane_id() & 7) == 0 && x + lane_id() * 4 < wend) mask[(x >> 5) + lane_id() / 8] = word;
        }
    }
}

// The same pass streamed with TMA: one CTA of 256 threads per SM, the columns arriving in
// 32 KB bulk copies (2 buffers in flight per SM, ~9.5 MB across the GPU) signalled on
// mbarriers, and the deleted-vertex bits of [hd_lo, hd_lo + span] copied into shared memory
// when they fit (32 KB), so the pass runs near HBM speed while leaving 7/8 of every SM's
// threads to the latency-bound edge-op kernels it overlaps.  Warp w turns kCcSub staged
// columns into kCcSub / 32 mask words (lane-interleaved reads, one ballot per word) and
// stores them with one coalesced store.
constexpr int kCcChunk = 8192;                 // columns per bulk copy
constexpr int kCcBuf = 2;
#ifndef H2TAP_CC_THREADS
#define H2TAP_CC_THREADS 256
#endif
constexpr int kCcThreads = H2TAP_CC_THREADS;
constexpr int kCcSub = kCcChunk / (kCcThreads / 32);  // columns per warp per chunk (<= 1024)
static_assert(kCcSub % 32 == 0 && kCcSub <= 1024, "a warp turns kCcSub columns into kCcSub / 32 mask words");
constexpr int kCcHdWords = 8192;               // deleted-vertex bitmap window in shared memory
constexpr int kCcSmem = kCcBuf * kCcChunk * 4 + kCcHdWords * 4;  // dynamic shared memory
__global__ void __launch_bounds__(kCcThreads, 1) k_casc_cols_tma(const uint32_t* __restrict__ old_cols, uint64_t E,
        const uint32_t* __restrict__ hd_bits, const uint32_t* __restrict__ hd_rows, const Counters* __restrict__ cn,
        uint32_t* __restrict__ mask) {
    extern __shared__ __align__(128) uint8_t cc_dsm[];
    uint32_t* sb = reinterpret_cast<uint32_t*>(cc_dsm);
    uint32_t* s_hd = sb + kCcBuf * kCcChunk;
    __shared__ __align__(8) uint64_t bar[kCcBuf];
    const uint64_t n_hd = cn->n_hd;
    const uint32_t hd_lo = n_hd ? hd_rows[0] : 1u;
    const uint32_t span = n_hd ? hd_rows[n_hd - 1] - hd_lo : 0u;
    const uint64_t nch = (E + kCcChunk - 1) / kCcChunk;
    const uint64_t wend = ((E + 31) >> 5) + 2 * kCascBlock / 32;  // mask words past E are written as 0
    const int tid = threadIdx.x, w = tid >> 5;
    const uint32_t lane = lane_id();
    const uint64_t G = gridDim.x;
    if (n_hd == 0) {  // no deleted vertex: an all-zero mask
        for (uint64_t q = blockIdx.x * (uint64_t)kCcThreads + tid; q < wend; q += G * kCcThreads) mask[q] = 0u;
        return;
    }
    auto issue = [&](uint64_t c, int b) {  // thread 0
        const uint64_t c0 = c * kCcChunk;
        const uint32_t nc = (uint32_t)min((uint64_t)kCcChunk, E - c0);
        const uint32_t bytes = ((nc + 3) & ~3u) * 4;  // 16-byte multiple (the buffers have slack)
        mbar_expect_tx(&bar[b], bytes);
        bulk_g2s(sb + b * kCcChunk, old_cols + c0, bytes, &bar[b]);
    };
    if (tid == 0) {
        for (int b = 0; b < kCcBuf; ++b) mbar_init(&bar[b], 1);
        fence_mbar_init();
        for (int b = 0; b < kCcBuf; ++b)
            if (blockIdx.x + b * G < nch) issue(blockIdx.x + b * G, b);
    }
    // the bitmap words of ids hd_lo .. hd_lo + span (word-aligned window)
    const uint32_t hw0 = hd_lo >> 5, hwn = ((hd_lo + span) >> 5) - hw0 + 1;
    const bool hd_smem = hwn <= (uint32_t)kCcHdWords;
    if (hd_smem)
        for (uint32_t q = tid; q < hwn; q += kCcThreads) s_hd[q] = hd_bits[hw0 + q];
    __syncthreads();
    uint64_t i = 0;
    for (uint64_t c = blockIdx.x; c < nch; c += G, ++i) {
        const int b = (int)(i % kCcBuf);
        mbar_wait(&bar[b], (uint32_t)((i / kCcBuf) & 1));
        const uint32_t* s = sb + b * kCcChunk;
        const uint64_t c0 = c * kCcChunk;
        const uint32_t nc = (uint32_t)min((uint64_t)kCcChunk, E - c0);
        {
            const int sub = w;
            uint32_t mine = 0;
#pragma unroll 8
            for (int q = 0; q < kCcSub / 32; ++q) {
                const uint32_t j = sub * kCcSub + q * 32 + lane;
                const uint32_t v = s[j], d = v - hd_lo;
                bool hit = false;
                if (j < nc && d <= span)
                    hit = hd_smem ? (s_hd[(v >> 5) - hw0] >> (v & 31)) & 1u : (hd_bits[v >> 5] >> (v & 31)) & 1u;
                const uint32_t word = __ballot_sync(0xffffffffu, hit);
                if (lane == (uint32_t)q) mine = word;
            }
            const uint64_t q = ((c0 + sub * kCcSub) >> 5) + lane;
            if (lane < kCcSub / 32 && q < wend) mask[q] = mine;
        }
        __syncthreads();  // buffer b fully consumed
        if (tid == 0 && c + kCcBuf * G < nch) {
            fence_proxy_async();
            issue(c + kCcBuf * G, b);
        }
    }
    if (blockIdx.x == 0)  // words past the last chunk
        for (uint64_t q = nch * (kCcChunk / 32) + tid; q < wend; q += kCcThreads) mask[q] = 0u;
}

// rows of deleted vertices -> whole bit ranges (warp per row), OR-ed into the mask
__global__ void k_casc_rows(const int64_t* __restrict__ old_off, const uint32_t* __restrict__ hd_rows,
                            const Counters* __restrict__ cn, uint64_t row_lo, uint64_t row_hi, uint32_t* __restrict__ mask) {
    const uint64_t n_hd = cn->n_hd;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t h = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; h < n_hd; h += nw) {
        if (hd_rows[h] < row_lo || hd_rows[h] >= row_hi) continue;  // not a row of this shard
        const uint64_t k = hd_rows[h] - row_lo;
        uint64_t b = (uint64_t)old_off[k], e = (uint64_t)old_off[k + 1];
        if (b == e) continue;
        uint64_t wb = b >> 5, we = (e - 1) >> 5;
        for (uint64_t q = wb + lane_id(); q <= we; q += 32) {
            uint32_t m = 0xFFFFFFFFu;
            if (q == wb) m &= 0xFFFFFFFFu << (b & 31);
            if (q == we) m &= 0xFFFFFFFFu >> (31 - ((e - 1) & 31));
            if (m == 0xFFFFFFFFu) mask[q] = m; else atomicOr(&mask[q], m);
        }
    }
}

// per 2048-element block: cascaded count = popcount of its 64 mask words, the
// per-word prefix inside the block (u16), then the exclusive scan over blocks
// (decoupled look-back), total at [nblk].  cascaded_before(x) =
// pre[x / 2048] + wrel[x / 32] + popc(mask[x / 32] below bit x % 32).
__global__ void __launch_bounds__(kThreads) k_casc_scan(const uint32_t* __restrict__ mask, uint64_t nblk,
        uint64_t* __restrict__ pre, uint16_t* __restrict__ wrel, uint64_t* __restrict__ status,
        unsigned int* __restrict__ ctr) {
    __shared__ uint32_t s_tile;
    __shared__ uint64_t s_scan[kThreads / 32 + 1];
    __shared__ uint64_t s_cnt[kThreads];
    __shared__ uint64_t s_base;
    if (threadIdx.x == 0) s_tile = atomicAdd(ctr, 1u);
    __syncthreads();
    const uint64_t blk0 = (uint64_t)s_tile * kThreads;  // one block count per thread
    const int w = threadIdx.x >> 5;
    // warp w handles blocks blk0 + w*32 + i (2 words per lane); the mask loads of 16 blocks are
    // issued together (one dependent L2 round trip per 16 blocks, not per block)
    for (int i0 = 0; i0 < 32; i0 += 16) {
        uint2 vv[16];
#pragma unroll
        for (int i = 0; i < 16; ++i) {
            const uint64_t bk = blk0 + w * 32 + i0 + i;
            vv[i] = bk < nblk ? reinterpret_cast<const uint2*>(mask + bk * (kCascBlock / 32))[lane_id()]
                              : make_uint2(0u, 0u);
        }
#pragma unroll
        for (int i = 0; i < 16; ++i) {
            const uint64_t bk = blk0 + w * 32 + i0 + i;
            uint32_t c = 0;
            if (bk < nblk) {
                const uint32_t c0 = __popc(vv[i].x), c1 = __popc(vv[i].y);
                const uint32_t inc = warp_inclusive_scan(c0 + c1);
                reinterpret_cast<ushort2*>(wrel + bk * (kCascBlock / 32))[lane_id()] =
                    make_ushort2((uint16_t)(inc - c0 - c1), (uint16_t)(inc - c1));
                c = __shfl_sync(0xffffffffu, inc, 31);
            }
            if (lane_id() == 0) s_cnt[w * 32 + i0 + i] = c;
        }
    }
    __syncthreads();
    uint64_t v = s_cnt[threadIdx.x], tot;
    uint64_t ex = block_exclusive_scan<kThreads>(v, s_scan, &tot);
    if (threadIdx.x < 32) {
        uint64_t b = lookback_warp(status, s_tile, tot);
        if (lane_id() == 0) s_base = b;
    }
    __syncthreads();
    uint64_t bk = blk0 + threadIdx.x;
    if (bk <= nblk) pre[bk] = s_base + ex;
}

// Row offsets with node ops (a4/a5): thread per old row k that survives,
//   new_off[u'] = x - (cascaded before x) - (deleted before x) + (inserted records in rows < u')
// with x = old_off[k]; the CTA narrows the sorted delete / insert-row lists first.
#ifndef H2TAP_ROW_TILE
#define H2TAP_ROW_TILE 256
#endif
constexpr int kRowTile = H2TAP_ROW_TILE;  // old ids per CTA of the node-mode row pass
struct RowArgs {
    const int64_t* old_off;
    uint64_t V_old, E_old;
    RemapView R;  // identity when R.shift == nullptr
    const uint32_t* casc_mask;
    const uint64_t* casc_pre;
    const uint16_t* casc_wrel;
    const uint64_t* del_pos;
    const uint32_t* del_row;  // k_offsets_direct
    uint64_t n_del;
    const uint32_t* ins_row;
    uint64_t n_ins;
    const uint32_t* dropped;
    uint64_t n_dropped;
    const uint32_t* ins_oldpos;
    uint64_t n_vins;
    int64_t* new_off;
    uint64_t* part;  // [n_cta + 1][2]: delete rank and insert-row rank at each CTA's first row
    uint64_t row_lo, row_hi;  // old rows of this shard (global dense ids); old_off is biased by row_lo
    uint64_t row_lo_new;      // first new row of this shard (new_off is local)
    OwnRange own;
    const uint64_t* nv_ext;
    const Counters* c;        // device-side list sizes (read by row_counts)
    const uint64_t* old_ext;  // ID maps (k_rows_fused); identity: old ext id == k
    uint64_t* new_ext;
    int identity;
    const uint8_t* old_live;  // tombstone mode: liveness carried to the new slots
    uint8_t* new_live;
    const unsigned long long* same;  // back ID-map buffer == front on [0, *same) (nullptr: unknown)
};
__device__ __forceinline__ RowArgs row_counts(RowArgs a) {
    a.n_del = a.c->n_del;
    a.n_ins = a.c->n_ins;
    a.n_dropped = a.c->n_dropped;
    a.n_vins = a.c->n_inserted;
    a.row_lo_new = a.c->row_lo_new;
    return a;
}
__device__ __forceinline__ uint64_t casc_before(const RowArgs& a, uint64_t x) {
    if (!a.casc_mask) return 0;
    if (x >= a.E_old) return a.casc_pre[(a.E_old + kCascBlock - 1) / kCascBlock];  // all cascaded
    const uint32_t r = x & 31;
    return a.casc_pre[x / kCascBlock] + a.casc_wrel[x >> 5] +
           (r ? __popc(a.casc_mask[x >> 5] & (0xFFFFFFFFu >> (32 - r))) : 0u);
}
// CTA boundaries of k_rows_fused (CTA c covers old ids [c*kRowTile, (c+1)*kRowTile)):
// ranks of each CTA's first shard row (clamped to [row_lo, row_hi]) in the sorted
// delete and insert-row lists
template <int TILE = kRowTile>
__global__ void k_rows_partition(RowArgs a_) {
    const RowArgs a = row_counts(a_);
    const uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    const uint64_t ncta = (a.V_old + TILE - 1) / TILE;
    if (c > ncta) return;
    const uint64_t k = min(max(c * TILE, a.row_lo), a.row_hi);
    uint64_t dr, ir;
    if (k >= a.row_hi) { dr = a.n_del; ir = a.n_ins; }
    else {
        dr = lower_bound_dev(a.del_pos, 0, a.n_del, (uint64_t)a.old_off[k]);
        // insert-row rank of the new id of the first surviving row >= k (compaction formula)
        const uint64_t u = k - lower_bound_dev(a.dropped, 0, a.n_dropped, (uint32_t)k) +
                           upper_bound_dev(a.ins_oldpos, 0, a.n_vins, (uint32_t)k);
        ir = lower_bound_dev(a.ins_row, 0, a.n_ins, (uint32_t)u);
    }
    a.part[2 * c] = dr;
    a.part[2 * c + 1] = ir;
}

// One pass over the old vertices k (node ops only; a2 + a4/a5): each survivor's
// new dense id u = remap(k) places its external id in the new ID map and, for the
// rows of this shard, its new row offset
//   new_off[u] = x - (cascaded before x) - (deleted before x) + (inserted records in rows < u)
// with x = old_off[k].  The CTA narrows the sorted delete / insert-row lists first.
#ifndef H2TAP_ROWS_MINB
#define H2TAP_ROWS_MINB 8
#endif
__global__ void __launch_bounds__(kThreads, H2TAP_ROWS_MINB) k_rows_fused(RowArgs a_) {
    const RowArgs a = row_counts(a_);
    const uint64_t k0 = (uint64_t)blockIdx.x * kRowTile, k1 = min(k0 + kRowTile, a.V_old);
    const uint64_t* pp = a.part + 2 * blockIdx.x;  // this CTA's slices of the delete / insert-row lists
    const uint64_t da = pp[0], ia = pp[1], db = pp[2], ib = pp[3];
    // ID-map prefix already in place: ids below R.lohi[0] keep their dense id (u = k) and
    // external id, and the back buffer equals the front one on [0, *same)
    const uint64_t keep = (a.same && !a.new_live) ? min((uint64_t)*a.same, (uint64_t)(uint32_t)a.R.lohi[0]) : 0;
    constexpr int PER = kRowTile / kThreads;  // ids per thread, all loads issued together
    uint32_t u[PER];
    uint64_t x[PER], ext[PER];
    bool row[PER], wext[PER];
#pragma unroll
    for (int j = 0; j < PER; ++j) {
        const uint64_t k = k0 + threadIdx.x + (uint64_t)j * kThreads;
        u[j] = kNone32;
        x[j] = 0;
        ext[j] = k;
        row[j] = false;
        wext[j] = k >= keep;
        if (k < k1) {
            u[j] = remap_of(a.R, (uint32_t)k);
            if (!a.identity && wext[j]) ext[j] = a.old_ext[k];
            if (a.new_live && u[j] != kNone32) a.new_live[u[j]] = a.old_live[k];
            row[j] = k >= a.row_lo && k < a.row_hi;
            if (row[j]) x[j] = (uint64_t)a.old_off[k];
        }
    }
    uint64_t cb[PER];
#pragma unroll
    for (int j = 0; j < PER; ++j) cb[j] = (u[j] != kNone32 && row[j]) ? casc_before(a, x[j]) : 0;
#pragma unroll
    for (int j = 0; j < PER; ++j) {
        if (u[j] == kNone32) continue;
        if (wext[j]) a.new_ext[u[j]] = ext[j];
        if (!row[j]) continue;
        const uint64_t kept = x[j] - cb[j] - lower_bound_dev(a.del_pos, da, db, x[j]);
        a.new_off[u[j] - a.row_lo_new] = (int64_t)(kept + lower_bound_dev(a.ins_row, ia, ib, u[j]));
    }
}

// ID-map prefix bookkeeping (node mode).  *same: the back ID-map buffer equals the front
// one on [0, *same).  The survivor pass rewrote the back buffer from min(*same, lo) on, so
// it then equals the front one only below that (what an abort leaves; k_rows_finish marks
// it); after the swap the two buffers hold consecutive snapshots, equal below this cycle's lo.
__global__ void k_idmap_commit(unsigned long long* same) { same[0] = same[1]; }

// Row offsets without node ops (a4/a5; identity remap, no cascade): the exclusive
// scan of the per-row degree delta at row k is a difference of two ranks in the
// sorted outcome lists, so one streaming pass replaces scatter + scan:
//   new_off[k] = x - (deleted old elements before x) + (inserted records in rows < k),
// x = old_off[k].  CTA c covers rows [c*kRowTile, (c+1)*kRowTile) of the shard;
// k_rows_partition supplies its slices of the two lists.
#ifndef H2TAP_OFF_TILE
#define H2TAP_OFF_TILE 4096
#endif
constexpr int kOffTile = H2TAP_OFF_TILE;  // rows per CTA of k_offsets_direct
// CTA boundaries for k_offsets_direct without searches: part[2c] / part[2c+1] = number of
// deletes / inserted records in rows < c*kOffTile.  Both lists are sorted by row, so
// element i writes the boundaries c in (tile(row[i-1]), tile(row[i])] (the last element
// also the ones past its tile): one pass over the lists, no dependent search chains.
__global__ void k_offsets_bounds(const uint32_t* __restrict__ del_row, const uint32_t* __restrict__ ins_row,
                                 const Counters* __restrict__ c, uint64_t n_ub, uint64_t ncta,
                                 uint64_t* __restrict__ part) {
    const uint64_t n_del = c->n_del, n_ins = c->n_ins;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n_ub + 1; i += stride) {
#pragma unroll
        for (int l = 0; l < 2; ++l) {
            const uint32_t* rows = l ? ins_row : del_row;
            const uint64_t n = l ? n_ins : n_del;
            if (n == 0) {  // empty list: every boundary is 0
                for (uint64_t cc = i; cc <= ncta; cc += n_ub + 1) part[2 * cc + l] = 0;
                continue;
            }
            if (i > n) continue;
            const uint64_t c_lo = i == 0 ? 0 : (uint64_t)rows[i - 1] / kOffTile + 1;
            const uint64_t c_hi = i == n ? ncta : (uint64_t)rows[i] / kOffTile;
            for (uint64_t cc = c_lo; cc <= c_hi && cc <= ncta; ++cc) part[2 * cc + l] = i;
        }
    }
}
__global__ void __launch_bounds__(kThreads) k_offsets_direct(RowArgs a_) {
    // per-row degree delta of the CTA's rows in a shared-memory histogram (from its
    // slices of the two sorted lists), scanned in place; old and new offsets move
    // with coalesced (row-strided) accesses
    constexpr int PER = kOffTile / kThreads;
    constexpr int kPad = kOffTile + kOffTile / 32;
    __shared__ int32_t s_cnt[kPad];  // padded: index i at i + i/32 (conflict-free blocked scan)
    __shared__ int64_t s_scan[kThreads / 32 + 1];
    const RowArgs a = row_counts(a_);
    const uint64_t c = blockIdx.x + a.row_lo / kOffTile, kb = c * kOffTile;
    const uint32_t l0 = (uint32_t)(max(kb, a.row_lo) - kb), l1 = (uint32_t)(min(kb + kOffTile, a.row_hi) - kb);
    const uint64_t* pp = a.part + 2 * c;
    const uint64_t da = pp[0], ia = pp[1], db = pp[2], ib = pp[3];
    const int64_t* oo = a.old_off + kb;
    int64_t x[PER];
#pragma unroll
    for (int j = 0; j < PER; ++j) {
        const uint32_t l = threadIdx.x + j * kThreads;
        x[j] = (l >= l0 && l < l1) ? oo[l] : 0;
    }
    auto P = [](uint32_t i) { return i + (i >> 5); };
#pragma unroll
    for (int j = 0; j < PER; ++j) s_cnt[P(threadIdx.x + j * kThreads)] = 0;
    __syncthreads();
    for (uint64_t i = ia + threadIdx.x; i < ib; i += kThreads) atomicAdd(&s_cnt[P((uint32_t)(a.ins_row[i] - kb))], 1);
    for (uint64_t i = da + threadIdx.x; i < db; i += kThreads) atomicAdd(&s_cnt[P((uint32_t)(a.del_row[i] - kb))], -1);
    __syncthreads();
    int32_t sum = 0;
#pragma unroll
    for (int j = 0; j < PER; ++j) sum += s_cnt[P(threadIdx.x * PER + j)];
    int32_t tot, run = block_exclusive_scan<kThreads>(sum, (int32_t*)s_scan, &tot);
#pragma unroll
    for (int j = 0; j < PER; ++j) { const int32_t dj = s_cnt[P(threadIdx.x * PER + j)]; s_cnt[P(threadIdx.x * PER + j)] = run; run += dj; }
    __syncthreads();
    const int64_t base = (int64_t)ia - (int64_t)da;
    int64_t* o = a.new_off + (kb - a.row_lo);
#pragma unroll
    for (int j = 0; j < PER; ++j) {
        const uint32_t l = threadIdx.x + j * kThreads;
        if (l >= l0 && l < l1) o[l] = x[j] + base + s_cnt[P(l)];
    }
}

// Sharded mode: the shard's row range in the new ID map, without the map itself:
// survivors below the old range start + inserted vertices below the owned ext range
__global__ void k_row_range_new(const uint32_t* __restrict__ dropped, const uint32_t* __restrict__ ins_q,
                                const uint64_t* __restrict__ nv_ext, uint64_t row_lo, uint64_t row_hi, OwnRange own,
                                Counters* __restrict__ c) {
    const uint64_t nd = c->n_dropped, ni = c->n_inserted;
    auto ins_below = [&](uint64_t x) {  // inserted vertices (ascending ext ids) with ext < x
        uint64_t lo = 0, hi = ni;
        while (lo < hi) { uint64_t m = (lo + hi) >> 1; if (nv_ext[ins_q[m]] < x) lo = m + 1; else hi = m; }
        return lo;
    };
    c->row_lo_new = row_lo - lower_bound_dev(dropped, 0, nd, (uint32_t)row_lo) + ins_below(own.lo);
    c->row_hi_new = own.hi == ~0ull ? c->Vn
                                    : row_hi - lower_bound_dev(dropped, 0, nd, (uint32_t)row_hi) + ins_below(own.hi);
}

// Device-wide exclusive scan of u64 values, single pass (decoupled look-back).
__global__ void __launch_bounds__(kThreads) k_scan_exclusive_u64(const uint64_t* __restrict__ in,
        uint64_t* __restrict__ out, uint64_t n, uint64_t* __restrict__ status, unsigned int* __restrict__ ctr) {
    __shared__ uint32_t s_tile;
    __shared__ uint64_t s_scan[kThreads / 32 + 1];
    __shared__ uint64_t s_base;
    if (threadIdx.x == 0) s_tile = atomicAdd(ctr, 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t i0 = (uint64_t)tile * kTile + (uint64_t)threadIdx.x * kItems;
    uint64_t v[kItems], sum = 0;
#pragma unroll
    for (int j = 0; j < kItems; ++j) { v[j] = (i0 + j < n) ? in[i0 + j] : 0; sum += v[j]; }
    uint64_t tot, ex = block_exclusive_scan<kThreads>(sum, s_scan, &tot);
    if (threadIdx.x < 32) {
        uint64_t b = lookback_warp(status, tile, tot);
        if (lane_id() == 0) s_base = b;
    }
    __syncthreads();
    uint64_t run = s_base + ex;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        if (i0 + j < n) out[i0 + j] = run;
        run += v[j];
    }
}

constexpr int kMerge3Smem = 6 * kMergeBuf * 4;  // dynamic shared memory of k_merge3


// ---- TMA bulk store (smem -> global) helpers
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                 ::"l"(dst), "r"(smem_u32(src)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// ---- cp.async (16 B, generic proxy) for small prefetches into shared memory
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

// Merge (a6).  Tile t covers merged items [t*2048, (t+1)*2048): old elements
// [j0, j1) (TMA-staged, double-buffered) and inserted records [r0, r1).
//   phase A (warp 0, per 32-element chunk): keep mask (not deleted, not cascaded),
//            scans of kept counts and of inserted-record counts -> s_chunk
//   phase B: old element i goes to e = kept_before(i) + I(i), I(i) = inserted records
//            at local positions <= i (uniform per chunk unless one falls inside);
//            values (remapped column, weight) staged in smem at e + (base & 3)
//   inserted records: e = kept_before(p) + s
//   store: scalar head/tail, one TMA bulk store per array for the aligned body
// Software pipeline: while tile t is processed, the TMA loads of tile t+G are in
// flight, tile t+2G's partition entries stream in by cp.async, and the heads of
// tile t+G's edit lists are loaded into registers; three barriers per tile
// (deleted/insert-count masks are double-buffered).
template <bool CASC, bool REMAP>
__global__ void __launch_bounds__(kThreads) k_merge3(MergeArgs a_, const TilePart* __restrict__ part) {
    const MergeArgs a = merge_counts(a_);
    constexpr int NCH = kMergeTile / 32;  // 64 chunks of 32 old elements
    extern __shared__ __align__(128) uint8_t dsm[];  // kMerge3Smem bytes
    auto s_col = reinterpret_cast<uint32_t(*)[kMergeBuf]>(dsm);
    auto s_w = reinterpret_cast<float(*)[kMergeBuf]>(dsm + 2 * kMergeBuf * 4);
    uint32_t* s_oc = reinterpret_cast<uint32_t*>(dsm + 4 * kMergeBuf * 4);
    float* s_ow = reinterpret_cast<float*>(dsm + 5 * kMergeBuf * 4);
    __shared__ uint16_t s_ins[kMergeTile + 1];
    __shared__ uint32_t s_dmask[2][NCH + 2];  // deleted old elements per chunk (by buffer)
    __shared__ uint32_t s_icnt[2][NCH + 2];   // inserted records per chunk of insertion positions
    __shared__ uint4 s_chunk[NCH + 1];        // {keep mask, kept before, inserted before, inserted inside}
    __shared__ __align__(8) uint64_t s_bar[2];
    __shared__ uint64_t s_meta[2][6];         // r0, r1, dl0, ul0, nd | nu << 16, cascaded before j0
    __shared__ __align__(16) TilePart s_tp[2][2];

    const int tid = threadIdx.x, wid = tid >> 5;
    const uint32_t lane = lane_id(), lt = lanemask_lt();
    const uint64_t Dtot = a.E_old + a.n_ins;
    const uint64_t G = gridDim.x;
    auto issue = [&](uint64_t tt, int bb, const TilePart& p0, const TilePart& p1) {  // thread 0
        s_meta[bb][0] = p0.r; s_meta[bb][1] = p1.r; s_meta[bb][2] = p0.dl; s_meta[bb][3] = p0.ul;
        s_meta[bb][4] = (p1.dl - p0.dl) | ((p1.ul - p0.ul) << 16);
        s_meta[bb][5] = p0.cb;
        const uint64_t j0 = min(tt * kMergeTile, Dtot) - p0.r, j1 = min((tt + 1) * kMergeTile, Dtot) - p1.r;
        const uint64_t a0 = j0 & ~3ull, a1 = (j1 + 3) & ~3ull;
        const uint32_t bytes = (uint32_t)((a1 - a0) * 4);
        mbar_expect_tx(&s_bar[bb], 2 * bytes);
        if (bytes) {
            bulk_g2s(&s_col[bb][0], a.old_cols + a0, bytes, &s_bar[bb]);
            bulk_g2s(&s_w[bb][0], a.old_w + a0, bytes, &s_bar[bb]);
        }
    };
    auto prefetch_part = [&](uint64_t tt, int slot) {  // thread 0: part[tt], part[tt + 1] -> s_tp[slot]
        const uint4* src = reinterpret_cast<const uint4*>(part + tt);
        uint4* dst = reinterpret_cast<uint4*>(&s_tp[slot][0]);
#pragma unroll
        for (int q = 0; q < 2 * (int)sizeof(TilePart) / 16; ++q) cp_async16(dst + q, src + q);
        cp_async_commit();
    };
    // remap fast paths: ids below lohi[0] keep their id, ids at or above lohi[1] shift by
    // lohi[2], ids in [lohi[3], lohi[4]) shift by lohi[5] (between the last dropped id and
    // the next insertion point: the bulk of the ids when deletes and inserts cluster)
    uint32_t rlo = 0, rhi = 0, mlo = 0, mspan = 0;
    int32_t rsh = 0, msh = 0;
    if (REMAP) {
        rlo = (uint32_t)a.R.lohi[0]; rhi = (uint32_t)a.R.lohi[1]; rsh = a.R.lohi[2];
        mlo = (uint32_t)a.R.lohi[3]; mspan = (uint32_t)a.R.lohi[4] - mlo; msh = a.R.lohi[5];
    }

    uint64_t t = blockIdx.x;
    if (tid == 0) {
        mbar_init(&s_bar[0], 1); mbar_init(&s_bar[1], 1); fence_mbar_init();
        if (t < a.n_tiles) issue(t, 0, part[t], part[t + 1]);
        if (t + G < a.n_tiles) prefetch_part(t + G, 1);
    }
    if (tid < NCH + 2) { s_dmask[0][tid] = 0; s_icnt[0][tid] = 0; s_dmask[1][tid] = 0; s_icnt[1][tid] = 0; }
    __syncthreads();
    // heads of the edit lists of the tile in buffer bb (lists longer than kThreads are
    // read directly in the loops below)
    uint64_t pf_del = 0, pf_ins = 0, pf_upd = 0;
    uint32_t pf_icol = 0;
    float pf_iw = 0.f, pf_uw = 0.f;
    uint32_t pf_cm[4] = {0u, 0u, 0u, 0u};
    auto load_pos = [&](int bb) {
        const uint64_t r0 = s_meta[bb][0], r1 = s_meta[bb][1], dl0 = s_meta[bb][2];
        const uint32_t nd = (uint32_t)(s_meta[bb][4] & 0xFFFF);
        pf_del = tid < nd ? a.del_pos[dl0 + tid] : 0;
        pf_ins = tid < (uint32_t)(r1 - r0) ? a.ins_pos[r0 + tid] : 0;
    };
    auto load_upd = [&](int bb, uint64_t tt) {
        const uint64_t ul0 = s_meta[bb][3];
        const uint32_t nu = (uint32_t)((s_meta[bb][4] >> 16) & 0xFFFF);
        pf_upd = tid < nu ? a.upd_pos[ul0 + tid] : 0;
        pf_uw = tid < nu ? a.upd_w[ul0 + tid] : 0.f;
        if (CASC && wid == 0) {  // cascade-mask words under warp 0's two chunks
            const uint64_t j0 = min(tt * kMergeTile, Dtot) - s_meta[bb][0];
            const uint64_t n_old = min((tt + 1) * kMergeTile, Dtot) - s_meta[bb][1] - j0;
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const uint32_t i0 = (2 * lane + h) * 32;
                pf_cm[2 * h] = pf_cm[2 * h + 1] = 0u;
                if (i0 < n_old) {
                    const uint64_t x = j0 + i0, q = x >> 5;
                    pf_cm[2 * h] = a.casc_mask[q];
                    pf_cm[2 * h + 1] = (x & 31) ? a.casc_mask[q + 1] : 0u;
                }
            }
        }
    };
    auto load_ins = [&](int bb) {
        const uint64_t r0 = s_meta[bb][0], r1 = s_meta[bb][1];
        pf_icol = tid < (uint32_t)(r1 - r0) ? a.ins_col[r0 + tid] : 0u;
        pf_iw = tid < (uint32_t)(r1 - r0) ? a.ins_w[r0 + tid] : 0.f;
    };
    if (t < a.n_tiles) { load_pos(0); load_upd(0, t); load_ins(0); }

    for (uint32_t it = 0; t < a.n_tiles; t += G, ++it) {
        const int b = it & 1;
        const uint64_t r0 = s_meta[b][0], r1 = s_meta[b][1], dl0 = s_meta[b][2], ul0 = s_meta[b][3];
        const uint32_t nd = (uint32_t)(s_meta[b][4] & 0xFFFF), nu = (uint32_t)((s_meta[b][4] >> 16) & 0xFFFF);
        const uint64_t cbefore = CASC ? s_meta[b][5] : 0;  // cascaded old elements before j0
        const uint64_t d0 = min(t * kMergeTile, Dtot), d1 = min((t + 1) * kMergeTile, Dtot);
        const uint64_t j0 = d0 - r0, j1 = d1 - r1;
        const uint32_t n_old = (uint32_t)(j1 - j0), ni = (uint32_t)(r1 - r0);
        const uint32_t sh = (uint32_t)(j0 & 3);
        const bool has_next = t + G < a.n_tiles;
        if (tid == 0 && has_next) {
            cp_async_wait_all();
            const int slot = (it + 1) & 1;
            const TilePart p0 = s_tp[slot][0], p1 = s_tp[slot][1];
            fence_proxy_async();
            issue(t + G, b ^ 1, p0, p1);
            if (t + 2 * G < a.n_tiles) prefetch_part(t + 2 * G, it & 1);
        }
        uint32_t* dmask = s_dmask[b];
        uint32_t* icnt = s_icnt[b];
        for (uint32_t i = tid; i < nd; i += kThreads) {
            const uint32_t p = (uint32_t)((i == (uint32_t)tid ? pf_del : a.del_pos[dl0 + i]) - j0);
            atomicOr(&dmask[p >> 5], 1u << (p & 31));
        }
        for (uint32_t s = tid; s < ni; s += kThreads) {
            const uint32_t p = (uint32_t)((s == (uint32_t)tid ? pf_ins : a.ins_pos[r0 + s]) - j0);
            s_ins[s] = (uint16_t)p;
            atomicAdd(&icnt[p >> 5], 1u);
        }
        __syncthreads();  // B1: masks complete; s_meta[b ^ 1] (next tile) visible
        if (has_next) load_pos(b ^ 1);
        if (wid == 0) {
            // keep masks of the 64 chunks (2 per lane): valid & not deleted & not cascaded,
            // then exclusive scans of kept counts and of inserted-record counts
            uint32_t m[2], k[2];
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                const uint32_t c = 2 * lane + h, i0 = c * 32;
                uint32_t v = (i0 >= n_old) ? 0u : (n_old - i0 >= 32 ? 0xFFFFFFFFu : (0xFFFFFFFFu >> (32 - (n_old - i0))));
                v &= ~dmask[c];
                if (CASC && v) v &= ~__funnelshift_r(pf_cm[2 * h], pf_cm[2 * h + 1], (uint32_t)((j0 + i0) & 31));
                m[h] = v;
                k[h] = icnt[c];
            }
            const uint32_t c0 = __popc(m[0]), c1 = __popc(m[1]);
            const uint32_t inc = warp_inclusive_scan(c0 + c1);
            const uint32_t ik = warp_inclusive_scan(k[0] + k[1]);
            s_chunk[2 * lane] = make_uint4(m[0], inc - c0 - c1, ik - k[0] - k[1], k[0]);
            s_chunk[2 * lane + 1] = make_uint4(m[1], inc - c1, ik - k[1], k[1]);
            if (lane == 31) s_chunk[NCH] = make_uint4(0u, inc, ik, 0u);
        }
        mbar_wait(&s_bar[b], (it >> 1) & 1);
        // columns of this tile's old elements (warp w owns chunks w, w+8, ..., w+56) and
        // their remap, unrolled so that the table lookups are in flight together; warps
        // 1-7 do this while warp 0 builds the chunk table
        constexpr int KCH = NCH / (kThreads / 32);  // 8 chunks per warp
        uint32_t colv[KCH];
        auto load_cols = [&]() {
#pragma unroll
            for (int k = 0; k < KCH; ++k) {
                const uint32_t c = wid + k * (kThreads / 32), i = c * 32 + lane;
                colv[k] = (i < n_old) ? s_col[b][i + sh] : 0u;
            }
        };
        if (REMAP) {
            load_cols();
            // three constant-shift id ranges need no table; any other id reads its
            // 32-id group entry.  Branch-free: a constant-shift id gets the synthetic
            // entry {id + shift - r, no drops}, so every id evaluates the same
            // expression  base + r - popc(dropped below r)
            uint2 g[KCH];
#pragma unroll
            for (int k = 0; k < KCH; ++k) {
                const uint32_t col = colv[k];
                const bool tab = !(col < rlo || col >= rhi || col - mlo < mspan);
                const int32_t shf = col < rlo ? 0 : (col >= rhi ? rsh : msh);
                g[k] = tab ? a.R.g32[col >> 5] : make_uint2((uint32_t)((int32_t)(col & ~31u) + shf), 0u);
            }
#pragma unroll
            for (int k = 0; k < KCH; ++k) {
                const uint32_t col = colv[k], r = col & 31;
                colv[k] = (g[k].x & 0x7FFFFFFFu) + r - __popc(g[k].y & ((1u << r) - 1u));
                if (g[k].x >> 31)  // an insertion point strictly inside the group (rare)
                    colv[k] = remap_of_slow(a.R.shift, a.R.g32, a.R.ins_oldpos, a.R.n_vins, col);
            }
        }
        for (uint32_t i = tid; i < nu; i += kThreads) {
            const bool pf = i == (uint32_t)tid;
            s_w[b][(pf ? pf_upd : a.upd_pos[ul0 + i]) - (j0 & ~3ull)] = pf ? pf_uw : a.upd_w[ul0 + i];
        }
        if (tid == 0) bulk_wait_read0();  // previous tile's bulk store has finished reading s_oc/s_ow
        __syncthreads();  // B2: chunk table, updated weights, staging buffers free
        if (has_next) load_upd(b ^ 1, t + G);
        const uint32_t kept = s_chunk[NCH].y;
        const uint32_t n_out = kept + ni;
        const uint64_t base = j0 - dl0 - cbefore + r0;
        const uint32_t ob = (uint32_t)(base & 3);
        // phase B: place the kept old elements (columns remapped above)
        {
            if (!REMAP) load_cols();
#pragma unroll
            for (int k = 0; k < KCH; ++k) {
                const uint32_t c = wid + k * (kThreads / 32), i = c * 32 + lane;
                if (c * 32 >= n_old) break;
                const uint4 ch = s_chunk[c];
                uint32_t I = ch.z;
                if (ch.w) I = (uint32_t)upper_bound_dev(s_ins, ch.z, ch.z + ch.w, (uint16_t)i);  // inserts inside
                if (ch.x >> lane & 1) {
                    const uint32_t e = ch.y + __popc(ch.x & lt) + I + ob;
                    s_oc[e] = colv[k];
                    s_ow[e] = s_w[b][i + sh];
                }
            }
        }
        // inserted records: local position p precedes old element p
        for (uint32_t s = tid; s < ni; s += kThreads) {
            const uint32_t p = s_ins[s], c = p >> 5, r = p & 31;
            const uint4 ch = s_chunk[c];
            const uint32_t e = ch.y + (r ? __popc(ch.x & (0xFFFFFFFFu >> (32 - r))) : 0u) + s + ob;
            const bool pf = s == (uint32_t)tid;
            s_oc[e] = pf ? pf_icol : a.ins_col[r0 + s];
            s_ow[e] = pf ? pf_iw : a.ins_w[r0 + s];
        }
        __syncthreads();  // B3: staged output complete; this tile's inputs no longer read
        if (has_next) load_ins(b ^ 1);
        if (tid < NCH + 2) { dmask[tid] = 0; icnt[tid] = 0; }  // for tile t + 2G (same buffer)
        // store the contiguous output chunk [base, base + n_out)
        {
            uint32_t head = (4 - ob) & 3;
            if (head > n_out) head = n_out;
            const uint32_t body = ((n_out - head) >> 2) << 2;
            if (tid < head) { a.new_cols[base + tid] = s_oc[ob + tid]; a.new_w[base + tid] = s_ow[ob + tid]; }
            for (uint32_t e = head + body + tid; e < n_out; e += kThreads) {
                a.new_cols[base + e] = s_oc[ob + e];
                a.new_w[base + e] = s_ow[ob + e];
            }
            if (tid == 0) {
                if (body) {
                    fence_proxy_async();
                    bulk_s2g(a.new_cols + base + head, &s_oc[ob + head], body * 4);
                    bulk_s2g(a.new_w + base + head, &s_ow[ob + head], body * 4);
                }
                bulk_commit();
            }
        }
    }
    if (tid == 0) bulk_wait_all();
}






// Remap tables in one launch (thread t: the 64K-id block t, then the 32-id group t):
// per 64K-id block of old ids: constant new-id shift, or kRemapMixed if a dropped id or an
// inserted id's insertion point lies strictly inside the block.  Thread 0 also writes
// lohi = {lo, hi, shift}: below lo = min(first dropped id, first insertion point) nothing
// moves; from hi = max(last dropped id + 1, last insertion point) on, every id is shifted by
// n_ins - n_dropped.
// Per 32 old ids: {new id of the group's first id (as if it survived) | exact << 31, dropped
// bitmask}; exact = an insertion point lies strictly inside the group.  Only the groups of the
// 64K-id blocks overlapping [lo, hi) are written: every reader (k_merge3's table path,
// remap_of on a mixed 64K block) looks up ids there only.
__global__ void k_remap_tables(uint64_t V, const uint32_t* __restrict__ dropped, const uint32_t* __restrict__ ins_oldpos,
                               Counters* __restrict__ c, int32_t* __restrict__ shift, int32_t* __restrict__ lohi,
                               uint2* __restrict__ out) {
    const uint64_t n_dropped = c->n_dropped, n_ins = c->n_inserted;
    {
    uint64_t bk = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    uint64_t nb = (V + (1u << kRemapBlockShift) - 1) >> kRemapBlockShift;
    if (bk == 0) {
        const uint64_t lo = min(n_dropped ? (uint64_t)dropped[0] : V, n_ins ? (uint64_t)ins_oldpos[0] : V);
        const uint64_t hi = max(n_dropped ? (uint64_t)dropped[n_dropped - 1] + 1 : 0ull,
                                n_ins ? (uint64_t)ins_oldpos[n_ins - 1] : 0ull);
        lohi[0] = (int32_t)lo;
        lohi[1] = (int32_t)max(hi, lo);
        lohi[2] = (int32_t)((int64_t)n_ins - (int64_t)n_dropped);
        // [mlo, mhi): above the last dropped id, below the first insertion point past it
        const uint64_t mlo = n_dropped ? (uint64_t)dropped[n_dropped - 1] + 1 : 0ull;
        const uint64_t ci = upper_bound_dev(ins_oldpos, 0, n_ins, (uint32_t)mlo);  // insertion points <= mlo
        const uint64_t mhi = ci < n_ins ? (uint64_t)ins_oldpos[ci] : V;
        lohi[3] = (int32_t)mlo;
        lohi[4] = (int32_t)max(mhi, mlo);
        lohi[5] = (int32_t)((int64_t)ci - (int64_t)n_dropped);
        c->Vn = V - n_dropped + n_ins;  // vertices of the new ID map
    }
    if (bk < nb) {
        uint64_t lo = bk << kRemapBlockShift, hi = min(lo + (1u << kRemapBlockShift), V);
        uint64_t d0 = lower_bound_dev(dropped, 0, n_dropped, (uint32_t)lo);
        uint64_t d1 = lower_bound_dev(dropped, d0, n_dropped, (uint32_t)hi);
        uint64_t i0 = upper_bound_dev(ins_oldpos, 0, n_ins, (uint32_t)lo);      // oldpos <= lo
        uint64_t i1 = upper_bound_dev(ins_oldpos, i0, n_ins, (uint32_t)(hi - 1));  // oldpos <= hi-1
        shift[bk] = (d1 > d0 || i1 > i0) ? kRemapMixed : (int32_t)((int64_t)i0 - (int64_t)d0);
    }
    }

    // the CTA's id range narrows both sorted lists once (4 searches), then every group
    // searches only its CTA's slices (empty for most CTAs)
    __shared__ uint64_t s_rng[4];
    const uint64_t n_vins = n_ins, ng = (V + 31) / 32;
    const uint64_t gb = (uint64_t)blockIdx.x * blockDim.x;
    // [lo, hi) widened to whole 64K-id blocks: remap_of reads the groups of a mixed block
    constexpr uint64_t B = 1ull << kRemapBlockShift;
    // (lo, hi as thread 0 computes them for lohi[0], lohi[1] above)
    const uint64_t lo0 = min(n_dropped ? (uint64_t)dropped[0] : V, n_vins ? (uint64_t)ins_oldpos[0] : V);
    const uint64_t hi0 = max(max(n_dropped ? (uint64_t)dropped[n_dropped - 1] + 1 : (uint64_t)0,
                                 n_vins ? (uint64_t)ins_oldpos[n_vins - 1] : (uint64_t)0), lo0);
    const uint64_t lo = lo0 & ~(B - 1), hi = (hi0 + B - 1) & ~(B - 1);
    if ((gb + blockDim.x) * 32 <= lo || gb * 32 >= hi) return;  // CTA-uniform
    if (threadIdx.x < 4) {
        const uint64_t lo = gb * 32, hi = min((gb + blockDim.x) * 32, (uint64_t)0xFFFFFFFFull);
        const uint32_t x = (uint32_t)((threadIdx.x & 1) ? hi : lo);
        s_rng[threadIdx.x] = threadIdx.x < 2 ? lower_bound_dev(dropped, 0, n_dropped, x)
                                             : upper_bound_dev(ins_oldpos, 0, n_vins, x);
    }
    __syncthreads();
    const uint64_t g = gb + threadIdx.x;
    if (g >= ng) return;
    const uint32_t c0 = (uint32_t)(g * 32);
    const uint64_t d0 = lower_bound_dev(dropped, s_rng[0], s_rng[1], c0);
    const uint64_t i0 = upper_bound_dev(ins_oldpos, s_rng[2], s_rng[3], c0);
    // insertion points past the last old id (appended vertices) shift no old id
    const uint64_t i1 = upper_bound_dev(ins_oldpos, i0, s_rng[3], (uint32_t)min((uint64_t)c0 + 31, V - 1));
    uint32_t m = 0;
    for (uint64_t d = d0; d < s_rng[1] && dropped[d] < c0 + 32; ++d) m |= 1u << (dropped[d] - c0);
    out[g] = make_uint2((uint32_t)(c0 - d0 + i0) | (i1 > i0 ? 0x80000000u : 0u), m);
}

// After the survivor pass (node mode), one launch: the inserted vertices' row offsets (kept
// old elements before the old position they are inserted at, plus inserted records in rows <
// their new id), the fence of the new ID map (its size is a device count), and (thread 0,
// mark) the ID-map prefix bookkeeping
__global__ void k_rows_finish(const NodeVtx* __restrict__ nv, const uint32_t* __restrict__ ins_q, RowArgs a_,
                              const uint64_t* __restrict__ new_ext, uint64_t* __restrict__ fence,
                              unsigned long long* same, const int32_t* __restrict__ lohi, int tomb, int mark) {
    const RowArgs a = row_counts(a_);
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (mark && i == 0) {
        const unsigned long long lo = (unsigned long long)(uint32_t)lohi[0];
        Counters* c = const_cast<Counters*>(a.c);
        c->idmap_lo = lo;
        c->idmap_keep = tomb ? 0ull : min(same[0], lo);
        same[0] = min(same[0], lo);
        same[1] = lo;  // what the swap makes of same[0]
    }
    if (i < a.n_vins && a.own.owns(a.nv_ext[ins_q[i]])) {  // (another shard's row otherwise)
        const NodeVtx& r = nv[ins_q[i]];
        const uint64_t x = (uint64_t)a.old_off[r.oldpos];
        const uint64_t kept = x - casc_before(a, x) - lower_bound_dev(a.del_pos, 0, a.n_del, x);
        a.new_off[r.newid - a.row_lo_new] = (int64_t)(kept + lower_bound_dev(a.ins_row, 0, a.n_ins, r.newid));
    }
    if ((i << kFenceShift) < a.c->Vn) fence[i] = new_ext[i << kFenceShift];
}


// V == ~0: the vertex count of the new ID map is c->Vn (device-side)
__global__ void k_row_range(const uint64_t* __restrict__ ext, uint64_t V, OwnRange own, Counters* c) {
    if (V == ~0ull) V = c->Vn;
    c->row_lo_new = lower_bound_dev(ext, 0, V, own.lo);
    c->row_hi_new = own.hi == ~0ull ? V : lower_bound_dev(ext, 0, V, own.hi);
}
__global__ void k_copy_u64(unsigned long long* dst, const uint64_t* src) { *dst = *src; }

// End of an apply (one thread): sizes of the new replica from the device counters,
// the final row offset, and whether the new ID map is the identity 0..Vn-1 (ext ids
// strictly increase, so the last one decides).  node_mode: the ID map was rebuilt.
__global__ void k_finish(Counters* __restrict__ c, uint64_t V, uint64_t Vr, uint64_t E, int node_mode, int sharded,
                         const uint64_t* __restrict__ new_ext, int64_t* __restrict__ new_off) {
    const uint64_t Vn = node_mode ? (uint64_t)c->Vn : V;
    const uint64_t Vr_new = !node_mode ? Vr : (sharded ? (uint64_t)(c->row_hi_new - c->row_lo_new) : Vn);
    const uint64_t En = E + c->n_ins - c->n_del - c->n_casc;
    c->Vn = Vn;
    c->Vr_new = Vr_new;
    c->En = En;
    c->new_identity = node_mode ? (Vn == 0 || new_ext[Vn - 1] == Vn - 1) : 2;  // 2: unchanged
    if (new_off) new_off[Vr_new] = (int64_t)En;
}


// ================================================================ checks ====
template <typename T>
__global__ void k_checksum(const T* __restrict__ a, uint64_t n, uint64_t salt, unsigned long long* out) {
    uint64_t acc = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t bits;
        if (sizeof(T) == 4) bits = (uint64_t)(*reinterpret_cast<const uint32_t*>(&a[i]));
        else bits = *reinterpret_cast<const uint64_t*>(&a[i]);
        acc += sm64(bits ^ sm64(i ^ salt));
    }
    acc = warp_sum(acc);
    if (lane_id() == 0 && acc) atomicAdd(out, (unsigned long long)acc);
}

// create_from_csr validation: monotone offsets, strictly increasing rows, cols < V, ext increasing
__global__ void k_validate_csr(const int64_t* __restrict__ off, const uint32_t* __restrict__ cols, uint64_t V,
                               const uint64_t* __restrict__ ext, unsigned long long* bad) {
    for (uint64_t u = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; u < V; u += (uint64_t)gridDim.x * blockDim.x) {
        int64_t b = off[u], e = off[u + 1];
        bool ok = b <= e && (u > 0 || b == 0);
        if (ext && u > 0 && !(ext[u - 1] < ext[u])) ok = false;
        for (int64_t x = b; ok && x < e; ++x) {
            if (cols[x] >= V) ok = false;
            if (x > b && !(cols[x - 1] < cols[x])) ok = false;
        }
        if (!ok) atomicOr(bad, 1ull);
    }
}

__global__ void k_iota_u64(uint64_t* p, uint64_t n) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) p[i] = i;
}

// ---------------------------------------------------------------- BFS ----
__global__ void k_bfs_expand(const int64_t* __restrict__ off, const uint32_t* __restrict__ cols,
                             const uint32_t* __restrict__ front, uint64_t n_front, int32_t* __restrict__ level,
                             int32_t depth, uint32_t* __restrict__ next, unsigned long long* __restrict__ n_next) {
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t f = warp; f < n_front; f += nwarps) {
        uint32_t u = front[f];
        for (int64_t e = off[u] + lane_id(); e < off[u + 1]; e += 32) {
            uint32_t v = cols[e];
            bool claim = false;
            if (level[v] < 0) claim = atomicCAS(&level[v], -1, depth + 1) == -1;
            uint32_t m = __ballot_sync(__activemask(), claim);
            if (claim) {
                uint32_t leader = __ffs(m) - 1;
                unsigned long long b = 0;
                if (lane_id() == leader) b = atomicAdd(n_next, (unsigned long long)__popc(m));
                b = __shfl_sync(m, b, leader);
                next[b + __popc(m & lanemask_lt())] = v;
            }
        }
    }
}

// ------------------------------------------------------------------ SSSP ----
// Frontier Bellman-Ford (reading A21): distances are fp64 bit patterns; for
// non-negative doubles (and +inf) the unsigned order of the patterns is the numeric
// order, so a relaxation is one 64-bit atomicMin.  A vertex whose distance dropped
// joins the next frontier once per round (stamp).  With weights >= 0 the fixpoint
// d(v) = min over in-edges of fl(d(u) + w) is unique, so the result equals Dijkstra's
// bit for bit, whatever the relaxation order.
__global__ void k_sssp_check_w(const float* __restrict__ w, uint64_t E, unsigned int* __restrict__ bad) {
    bool b = false;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < E; i += (uint64_t)gridDim.x * blockDim.x) {
        const float x = w[i];
        b |= (x != x) || (x < 0.0f);  // NaN or negative (-0.0 passes)
    }
    if (__any_sync(0xffffffffu, b) && lane_id() == 0) atomicOr(bad, 1u);
}
__global__ void k_sssp_relax(const int64_t* __restrict__ off, const uint32_t* __restrict__ cols,
                             const float* __restrict__ w, const uint32_t* __restrict__ front, uint64_t n_front,
                             unsigned long long* dist, uint32_t* __restrict__ stamp, uint32_t round,
                             uint32_t* __restrict__ next, unsigned long long* __restrict__ n_next) {
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t f = warp; f < n_front; f += nwarps) {
        const uint32_t u = front[f];
        const double du = __longlong_as_double((long long)ld_volatile(reinterpret_cast<const uint64_t*>(dist + u)));
        for (int64_t e = off[u] + lane_id(); e < off[u + 1]; e += 32) {
            const uint32_t v = cols[e];
            const double nd = du + (double)w[e];
            const unsigned long long nb = (unsigned long long)__double_as_longlong(nd);
            bool push = false;
            if (nb < ld_volatile(reinterpret_cast<const uint64_t*>(dist + v)) && atomicMin(dist + v, nb) > nb)
                push = atomicExch(stamp + v, round) != round;
            const uint32_t m = __ballot_sync(__activemask(), push);
            if (push) {
                const uint32_t leader = __ffs(m) - 1;
                unsigned long long b = 0;
                if (lane_id() == leader) b = atomicAdd(n_next, (unsigned long long)__popc(m));
                b = __shfl_sync(m, b, leader);
                next[b + __popc(m & lanemask_lt())] = v;
            }
        }
    }
}

__global__ void k_fill_i32(int32_t* p, uint64_t n, int32_t v) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) p[i] = v;
}

// ---------------------------------------------- checks on a sharded replica ----
// (SURVEY.md §8(e) "Checks").  Global per-vertex arrays (every shard keeps the whole ID
// map, so dense ids are global); each shard touches the rows it owns (local offsets,
// global row = row_lo + i) and the caller combines the shards with a collective
// (MAX of the BFS marks, SUM of the PageRank contributions, MIN of the distances).
__global__ void k_shard_bfs_expand(const int64_t* __restrict__ off, const uint32_t* __restrict__ cols, uint64_t Vr,
                                   uint64_t row_lo, const int32_t* __restrict__ level, int32_t depth,
                                   uint8_t* __restrict__ mark) {
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t i = warp; i < Vr; i += nwarps) {
        if (level[row_lo + i] != depth) continue;
        for (int64_t e = off[i] + lane_id(); e < off[i + 1]; e += 32) {
            const uint32_t v = cols[e];
            if (level[v] < 0) mark[v] = 1;
        }
    }
}
__global__ void k_shard_bfs_settle(int32_t* __restrict__ level, const uint8_t* __restrict__ mark, uint64_t V,
                                   int32_t depth, unsigned long long* __restrict__ n_new) {
    const uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    bool nw = false;
    if (v < V && mark[v] && level[v] < 0) { level[v] = depth + 1; nw = true; }
    const uint32_t m = __ballot_sync(0xffffffffu, nw);
    if (lane_id() == 0 && m) atomicAdd(n_new, (unsigned long long)__popc(m));
}
__global__ void k_shard_pr_push(const int64_t* __restrict__ off, const uint32_t* __restrict__ cols, uint64_t Vr,
                                uint64_t row_lo, const double* __restrict__ pr, double* __restrict__ acc,
                                double* __restrict__ dangling) {
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t i = warp; i < Vr; i += nwarps) {
        const int64_t b = off[i], e = off[i + 1];
        const double p = pr[row_lo + i];
        if (b == e) { if (lane_id() == 0) atomicAdd(dangling, p); continue; }
        const double c = p / (double)(e - b);
        for (int64_t x = b + lane_id(); x < e; x += 32) atomicAdd(&acc[cols[x]], c);
    }
}
__global__ void k_shard_pr_finish(double* __restrict__ nxt, uint64_t V, double d, const double* __restrict__ dsum) {
    const uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (v < V) nxt[v] = (1.0 - d) / (double)V + d * (nxt[v] + *dsum / (double)V);
}
__global__ void k_shard_sssp_relax(const int64_t* __restrict__ off, const uint32_t* __restrict__ cols,
                                   const float* __restrict__ w, uint64_t Vr, uint64_t row_lo,
                                   const uint8_t* __restrict__ frontier, const double* __restrict__ dist,
                                   unsigned long long* nd) {
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t i = warp; i < Vr; i += nwarps) {
        if (!frontier[row_lo + i]) continue;
        const double du = dist[row_lo + i];
        for (int64_t e = off[i] + lane_id(); e < off[i + 1]; e += 32) {
            const unsigned long long b = (unsigned long long)__double_as_longlong(du + (double)w[e]);
            if (b < ld_volatile(reinterpret_cast<const uint64_t*>(nd + cols[e]))) atomicMin(nd + cols[e], b);
        }
    }
}
__global__ void k_shard_sssp_settle(double* __restrict__ dist, const double* __restrict__ nd, uint8_t* __restrict__ frontier,
                                    uint64_t V, unsigned long long* __restrict__ n_changed) {
    const uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    bool ch = false;
    if (v < V) {
        ch = nd[v] < dist[v];
        frontier[v] = ch ? 1 : 0;
        if (ch) dist[v] = nd[v];
    }
    const uint32_t m = __ballot_sync(0xffffffffu, ch);
    if (lane_id() == 0 && m) atomicAdd(n_changed, (unsigned long long)__popc(m));
}

// ---------------------------------------------------------- PageRank ----
// live (nullable, tombstone mode): PageRank of the live subgraph, nl = live vertices;
// a tombstoned vertex has no edges and rank 0
__global__ void k_pr_init(double* pr, uint64_t n, const uint8_t* __restrict__ live, uint64_t nl) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) pr[i] = (!live || live[i]) ? 1.0 / (double)nl : 0.0;
}
__global__ void k_pr_dangling(const int64_t* __restrict__ off, const double* __restrict__ pr, uint64_t n, double* out) {
    double acc = 0;
    for (uint64_t u = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; u < n; u += (uint64_t)gridDim.x * blockDim.x)
        if (off[u + 1] == off[u]) acc += pr[u];  // tombstones hold 0
    acc = warp_sum(acc);
    if (lane_id() == 0 && acc != 0.0) atomicAdd(out, acc);
}
__global__ void k_pr_push(const int64_t* __restrict__ off, const uint32_t* __restrict__ cols,
                          const double* __restrict__ pr, uint64_t n, double* __restrict__ nxt) {
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t u = warp; u < n; u += nwarps) {
        int64_t b = off[u], e = off[u + 1];
        if (b == e) continue;
        double c = pr[u] / (double)(e - b);
        for (int64_t x = b + lane_id(); x < e; x += 32) atomicAdd(&nxt[cols[x]], c);
    }
}
__global__ void k_pr_finish(double* __restrict__ nxt, uint64_t n, double d, const double* __restrict__ dsum,
                            const uint8_t* __restrict__ live, uint64_t nl) {
    uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (v < n) nxt[v] = (!live || live[v]) ? (1.0 - d) / (double)nl + d * (nxt[v] + *dsum / (double)nl) : 0.0;
}
__global__ void k_count_u8(const uint8_t* __restrict__ x, uint64_t n, unsigned long long* __restrict__ out) {
    unsigned long long acc = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        acc += x[i] ? 1 : 0;
    acc = warp_sum(acc);
    if (lane_id() == 0 && acc) atomicAdd(out, acc);
}

}  // namespace h2tap
