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
enum : uint64_t { ST_BAD_KIND = 1, ST_STALE = 2, ST_CREATE_ENDPOINT = 4 };

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
    unsigned int tiles[16];
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
enum : uint32_t { NV_FINAL = 1, NV_HASD = 2, NV_OLD = 4 };

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
            if (cat[j] < 3) cnt[cat[j]]++;
        }
    }
    if (bad) atomicOr(&c->status, (unsigned long long)bad);
    if (tmin != ~0ull) {
        atomicMin(&c->ts_min, tmin); atomicMax(&c->ts_max, tmax);
        atomicMin(&c->v_min, vmin); atomicMax(&c->v_max, vmax);
    }
    uint64_t excl[3], tot[3];
#pragma unroll
    for (int q = 0; q < 3; ++q) excl[q] = block_exclusive_scan<kThreads>(cnt[q], s_scan, &tot[q]);
    const int wid = threadIdx.x >> 5;
    if (wid < 3) {
        uint64_t b = lookback_warp(status3 + (uint64_t)wid * n_tiles, tile, tot[wid]);
        if (lane_id() == 0) {
            s_base[wid] = b;
            if (tile == n_tiles - 1) {
                unsigned long long* dst = wid == 0 ? &c->n_pend : (wid == 1 ? &c->n_node : &c->n_edge);
                *dst = b + tot[wid];
            }
        }
    }
    __syncthreads();
    uint64_t o[3] = {s_base[0] + excl[0], s_base[1] + excl[1], s_base[2] + excl[2]};
    uint32_t* outs[3] = {pend_idx, node_idx, edge_idx};
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        if (cat[j] < 3) outs[cat[j]][o[cat[j]]++] = (uint32_t)(i0 + j);
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

// old dense index of external id x (identity fast path or binary search)
__device__ __forceinline__ uint64_t old_lookup(const uint64_t* ext, uint64_t V, bool identity, uint64_t x,
                                               bool* present) {
    if (identity) { *present = x < V; return x < V ? x : V; }
    uint64_t k = lower_bound_dev(ext, 0, V, x);
    *present = (k < V && ext[k] == x);
    return k;
}

// ===================================================================== a2 ====
// Unique vertices of the (v, ts, seq)-sorted visible node ops: final liveness
// (last op), latest delete point tD, old presence.  Compaction via look-back.
__global__ void __launch_bounds__(kThreads) k_node_segments(
    Ops ops, const uint32_t* __restrict__ sidx, uint64_t n, const uint64_t* __restrict__ old_ext,
    uint64_t V, int identity, NodeVtx* __restrict__ nv, uint64_t* __restrict__ nv_ext,
    uint64_t* __restrict__ status, uint64_t n_tiles, Counters* __restrict__ c) {
    __shared__ uint32_t s_tile;
    __shared__ uint64_t s_scan[kThreads / 32 + 1];
    __shared__ uint64_t s_base;
    if (threadIdx.x == 0) s_tile = atomicAdd(&c->tiles[1], 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t i0 = (uint64_t)tile * kTile + (uint64_t)threadIdx.x * kItems;
    uint64_t heads = 0;
    uint32_t hmask = 0;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        uint64_t i = i0 + j;
        if (i < n && (i == 0 || ops.src[sidx[i]] != ops.src[sidx[i - 1]])) { hmask |= 1u << j; heads++; }
    }
    uint64_t tot, excl = block_exclusive_scan<kThreads>(heads, s_scan, &tot);
    if (threadIdx.x < 32) {
        uint64_t b = lookback_warp(status, tile, tot);
        if (lane_id() == 0) { s_base = b; if (tile == n_tiles - 1) c->n_unique = b + tot; }
    }
    __syncthreads();
    uint64_t q = s_base + excl;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        if (!(hmask >> j & 1)) continue;
        uint64_t i = i0 + j;
        uint64_t v = ops.src[sidx[i]];
        uint64_t e = i;
        NodeVtx r;
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
        uint64_t k = old_lookup(old_ext, V, identity, v, &present);
        if (present) r.flags |= NV_OLD;
        r.oldpos = (uint32_t)k;
        r.start = (uint32_t)i;
        r.end = (uint32_t)e;
        r.newid = kNone32;
        r.pad = 0;
        nv[q] = r;
        nv_ext[q] = v;
        ++q;
    }
}

// dropped (old-live -> dead), inserted (new & finally live), hd (old-present with a delete)
__global__ void __launch_bounds__(kThreads) k_node_lists(
    const NodeVtx* __restrict__ nv, uint64_t U, uint32_t* __restrict__ dropped,
    uint32_t* __restrict__ ins_q, uint32_t* __restrict__ ins_oldpos, uint32_t* __restrict__ hd_rows,
    uint64_t* __restrict__ status3, uint64_t n_tiles, Counters* __restrict__ c) {
    __shared__ uint32_t s_tile;
    __shared__ uint64_t s_scan[kThreads / 32 + 1];
    __shared__ uint64_t s_base[3];
    if (threadIdx.x == 0) s_tile = atomicAdd(&c->tiles[2], 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t i0 = (uint64_t)tile * kTile + (uint64_t)threadIdx.x * kItems;
    uint64_t cnt[3] = {0, 0, 0};
    uint32_t fl[kItems];
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        uint64_t i = i0 + j;
        fl[j] = 0;
        if (i < U) {
            uint32_t f = nv[i].flags;
            bool old = f & NV_OLD, fin = f & NV_FINAL, hd = f & NV_HASD;
            if (old && !fin) { fl[j] |= 1; cnt[0]++; }
            if (!old && fin) { fl[j] |= 2; cnt[1]++; }
            if (old && hd) { fl[j] |= 4; cnt[2]++; }
        }
    }
    uint64_t excl[3], tot[3];
#pragma unroll
    for (int q = 0; q < 3; ++q) excl[q] = block_exclusive_scan<kThreads>(cnt[q], s_scan, &tot[q]);
    const int wid = threadIdx.x >> 5;
    if (wid < 3) {
        uint64_t b = lookback_warp(status3 + (uint64_t)wid * n_tiles, tile, tot[wid]);
        if (lane_id() == 0) {
            s_base[wid] = b;
            if (tile == n_tiles - 1) {
                unsigned long long* d = wid == 0 ? &c->n_dropped : (wid == 1 ? &c->n_inserted : &c->n_hd);
                *d = b + tot[wid];
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
        if (fl[j] & 4) hd_rows[o2++] = nv[i].oldpos;
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

// ID-map compaction (reading A9): remap[k] = new dense id of old vertex k or
// kNone32 (dropped); new_ext[remap[k]] = ext[k].  Survivor rank minus dropped
// before plus inserted (by old position) at or before.
__global__ void __launch_bounds__(kThreads) k_remap(
    const uint64_t* __restrict__ old_ext, int identity, uint64_t V, const uint32_t* __restrict__ dropped,
    uint64_t n_dropped, const uint32_t* __restrict__ ins_oldpos, uint64_t n_ins,
    uint32_t* __restrict__ remap, uint64_t* __restrict__ new_ext) {
    uint64_t k0 = ((uint64_t)blockIdx.x * kThreads + threadIdx.x) * kItems;
    if (k0 >= V) return;
    uint64_t dp = lower_bound_dev(dropped, 0, n_dropped, (uint32_t)k0);
    uint64_t ip = lower_bound_dev(ins_oldpos, 0, n_ins, (uint32_t)k0);
    for (int j = 0; j < kItems; ++j) {
        uint64_t k = k0 + j;
        if (k >= V) break;
        dp = gallop_lb(dropped, dp, n_dropped, (uint32_t)k);
        ip = gallop_ub(ins_oldpos, ip, n_ins, (uint32_t)k);
        bool is_dropped = dp < n_dropped && dropped[dp] == (uint32_t)k;
        uint32_t r = is_dropped ? kNone32 : (uint32_t)(k - dp + ip);
        remap[k] = r;
        if (!is_dropped) new_ext[r] = identity ? k : old_ext[k];
    }
}

// inserted vertex i lands at oldpos_i - (#dropped before oldpos_i) + i
__global__ void k_place_inserted(NodeVtx* __restrict__ nv, const uint64_t* __restrict__ nv_ext,
                                 const uint32_t* __restrict__ ins_q, const uint32_t* __restrict__ ins_oldpos,
                                 uint64_t n_ins, const uint32_t* __restrict__ dropped, uint64_t n_dropped,
                                 uint64_t* __restrict__ new_ext) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n_ins) return;
    uint32_t op = ins_oldpos[i];
    uint64_t pos = op - lower_bound_dev(dropped, 0, n_dropped, op) + i;
    new_ext[pos] = nv_ext[ins_q[i]];
    nv[ins_q[i]].newid = (uint32_t)pos;
}

// new ids of surviving old vertices that have node ops
__global__ void k_nv_newid(NodeVtx* __restrict__ nv, uint64_t U, const uint32_t* __restrict__ remap, int has_remap) {
    uint64_t q = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (q >= U) return;
    uint32_t f = nv[q].flags;
    if ((f & NV_OLD) && (f & NV_FINAL)) nv[q].newid = has_remap ? remap[nv[q].oldpos] : nv[q].oldpos;
}

__global__ void k_set_bits(const uint32_t* __restrict__ rows, uint64_t n, uint32_t* __restrict__ bits) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) atomicOr(&bits[rows[i] >> 5], 1u << (rows[i] & 31));
}

// ===================================================================== a3 ====
struct Lookup {
    int64_t q;        // index in the node-vertex list or -1
    uint32_t oldpos;  // old dense index (present) or insertion rank
    uint32_t newid;
    bool old_present, final_live, hasD;
    uint64_t tD_ts, tD_seq;
};

struct PrepArgs {
    Ops ops;
    const uint32_t* edge_idx;
    uint64_t n_edge;
    const uint64_t* old_ext;
    uint64_t V;
    int identity;
    const uint32_t* remap;  // nullable (identity remap)
    const NodeVtx* nv;
    const uint64_t* nv_ext;
    uint64_t U;
    const uint32_t* node_sorted;  // (v, ts, seq)-sorted node op indices
    int bits;                     // bits of a dense id in the packed key
    int create;                   // create_from_edges: endpoints must exist
    uint64_t* keys;
    uint32_t* vals;
    uint8_t* op_flags;            // per W index: bit0 u old-present, bit1 w old-present, bit2 key had node delete
    uint32_t* op_opos_u;
    uint32_t* op_opos_w;
    uint64_t* status;
    uint64_t n_tiles;
    Counters* c;
};

__device__ __forceinline__ Lookup do_lookup(const PrepArgs& a, uint64_t x) {
    Lookup L;
    L.q = -1;
    L.hasD = false;
    L.tD_ts = 0; L.tD_seq = 0;
    if (a.U) {
        uint64_t q = lower_bound_dev(a.nv_ext, 0, a.U, x);
        if (q < a.U && a.nv_ext[q] == x) {
            const NodeVtx& r = a.nv[q];
            L.q = (int64_t)q;
            L.oldpos = r.oldpos;
            L.newid = r.newid;
            L.old_present = r.flags & NV_OLD;
            L.final_live = r.flags & NV_FINAL;
            L.hasD = r.flags & NV_HASD;
            L.tD_ts = r.tD_ts; L.tD_seq = r.tD_seq;
            return L;
        }
    }
    bool present;
    uint64_t k = old_lookup(a.old_ext, a.V, a.identity, x, &present);
    L.oldpos = (uint32_t)k;
    L.old_present = present;
    L.final_live = present;
    L.newid = present ? (a.remap ? a.remap[k] : (uint32_t)k) : kNone32;
    return L;
}

// liveness of a vertex with node ops just before point (ts, seq) (reading A13)
__device__ __forceinline__ bool live_at(const PrepArgs& a, const Lookup& L, uint64_t ts, uint64_t seq) {
    if (L.q < 0) return L.old_present;
    const NodeVtx& r = a.nv[L.q];
    uint64_t lo = r.start, hi = r.end;  // first node op with point >= p
    while (lo < hi) {
        uint64_t mid = (lo + hi) >> 1;
        uint32_t o = a.node_sorted[mid];
        if (pt_less(a.ops.ts[o], a.ops.seq[o], ts, seq)) lo = mid + 1; else hi = mid;
    }
    if (lo == r.start) return L.old_present;
    return a.ops.kind[a.node_sorted[lo - 1]] == NODE_INSERT;
}

// Per visible edge op: endpoint lookups, liveness gating and node-delete
// supersession (order-free form of the replay), packed key
// (src' << bits | dst'), compaction of surviving ops via look-back.
__global__ void __launch_bounds__(kThreads) k_edge_prep(PrepArgs a) {
    __shared__ uint32_t s_tile;
    __shared__ uint64_t s_scan[kThreads / 32 + 1];
    __shared__ uint64_t s_base;
    if (threadIdx.x == 0) s_tile = atomicAdd(&a.c->tiles[3], 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t i0 = (uint64_t)tile * kTile + (uint64_t)threadIdx.x * kItems;
    uint64_t key[kItems];
    uint32_t valid = 0;
    uint64_t nvalid = 0, ngated = 0, nbad = 0;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        uint64_t i = i0 + j;
        key[j] = 0;
        if (i >= a.n_edge) continue;
        uint32_t o = a.edge_idx[i];
        uint8_t kind = a.ops.kind[o];
        uint64_t ts = a.ops.ts[o], seq = a.ops.seq[o];
        Lookup Lu = do_lookup(a, a.ops.src[o]);
        Lookup Lw = do_lookup(a, a.ops.dst[o]);
        bool ok = Lu.final_live && Lw.final_live;
        if (a.create && !(Lu.old_present && Lw.old_present)) nbad++;
        if (ok && (Lu.hasD || Lw.hasD)) {
            // superseded by a later node delete of an endpoint (A8)
            if (Lu.hasD && pt_less(ts, seq, Lu.tD_ts, Lu.tD_seq)) ok = false;
            if (Lw.hasD && pt_less(ts, seq, Lw.tD_ts, Lw.tD_seq)) ok = false;
        }
        if (ok && kind != EDGE_DELETE && (Lu.q >= 0 || Lw.q >= 0)) {
            if (!live_at(a, Lu, ts, seq) || !live_at(a, Lw, ts, seq)) ok = false;
        }
        if (ok) {
            valid |= 1u << j;
            nvalid++;
            key[j] = ((uint64_t)Lu.newid << a.bits) | (uint64_t)Lw.newid;
            a.op_flags[o] = (uint8_t)((Lu.old_present ? 1 : 0) | (Lw.old_present ? 2 : 0) |
                                      ((Lu.hasD || Lw.hasD) ? 4 : 0));
            a.op_opos_u[o] = Lu.oldpos;
            a.op_opos_w[o] = Lw.oldpos;
        } else {
            ngated++;
        }
    }
    uint64_t gsum = warp_sum(ngated);
    if (lane_id() == 0 && gsum) atomicAdd(&a.c->n_gated, (unsigned long long)gsum);
    uint64_t bsum = warp_sum(nbad);
    if (lane_id() == 0 && bsum) atomicOr(&a.c->status, (unsigned long long)ST_CREATE_ENDPOINT);
    uint64_t tot, excl = block_exclusive_scan<kThreads>(nvalid, s_scan, &tot);
    if (threadIdx.x < 32) {
        uint64_t b = lookback_warp(a.status, tile, tot);
        if (lane_id() == 0) { s_base = b; if (tile == a.n_tiles - 1) a.c->n_valid = b + tot; }
    }
    __syncthreads();
    uint64_t p = s_base + excl;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        if (valid >> j & 1) { a.keys[p] = key[j]; a.vals[p] = a.edge_idx[i0 + j]; ++p; }
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
    const uint8_t* op_flags;
    const uint32_t* op_opos_u;
    const uint32_t* op_opos_w;
    const int64_t* old_off;
    const uint32_t* old_cols;
    uint64_t* ins_pos;
    uint32_t* ins_row;
    uint32_t* ins_col;
    float* ins_w;
    uint64_t* del_pos;
    uint64_t* upd_pos;
    float* upd_w;
    uint64_t* status3;
    uint64_t n_tiles;
    Counters* c;
};

__global__ void __launch_bounds__(kThreads) k_reduce_classify(ClassArgs a) {
    __shared__ uint32_t s_tile;
    __shared__ uint64_t s_scan[kThreads / 32 + 1];
    __shared__ uint64_t s_base[3];
    if (threadIdx.x == 0) s_tile = atomicAdd(&a.c->tiles[4], 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t i0 = (uint64_t)tile * kTile + (uint64_t)threadIdx.x * kItems;
    uint8_t cat[kItems];
    uint64_t pos[kItems];
    float wv[kItems];
    uint64_t cnt[3] = {0, 0, 0};
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        cat[j] = 0;
        uint64_t i = i0 + j;
        if (i >= a.n) continue;
        uint64_t key = a.keys[i];
        if (i > 0 && a.keys[i - 1] == key) continue;
        // segment [i, e)
        uint64_t nw_ts = 0, nw_seq = 0, w_ts = 0, w_seq = 0;
        bool has_nw = false, has_w = false;
        uint8_t nw_kind = 0;
        float w_val = 0.f;
        for (uint64_t e = i; e < a.n && a.keys[e] == key; ++e) {
            uint32_t o = a.vals[e];
            uint8_t k = a.ops.kind[o];
            uint64_t ts = a.ops.ts[o], sq = a.ops.seq[o];
            if (k == EDGE_INSERT || k == EDGE_DELETE) {
                if (!has_nw || pt_less(nw_ts, nw_seq, ts, sq)) { has_nw = true; nw_ts = ts; nw_seq = sq; nw_kind = k; }
            }
            if (k == EDGE_INSERT || k == EDGE_WEIGHT) {
                if (!has_w || pt_less(w_ts, w_seq, ts, sq)) { has_w = true; w_ts = ts; w_seq = sq; w_val = a.ops.w[o]; }
            }
        }
        uint32_t o0 = a.vals[i];
        uint8_t fl = a.op_flags[o0];
        bool u_old = fl & 1, w_old = fl & 2, hd = fl & 4;
        uint32_t ou = a.op_opos_u[o0], ow = a.op_opos_w[o0];
        uint64_t p;
        bool found = false;
        if (u_old) {
            uint64_t beg = (uint64_t)a.old_off[ou], end = (uint64_t)a.old_off[ou + 1];
            p = lower_bound_dev(a.old_cols, beg, end, ow);
            found = w_old && p < end && a.old_cols[p] == ow;
        } else {
            p = (uint64_t)a.old_off[ou];
        }
        bool present = found && !hd;  // a node delete of an endpoint cleared the old edge
        uint8_t ct = 0;
        if (has_nw && nw_kind == EDGE_INSERT) ct = present ? 3 : 1;
        else if (has_nw && nw_kind == EDGE_DELETE) ct = present ? 2 : 0;
        else if (has_w) ct = present ? 3 : 0;
        cat[j] = ct;
        pos[j] = p;
        wv[j] = w_val;
        if (ct) cnt[ct - 1]++;
    }
    uint64_t excl[3], tot[3];
#pragma unroll
    for (int q = 0; q < 3; ++q) excl[q] = block_exclusive_scan<kThreads>(cnt[q], s_scan, &tot[q]);
    const int wid = threadIdx.x >> 5;
    if (wid < 3) {
        uint64_t b = lookback_warp(a.status3 + (uint64_t)wid * a.n_tiles, tile, tot[wid]);
        if (lane_id() == 0) {
            s_base[wid] = b;
            if (tile == a.n_tiles - 1) {
                unsigned long long* d = wid == 0 ? &a.c->n_ins : (wid == 1 ? &a.c->n_del : &a.c->n_upd);
                *d = b + tot[wid];
            }
        }
    }
    __syncthreads();
    uint64_t oi = s_base[0] + excl[0], od = s_base[1] + excl[1], ou = s_base[2] + excl[2];
    const uint64_t mask = (1ull << a.bits) - 1;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        if (cat[j] == 1) {
            uint64_t key = a.keys[i0 + j];
            a.ins_pos[oi] = pos[j];
            a.ins_row[oi] = (uint32_t)(key >> a.bits);
            a.ins_col[oi] = (uint32_t)(key & mask);
            a.ins_w[oi] = wv[j];
            ++oi;
        } else if (cat[j] == 2) {
            a.del_pos[od++] = pos[j];
        } else if (cat[j] == 3) {
            a.upd_pos[ou] = pos[j];
            a.upd_w[ou] = wv[j];
            ++ou;
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
constexpr int kMergeItems = 8;
constexpr int kMergeTile = kThreads * kMergeItems;  // 2048 merged items per CTA

struct MergeArgs {
    const uint32_t* old_cols;
    const float* old_w;
    const int64_t* old_off;
    uint64_t E_old, V_old;
    const uint64_t* ins_pos;
    const uint32_t* ins_col;
    const float* ins_w;
    uint64_t n_ins;
    const uint64_t* del_pos;
    uint64_t n_del;
    const uint64_t* upd_pos;
    const float* upd_w;
    uint64_t n_upd;
    const uint32_t* remap;
    const uint32_t* hd_bits;
    const uint32_t* hd_rows;
    uint64_t n_hd;
    uint32_t* new_cols;
    float* new_w;
    int64_t* KR;  // CASC: kept elements before each old row start, [V_old + 1]
    uint64_t* status;
    uint64_t n_tiles;
    Counters* c;
};

// smallest r with ins_pos[r] + r >= d  (number of inserted records among the first d merged items)
__device__ __forceinline__ uint64_t ins_split(const uint64_t* ins_pos, uint64_t n_ins, uint64_t d) {
    uint64_t lo = 0, hi = n_ins;
    while (lo < hi) {
        uint64_t mid = (lo + hi) >> 1;
        if (ins_pos[mid] + mid < d) lo = mid + 1; else hi = mid;
    }
    return lo;
}

template <bool CASC, bool REMAP>
__global__ void __launch_bounds__(kThreads) k_merge(MergeArgs a) {
    __shared__ __align__(16) uint32_t s_col[kMergeTile + 8];
    __shared__ __align__(16) float s_w[kMergeTile + 8];
    __shared__ uint32_t s_slot[kMergeTile + 1];
    __shared__ uint32_t s_oc[kMergeTile];
    __shared__ float s_ow[kMergeTile];
    __shared__ uint8_t s_keep[kMergeTile];
    // kept-before per old element (CASC); aliases s_slot, which is dead once the
    // blocked pass has loaded it into registers (two block scans = barriers in between)
    uint32_t* const s_kp = s_slot;
    __shared__ uint64_t s_scan[kThreads / 32 + 1];
    __shared__ uint64_t s_r[2], s_d[2], s_u[2], s_h[2], s_base;
    __shared__ uint32_t s_tile;

    const int tid = threadIdx.x;
    if (tid == 0) s_tile = CASC ? atomicAdd(&a.c->tiles[5], 1u) : blockIdx.x;
    __syncthreads();
    const uint64_t tile = s_tile;
    const uint64_t Dtot = a.E_old + a.n_ins;
    const uint64_t d0 = tile * kMergeTile;
    const uint64_t d1 = min(d0 + (uint64_t)kMergeTile, Dtot);
    if (tid < 2) {
        uint64_t d = tid == 0 ? d0 : d1;
        s_r[tid] = (d == Dtot) ? a.n_ins : ins_split(a.ins_pos, a.n_ins, d);
    }
    __syncthreads();
    const uint64_t r0 = s_r[0], r1 = s_r[1];
    const uint64_t j0 = d0 - r0, j1 = d1 - r1;
    const uint32_t n_old = (uint32_t)(j1 - j0), n_new = (uint32_t)(r1 - r0), n_tot = n_old + n_new;
    if (tid < 2) {
        uint64_t j = tid == 0 ? j0 : j1;
        s_d[tid] = lower_bound_dev(a.del_pos, 0, a.n_del, j);
        s_u[tid] = lower_bound_dev(a.upd_pos, 0, a.n_upd, j);
    }
    if (CASC && tid >= 32 && tid < 34) {
        // hd rows whose row range [off[k], off[k+1]) intersects [j0, j1)
        const int which = tid - 32;
        uint64_t lo = 0, hi = a.n_hd;
        if (which == 0) {  // first hd row with end > j0
            while (lo < hi) { uint64_t mid = (lo + hi) >> 1; if ((uint64_t)a.old_off[a.hd_rows[mid] + 1] <= j0) lo = mid + 1; else hi = mid; }
        } else {           // first hd row with start >= j1
            while (lo < hi) { uint64_t mid = (lo + hi) >> 1; if ((uint64_t)a.old_off[a.hd_rows[mid]] < j1) lo = mid + 1; else hi = mid; }
        }
        s_h[which] = lo;
    }
    // stage old elements [j0, j1) (aligned 16 B chunks; buffers are padded)
    const uint64_t a0 = j0 & ~3ull;
    {
        const uint64_t c0 = a0 >> 2, c1 = (j1 + 3) >> 2;
        const uint4* gc = reinterpret_cast<const uint4*>(a.old_cols);
        const uint4* gw = reinterpret_cast<const uint4*>(a.old_w);
        for (uint64_t q = c0 + tid; q < c1; q += kThreads) {
            uint4 vc = gc[q], vw = gw[q];
            uint32_t o = (uint32_t)((q << 2) - a0);
            *reinterpret_cast<uint4*>(&s_col[o]) = vc;
            *reinterpret_cast<uint4*>(&s_w[o]) = vw;
        }
    }
    for (uint32_t i = tid; i < kMergeTile; i += kThreads) { s_keep[i] = 1; s_slot[i] = 0; }
    __syncthreads();
    const uint32_t sh = (uint32_t)(j0 - a0);
    // deletes and weight overrides (sorted old positions in [j0, j1))
    for (uint64_t i = s_d[0] + tid; i < s_d[1]; i += kThreads) s_keep[a.del_pos[i] - j0] = 0;
    for (uint64_t i = s_u[0] + tid; i < s_u[1]; i += kThreads) s_w[a.upd_pos[i] - a0] = a.upd_w[i];
    if (CASC) {
        for (uint64_t h = s_h[0]; h < s_h[1]; ++h) {
            uint32_t k = a.hd_rows[h];
            uint64_t b = max((uint64_t)a.old_off[k], j0), e = min((uint64_t)a.old_off[k + 1], j1);
            for (uint64_t x = b + tid; x < e; x += kThreads) s_keep[x - j0] = 0;
        }
    }
    for (uint32_t s = tid; s < n_new; s += kThreads) {
        uint64_t m = (a.ins_pos[r0 + s] - j0) + s;
        s_slot[m] = 0x80000000u | s;
    }
    __syncthreads();
    if (CASC) {
        for (uint32_t i = tid; i < n_old; i += kThreads) {
            if (s_keep[i]) {
                uint32_t col = s_col[i + sh];
                if (a.hd_bits[col >> 5] >> (col & 31) & 1) s_keep[i] = 0;
            }
        }
        __syncthreads();
    }
    // blocked pass over merged slots: old-element index, emit flag, output index
    const uint32_t m0 = tid * kMergeItems;
    uint32_t slot[kMergeItems];
    uint64_t n_oldc = 0;
#pragma unroll
    for (int j = 0; j < kMergeItems; ++j) {
        uint32_t m = m0 + j;
        slot[j] = (m < n_tot) ? s_slot[m] : 0xFFFFFFFFu;
        if (m < n_tot && !(slot[j] & 0x80000000u)) n_oldc++;
    }
    uint64_t tot_old, oi0 = block_exclusive_scan<kThreads>(n_oldc, s_scan, &tot_old);
    uint32_t oi[kMergeItems];
    uint64_t n_emit = 0;
    {
        uint32_t o = (uint32_t)oi0;
#pragma unroll
        for (int j = 0; j < kMergeItems; ++j) {
            uint32_t m = m0 + j;
            oi[j] = o;
            if (m < n_tot) {
                if (slot[j] & 0x80000000u) n_emit++;
                else { n_emit += s_keep[o]; ++o; }
            }
        }
    }
    uint64_t tot_emit, e0 = block_exclusive_scan<kThreads>(n_emit, s_scan, &tot_emit);
    if (CASC) {
        if (tid < 32) {
            uint64_t b = lookback_warp(a.status, (uint32_t)tile, tot_emit);
            if (lane_id() == 0) s_base = b;
        }
    } else if (tid == 0) {
        s_base = j0 - s_d[0] + r0;  // kept old elements before j0 + inserted records before d0
    }
    // stage the output chunk in merged order
    {
        uint32_t e = (uint32_t)e0;
#pragma unroll
        for (int j = 0; j < kMergeItems; ++j) {
            uint32_t m = m0 + j;
            if (m >= n_tot) break;
            if (slot[j] & 0x80000000u) {
                uint32_t s = slot[j] & 0x7FFFFFFFu;
                s_oc[e] = a.ins_col[r0 + s];
                s_ow[e] = a.ins_w[r0 + s];
                ++e;
            } else {
                uint32_t o = oi[j];
                if (CASC) s_kp[o] = e - (m - o);
                if (s_keep[o]) {
                    uint32_t col = s_col[o + sh];
                    s_oc[e] = REMAP ? a.remap[col] : col;
                    s_ow[e] = s_w[o + sh];
                    ++e;
                }
            }
        }
        if (CASC && tid == 0) s_kp[n_old] = (uint32_t)(tot_emit - n_new);
    }
    __syncthreads();
    const uint64_t base = s_base;
    const uint32_t cnt = (uint32_t)tot_emit;
    // coalesced store: scalar head to a 16 B boundary, 128-bit body, scalar tail
    {
        uint32_t head = (uint32_t)((4 - (base & 3)) & 3);
        if (head > cnt) head = cnt;
        if (tid < head) { a.new_cols[base + tid] = s_oc[tid]; a.new_w[base + tid] = s_ow[tid]; }
        const uint32_t body = (cnt - head) >> 2;
        uint4* gc = reinterpret_cast<uint4*>(a.new_cols + base + head);
        uint4* gw = reinterpret_cast<uint4*>(a.new_w + base + head);
        for (uint32_t q = tid; q < body; q += kThreads) {
            uint32_t s = head + (q << 2);
            gc[q] = make_uint4(s_oc[s], s_oc[s + 1], s_oc[s + 2], s_oc[s + 3]);
            gw[q] = make_uint4(__float_as_uint(s_ow[s]), __float_as_uint(s_ow[s + 1]),
                               __float_as_uint(s_ow[s + 2]), __float_as_uint(s_ow[s + 3]));
        }
        for (uint32_t s = head + (body << 2) + tid; s < cnt; s += kThreads) {
            a.new_cols[base + s] = s_oc[s];
            a.new_w[base + s] = s_ow[s];
        }
    }
    if (CASC) {
        // kept-before at every old row that starts inside this tile (last tile: also at E)
        const bool last = (tile == a.n_tiles - 1);
        __shared__ uint64_t s_k[2];
        if (tid < 2) {
            if (tid == 0) s_k[0] = lower_bound_dev(a.old_off, 0, a.V_old + 1, (int64_t)j0);
            else s_k[1] = last ? a.V_old + 1 : lower_bound_dev(a.old_off, 0, a.V_old + 1, (int64_t)j1);
        }
        __syncthreads();
        const uint64_t kept_before = base - r0;
        for (uint64_t k = s_k[0] + tid; k < s_k[1]; k += kThreads)
            a.KR[k] = (int64_t)(kept_before + s_kp[(uint64_t)a.old_off[k] - j0]);
        if (tid == 0) {
            uint64_t casc = (uint64_t)n_old - (tot_emit - n_new) - (s_d[1] - s_d[0]);
            if (casc) atomicAdd(&a.c->n_casc, (unsigned long long)casc);
        }
    }
}

// ============================================================== a4 + a5 ====
// New row offsets.  The per-row degree delta is non-zero only in rows that own
// an inserted record or a removed element; its exclusive scan at row u is
//   (kept old elements before row u's old start) + (inserted records in rows < u')
// where both terms are ranks in sorted lists (no cascade) or the kept-before
// table KR written by the merge's decoupled look-back (cascade).
template <bool CASC, bool REMAP>
__global__ void __launch_bounds__(kThreads) k_offsets_old(
    const int64_t* __restrict__ old_off, uint64_t V_old, const int64_t* __restrict__ KR,
    const uint64_t* __restrict__ del_pos, uint64_t n_del, const uint32_t* __restrict__ ins_row, uint64_t n_ins,
    const uint32_t* __restrict__ remap, int64_t* __restrict__ new_off) {
    uint64_t k0 = ((uint64_t)blockIdx.x * kThreads + threadIdx.x) * kItems;
    if (k0 >= V_old) return;
    uint64_t dp = 0, ip = 0;
    bool first = true;
    for (int j = 0; j < kItems; ++j) {
        uint64_t k = k0 + j;
        if (k >= V_old) break;
        uint32_t u = REMAP ? remap[k] : (uint32_t)k;
        if (u == kNone32) continue;
        int64_t kept;
        if (CASC) kept = KR[k];
        else {
            uint64_t x = (uint64_t)old_off[k];
            dp = first ? lower_bound_dev(del_pos, 0, n_del, x) : gallop_lb(del_pos, dp, n_del, x);
            kept = (int64_t)(x - dp);
        }
        ip = first ? lower_bound_dev(ins_row, 0, n_ins, u) : gallop_lb(ins_row, ip, n_ins, u);
        first = false;
        new_off[u] = kept + (int64_t)ip;
    }
}

template <bool CASC>
__global__ void k_offsets_inserted(const NodeVtx* __restrict__ nv, const uint32_t* __restrict__ ins_q,
                                   uint64_t n_vins, const int64_t* __restrict__ old_off,
                                   const int64_t* __restrict__ KR, const uint64_t* __restrict__ del_pos,
                                   uint64_t n_del, const uint32_t* __restrict__ ins_row, uint64_t n_ins,
                                   int64_t* __restrict__ new_off) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n_vins) return;
    const NodeVtx& r = nv[ins_q[i]];
    int64_t kept;
    if (CASC) kept = KR[r.oldpos];
    else {
        uint64_t x = (uint64_t)old_off[r.oldpos];
        kept = (int64_t)(x - lower_bound_dev(del_pos, 0, n_del, x));
    }
    new_off[r.newid] = kept + (int64_t)lower_bound_dev(ins_row, 0, n_ins, r.newid);
}

__global__ void k_set_i64(int64_t* p, int64_t v) { *p = v; }

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

__global__ void k_fill_i32(int32_t* p, uint64_t n, int32_t v) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) p[i] = v;
}

// ---------------------------------------------------------- PageRank ----
__global__ void k_pr_init(double* pr, uint64_t n) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) pr[i] = 1.0 / (double)n;
}
__global__ void k_pr_dangling(const int64_t* __restrict__ off, const double* __restrict__ pr, uint64_t n, double* out) {
    double acc = 0;
    for (uint64_t u = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; u < n; u += (uint64_t)gridDim.x * blockDim.x)
        if (off[u + 1] == off[u]) acc += pr[u];
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
__global__ void k_pr_finish(double* __restrict__ nxt, uint64_t n, double d, const double* __restrict__ dsum) {
    uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (v < n) nxt[v] = (1.0 - d) / (double)n + d * (nxt[v] + *dsum / (double)n);
}

}  // namespace h2tap
