// dyn.cuh - the dynamic replica: Algorithm 1 (§5.4 "Dynamic
// Data Structures") ingesting one cycle's delta records into a GPU graph of
// per-vertex hash tables - "a hash table per node to store edges" ([7]) - included
// by h2tap.cu (shares its allocator, stream, radix sort and record layout).
//
// Storage: one slab of u32 destination keys (EMPTY = ~0, TOMB = ~0 - 1) and a
// parallel slab of f32 weights.  Vertex v owns the slots [base[v], base[v] + cap[v]) - an
// open-addressing table (linear probing from a 32-bit mix of the key), cap a power of two
// (>= 4, 16-byte aligned) or 0 - with cnt[v] live keys and used[v] = live + tombstones.  A
// table grows (into fresh slots at the slab's tail, the old slots becoming garbage) when a
// cycle would push used over 3/4 of cap; the new cap keeps the load at or below 1/2.  The
// slab is rebuilt (every vertex's live keys re-hashed into tables sized for load 1/2,
// garbage dropped) when it runs out of room.  Inserts claim only EMPTY slots (a CAS on the
// key word); a key is unique within a launch (the items were sorted first).  Vertices: ext ids
// ascending (new IDs are > xid, Alg. 1 line 5/8, so they append) and a u32 liveness word per
// dense id (D3: dense ids never move, dead ones keep an empty table).
//
// One cycle (h2tap_dyn_apply_records), all on the replica stream:
//   k_dyn_rec        classify records (lines 2-9): deletion / new-node queues, per-record
//                    insert / delete item counts (+ record validation)
//   scan             item offsets, inserts and deletes packed in one u64 (k_scan_exclusive_u64)
//   new nodes        radix sort of the new IDs, k_dyn_kill (created and deleted in the same
//                    cycle: D3), k_dyn_heads + scan + k_dyn_append (line 10)
//   k_dyn_expand_ins thread per record (warp per large record): resolve endpoints, gate (D2), pack keys
//   radix sort       (key, item) - stable, so the last item of a key is the latest (D1)
//   k_dyn_inc / k_dyn_plan / k_dyn_grow   per source: incoming keys, tables that must grow
//                    (+ one read-back to place them in the slab), re-hash into the new tables
//   k_dyn_upsert     last item of each key: overwrite, or CAS-claim an EMPTY slot (lines 6, 10)
//   k_dyn_delete     thread per record (warp per large record): probe + CAS to TOMB (line 7)
//   k_dyn_node_del   liveness off (line 11) + k_dyn_cascade over every table if any died
// Reads traverse the tables in place (no materialisation): BFS, PageRank and SSSP scan a
// vertex's slots and skip EMPTY / TOMB.  Export (tests, checkpoints) materialises a CSR.

namespace dyn {

constexpr uint32_t kFilterBits = 1u << 18;   // cascade filter: 32 KB of shared memory

struct Ctr {
    unsigned long long n_new_ids, n_del_ids, bad, max_new, n_new, n_upd, n_del, n_casc, n_gated, n_vdel, n_out, last_ext, n_big_ins, n_big_del, sum_ins, sum_del;
    unsigned long long n_grow, grow_slots, alloc_tail, garbage, n_big_casc, n_front, bad_w;
};

__device__ __forceinline__ uint64_t hmix(uint64_t k) {
    k ^= k >> 33; k *= 0xff51afd7ed558ccdull; k ^= k >> 33; k *= 0xc4ceb9fe1a85ec53ull; k ^= k >> 33;
    return k;
}
__device__ __forceinline__ int64_t find_ext(const uint64_t* __restrict__ ext, uint64_t V, uint64_t x) {
    if (V == 0) return -1;
    const uint64_t e0 = __ldg(ext);
    if (x >= e0 && x - e0 < V && __ldg(ext + (x - e0)) == x) return (int64_t)(x - e0);  // dense id space: one load
    uint64_t lo = 0, hi = V;
    while (lo < hi) {
        const uint64_t m = (lo + hi) >> 1;
        if (ext[m] < x) lo = m + 1; else hi = m;
    }
    return (lo < V && ext[lo] == x) ? (int64_t)lo : -1;
}
__device__ __forceinline__ void wadd(unsigned long long* c, bool pred) {  // warp-aggregated count
    const unsigned m = __ballot_sync(__activemask(), pred);
    if (pred && (threadIdx.x & 31) == __ffs(m) - 1) atomicAdd(c, (unsigned long long)__popc(m));
}

// Alg. 1 lines 2-9 per record
__global__ void k_dyn_rec(const DeltaRec* __restrict__ rec, uint64_t nr, uint64_t n_ins, uint64_t n_del,
                          uint64_t xid, int has_xid, uint64_t* __restrict__ cnt,
                          uint64_t* __restrict__ new_ids, uint64_t* __restrict__ del_ids, Ctr* __restrict__ c) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    uint64_t ci = 0, cd = 0;
    unsigned bad = 0;
    if (i < nr) {
        const DeltaRec r = rec[i];
        if (r.valid > 1 || r.deleted > 1 || r.inserted > 1) bad |= REC_BAD_FLAG;
        if (r.valid) {
            if (r.ins_off > n_ins || r.ins_cnt > n_ins - r.ins_off || r.del_off > n_del || r.del_cnt > n_del - r.del_off)
                bad |= REC_BAD_SLICE;
            if (r.deleted) {                                       // lines 3-4
                del_ids[atomicAdd(&c->n_del_ids, 1ull)] = r.node;
            } else if (has_xid && r.node <= xid) {                // lines 5-7
                ci = r.ins_cnt;
                cd = r.del_cnt;
            } else {                                               // line 9 (D5: its deletes ignored)
                new_ids[atomicAdd(&c->n_new_ids, 1ull)] = r.node;
                atomicMax(&c->max_new, (unsigned long long)r.node);
                ci = r.ins_cnt;
            }
        }
        if (bad) atomicOr(&c->bad, (unsigned long long)bad);
        cnt[i] = ci << 32 | cd;   // packed insert / delete item counts (one scan places both)
    } else if (i == nr) {
        cnt[nr] = 0;
    }
    // exact totals: the packed scan is carry-free iff the insert total is < 2^30 and the delete
    // total < 2^32 (host check after the scan, before anything reads its output)
    const unsigned long long si = warp_sum<unsigned long long>(ci), sd = warp_sum<unsigned long long>(cd);
    if ((threadIdx.x & 31) == 0) {
        if (si) atomicAdd(&c->sum_ins, si);
        if (sd) atomicAdd(&c->sum_del, sd);
    }
}

// a new ID the cycle also deletes is never inserted (D3): flag its first copy in the sorted list
__global__ void k_dyn_kill(const uint64_t* __restrict__ del_ids, uint64_t nd, const uint64_t* __restrict__ sk,
                           uint64_t u, uint64_t base, uint8_t* __restrict__ kill) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= nd) return;
    const uint64_t x = del_ids[i];
    if (x < base) return;
    const uint64_t key = x - base;
    uint64_t lo = 0, hi = u;
    while (lo < hi) {
        const uint64_t m = (lo + hi) >> 1;
        if (sk[m] < key) lo = m + 1; else hi = m;
    }
    if (lo < u && sk[lo] == key) kill[lo] = 1;
}
__global__ void k_dyn_heads(const uint64_t* __restrict__ sk, uint64_t u, const uint8_t* __restrict__ kill,
                            uint64_t* __restrict__ flag) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i > u) return;
    flag[i] = (i < u && (i == 0 || sk[i] != sk[i - 1]) && !kill[i]) ? 1 : 0;
}
__global__ void k_dyn_append(const uint64_t* __restrict__ sk, uint64_t u, const uint64_t* __restrict__ flag,
                             const uint64_t* __restrict__ pos, uint64_t base, uint64_t* __restrict__ ext_tail,
                             uint32_t* __restrict__ live_tail, Ctr* __restrict__ c) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= u || !flag[i]) return;
    ext_tail[pos[i]] = sk[i] + base;   // line 10: ascending, after every old id
    live_tail[pos[i]] = 1;
    if (pos[i] + 1 == pos[u]) c->last_ext = sk[i] + base;  // the new xid
}

// The record's inserted edges as packed sort keys (invalid -> key_bad, sorts last).  Pass 0:
// one thread per record, serially over a slice of <= kSmall items (most records: the
// delta of one node in one transaction); larger records are queued for pass 1, one warp
// per queued record (a hub's slice may hold thousands of items).
constexpr uint64_t kSmall = 16;
__device__ __forceinline__ bool ins_item(uint64_t j, int64_t s, uint64_t o, uint64_t io, const uint64_t* __restrict__ ins,
                                         const float* __restrict__ wts, const uint64_t* __restrict__ ext,
                                         const uint32_t* __restrict__ live, uint64_t V, uint64_t* __restrict__ keys,
                                         uint32_t* __restrict__ vals, float* __restrict__ witem) {
    const int64_t d = s >= 0 ? find_ext(ext, V, ins[io + j]) : -1;
    const bool ok = d >= 0 && live[d];                            // D2
    keys[o + j] = ok ? (uint64_t)s * V + (uint64_t)d : V * V;     // sort key
    vals[o + j] = (uint32_t)(o + j);
    witem[o + j] = wts[io + j];
    return !ok;
}
__device__ __forceinline__ int64_t live_src(const uint64_t* __restrict__ ext, const uint32_t* __restrict__ live,
                                            uint64_t V, uint64_t x) {
    const int64_t s = find_ext(ext, V, x);
    return (s >= 0 && live[s]) ? s : -1;
}
template <int kPass>
__global__ void __launch_bounds__(256) k_dyn_expand_ins(const DeltaRec* __restrict__ rec, uint64_t nr,
        const uint64_t* __restrict__ off, const uint64_t* __restrict__ ins, const float* __restrict__ wts,
        const uint64_t* __restrict__ ext, const uint32_t* __restrict__ live, uint64_t V, uint64_t* __restrict__ keys,
        uint32_t* __restrict__ vals, float* __restrict__ witem, uint64_t* __restrict__ big,
        unsigned long long* __restrict__ n_big, Ctr* __restrict__ c) {
    unsigned long long gated = 0;
    if (kPass == 0) {
        const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
        if (i < nr) {
            const uint64_t o = off[i] >> 32, n = (off[i + 1] >> 32) - o;
            if (n > kSmall) big[atomicAdd(n_big, 1ull)] = i;
            else if (n) {
                const DeltaRec r = rec[i];
                const int64_t s = live_src(ext, live, V, r.node);
                for (uint64_t j = 0; j < n; ++j) gated += ins_item(j, s, o, r.ins_off, ins, wts, ext, live, V, keys, vals, witem);
            }
        }
    } else {
        const uint64_t nb = *n_big, nw = (uint64_t)gridDim.x * (blockDim.x >> 5);
        const unsigned lane = threadIdx.x & 31;
        for (uint64_t q = blockIdx.x * (uint64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); q < nb; q += nw) {
            const uint64_t i = big[q], o = off[i] >> 32, n = (off[i + 1] >> 32) - o;
            int64_t s = lane == 0 ? live_src(ext, live, V, rec[i].node) : -1;
            s = __shfl_sync(0xffffffffu, s, 0);
            const uint64_t io = rec[i].ins_off;
            for (uint64_t j = lane; j < n; j += 32) gated += ins_item(j, s, o, io, ins, wts, ext, live, V, keys, vals, witem);
        }
    }
    gated = warp_sum<unsigned long long>(gated);
    if ((threadIdx.x & 31) == 0 && gated) atomicAdd(&c->n_gated, gated);
}

// ---- per-vertex hash tables over the slab
constexpr uint32_t kKEmpty = 0xFFFFFFFFu, kKTomb = 0xFFFFFFFEu;
__device__ __forceinline__ uint32_t hmix32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16;
    return x;
}
struct Tabs {
    uint64_t* base;   // first slot of vertex v's table
    uint32_t* cap;    // slots (power of two >= 4, or 0)
    uint32_t* cnt;    // live keys
    uint32_t* used;   // live keys + tombstones
    uint32_t* key;    // slab: destination dense ids, EMPTY / TOMB
    float* val;       // slab: weights
    uint32_t* own;    // slab: owner vertex of every 4-slot group (kNoOwner: free or garbage)
};
constexpr uint32_t kNoOwner = 0xFFFFFFFFu;
__device__ __forceinline__ uint32_t pow2_cap(uint64_t live) {  // load <= 1/2, >= 4 slots
    uint32_t c = 4;
    while ((uint64_t)c < 2 * live) c <<= 1;
    return c;
}
// insert a key that is not in the table (re-hash / first insert): claim the first EMPTY slot
__device__ __forceinline__ void tab_claim(uint32_t* key, float* val, uint64_t b, uint32_t mask, uint32_t k, float w) {
    uint32_t h = hmix32(k) & mask;
    while (atomicCAS(&key[b + h], kKEmpty, k) != kKEmpty) h = (h + 1) & mask;
    val[b + h] = w;
}

// per source: the distinct keys this cycle upserts (the latest item of every key)
__global__ void k_dyn_inc(const uint64_t* __restrict__ sk, uint64_t n, uint64_t V, uint32_t* __restrict__ inc) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint64_t k = sk[i];
    if (k >= V * V || (i + 1 < n && sk[i + 1] == k)) return;
    atomicAdd(&inc[k / V], 1u);
}
// the first key of every source decides: the table grows when used + incoming would pass 3/4
// of its slots (a missing table always "grows"); the new size keeps the load <= 1/2
__global__ void k_dyn_plan(const uint64_t* __restrict__ sk, uint64_t n, uint64_t V, Tabs T, uint32_t* __restrict__ inc,
                           uint32_t* __restrict__ grow_v, uint32_t* __restrict__ grow_cap, Ctr* __restrict__ c) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint64_t k = sk[i];
    if (k >= V * V) return;
    const uint64_t s = k / V;
    if (i > 0 && sk[i - 1] / V == s) return;
    const uint32_t in = inc[s];
    inc[s] = 0;
    const uint32_t cap = T.cap[s];
    if (cap && 4ull * ((uint64_t)T.used[s] + in) <= 3ull * cap) return;
    const uint32_t nc = pow2_cap((uint64_t)T.cnt[s] + in);
    const uint64_t g = atomicAdd(&c->n_grow, 1ull);
    grow_v[g] = (uint32_t)s;
    grow_cap[g] = nc;
    atomicAdd(&c->grow_slots, (unsigned long long)nc);
}
// warp per growing table: fresh slots at the slab tail, live keys re-hashed, old slots -> garbage
__global__ void k_dyn_grow(const uint32_t* __restrict__ grow_v, const uint32_t* __restrict__ grow_cap, Tabs T,
                           uint64_t tail0, Ctr* __restrict__ c) {
    const uint64_t ng = c->n_grow;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint32_t lane = threadIdx.x & 31;
    for (uint64_t g = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; g < ng; g += nw) {
        const uint32_t v = grow_v[g], nc = grow_cap[g];
        unsigned long long nb = 0;
        if (lane == 0) nb = tail0 + atomicAdd(&c->alloc_tail, (unsigned long long)nc);
        nb = __shfl_sync(0xffffffffu, nb, 0);
        const uint64_t ob = T.base[v];
        const uint32_t oc = T.cap[v];
        for (uint32_t j = lane; j < oc; j += 32) {
            const uint32_t k = T.key[ob + j];
            if (k < kKTomb) tab_claim(T.key, T.val, nb, nc - 1, k, T.val[ob + j]);
        }
        for (uint32_t q = lane; q < nc / 4; q += 32) T.own[nb / 4 + q] = v;
        for (uint32_t q = lane; q < oc / 4; q += 32) T.own[ob / 4 + q] = kNoOwner;
        __syncwarp();
        if (lane == 0) {
            T.base[v] = nb;
            T.cap[v] = nc;
            T.used[v] = T.cnt[v];
            if (oc) atomicAdd(&c->garbage, (unsigned long long)oc);
        }
    }
}
// lines 6 + 10: the latest item of every key overwrites its weight, or claims an EMPTY slot
__global__ void k_dyn_upsert(const uint64_t* __restrict__ sk, const uint32_t* __restrict__ sv, uint64_t n,
                             const float* __restrict__ witem, uint64_t V, Tabs T, Ctr* __restrict__ c) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    bool nw = false, up = false;
    if (i < n) {
        const uint64_t k = sk[i];
        if (k < V * V && (i + 1 == n || sk[i + 1] != k)) {   // D1: the latest item of its key
            const uint64_t s = k / V;
            const uint32_t d = (uint32_t)(k - s * V), mask = T.cap[s] - 1;
            const uint64_t b = T.base[s];
            const float w = witem[sv[i]];
            uint32_t h = hmix32(d) & mask;
            while (true) {
                uint32_t cur = *((volatile uint32_t*)&T.key[b + h]);
                if (cur == d) { T.val[b + h] = w; up = true; break; }
                if (cur == kKEmpty) {
                    cur = atomicCAS(&T.key[b + h], kKEmpty, d);
                    if (cur == kKEmpty) {
                        T.val[b + h] = w;
                        atomicAdd(&T.cnt[s], 1u);
                        atomicAdd(&T.used[s], 1u);
                        nw = true;
                        break;
                    }
                    continue;   // another key took the slot: look at it again
                }
                h = (h + 1) & mask;
            }
        }
    }
    wadd(&c->n_new, nw);
    wadd(&c->n_upd, up);
}

__device__ __forceinline__ bool del_item(int64_t s, uint64_t x, const uint64_t* __restrict__ ext, uint64_t V, Tabs T) {
    const int64_t d = find_ext(ext, V, x);
    const uint32_t cap = T.cap[s];
    if (d < 0 || cap == 0) return false;
    const uint64_t b = T.base[s];
    uint32_t h = hmix32((uint32_t)d) & (cap - 1);
    while (true) {   // at least a quarter of the slots are EMPTY: the probe ends
        const uint32_t cur = *((volatile uint32_t*)&T.key[b + h]);
        if (cur == (uint32_t)d) {
            if (atomicCAS(&T.key[b + h], (uint32_t)d, kKTomb) != (uint32_t)d) return false;
            atomicSub(&T.cnt[s], 1u);
            return true;
        }
        if (cur == kKEmpty) return false;
        h = (h + 1) & (cap - 1);
    }
}
// line 7: the records' deleted edges to TOMB; passes as in k_dyn_expand_ins
template <int kPass>
__global__ void __launch_bounds__(256) k_dyn_delete(const DeltaRec* __restrict__ rec, uint64_t nr,
        const uint64_t* __restrict__ off, const uint64_t* __restrict__ del, const uint64_t* __restrict__ ext,
        uint64_t V, Tabs T, uint64_t* __restrict__ big, unsigned long long* __restrict__ n_big, Ctr* __restrict__ c) {
    unsigned long long hits = 0;
    if (kPass == 0) {
        const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
        if (i < nr) {
            const uint64_t n = (off[i + 1] & 0xffffffffu) - (off[i] & 0xffffffffu);
            if (n > kSmall) big[atomicAdd(n_big, 1ull)] = i;
            else if (n) {
                const DeltaRec r = rec[i];
                const int64_t s = find_ext(ext, V, r.node);
                if (s >= 0)                                      // D4
                    for (uint64_t j = 0; j < n; ++j) hits += del_item(s, del[r.del_off + j], ext, V, T);
            }
        }
    } else {
        const uint64_t nb = *n_big, nw = (uint64_t)gridDim.x * (blockDim.x >> 5);
        const unsigned lane = threadIdx.x & 31;
        for (uint64_t q = blockIdx.x * (uint64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); q < nb; q += nw) {
            const uint64_t i = big[q], n = (off[i + 1] & 0xffffffffu) - (off[i] & 0xffffffffu);
            int64_t s = lane == 0 ? find_ext(ext, V, rec[i].node) : -1;
            s = __shfl_sync(0xffffffffu, s, 0);
            if (s < 0) continue;
            const uint64_t dO = rec[i].del_off;
            for (uint64_t j = lane; j < n; j += 32) hits += del_item(s, del[dO + j], ext, V, T);
        }
    }
    hits = warp_sum<unsigned long long>(hits);
    if ((threadIdx.x & 31) == 0 && hits) atomicAdd(&c->n_del, hits);
}

// slab rebuild: every vertex's table re-sized for load <= 1/2 (live keys only) into a new slab
__global__ void k_dyn_caps(const uint32_t* __restrict__ cnt, uint64_t V, uint64_t* __restrict__ capn) {
    const uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (v < V) capn[v] = cnt[v] ? pow2_cap(cnt[v]) : 0;
    else if (v == V) capn[V] = 0;
}
__global__ void k_dyn_rebuild(Tabs T, uint64_t V, const uint64_t* __restrict__ capn, const uint64_t* __restrict__ nbase,
                              uint32_t* __restrict__ nkey, float* __restrict__ nval, uint32_t* __restrict__ nown) {
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint32_t lane = threadIdx.x & 31;
    for (uint64_t v = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; v < V; v += nw) {
        const uint32_t oc = T.cap[v], nc = (uint32_t)capn[v];
        const uint64_t ob = T.base[v], nb = nbase[v];
        for (uint32_t j = lane; j < oc; j += 32) {
            const uint32_t k = T.key[ob + j];
            if (k < kKTomb) tab_claim(nkey, nval, nb, nc - 1, k, T.val[ob + j]);
        }
        for (uint32_t q = lane; q < nc / 4; q += 32) nown[nb / 4 + q] = (uint32_t)v;
        __syncwarp();
        if (lane == 0) { T.base[v] = nb; T.cap[v] = nc; T.used[v] = T.cnt[v]; }
    }
}

__global__ void k_dyn_node_del(const uint64_t* __restrict__ del_ids, uint64_t nd, const uint64_t* __restrict__ ext,
                               uint64_t V, uint32_t* live, uint32_t* __restrict__ died_bits, uint32_t* __restrict__ filter,
                               Ctr* __restrict__ c) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    bool died = false;
    if (i < nd) {
        const int64_t d = find_ext(ext, V, del_ids[i]);
        died = d >= 0 && atomicExch(&live[d], 0u) == 1u;       // line 11 (D4: dead / unknown: no-op)
        if (died) {
            atomicOr(&died_bits[d >> 5], 1u << (d & 31));
            const uint64_t f = (uint64_t)d & (kFilterBits - 1);   // filter word for the cascade
            atomicOr(&filter[f >> 5], 1u << (f & 31));
        }
    }
    wadd(&c->n_vdel, died);
}

// line 11's cascade.  First the dead vertices' own tables are dropped (their keys are
// cascaded; the slots become garbage).  Then one linear pass over the slab: a key is removed
// iff its destination died this cycle (bitmap, V/8 bytes, L2-resident; a 32 KB shared-memory
// filter of the dead ids screens the keys before the bitmap is read).  16-byte loads of 4-slot
// groups, coalesced; only a group with a hit reads its owner (garbage groups have none and are
// skipped) to turn the keys into tombstones and lower the owner's live count.
__device__ __forceinline__ bool died_of(const uint32_t* __restrict__ b, const uint32_t* __restrict__ filt, uint32_t d) {
    const uint32_t fd = d & (kFilterBits - 1);
    if (((filt[fd >> 5] >> (fd & 31)) & 1u) == 0) return false;
    return (__ldg(b + (d >> 5)) >> (d & 31)) & 1u;
}
__global__ void k_dyn_drop_dead(const uint64_t* __restrict__ del_ids, uint64_t nd, const uint64_t* __restrict__ ext,
                                uint64_t V, const uint32_t* __restrict__ died_bits, Tabs T, Ctr* __restrict__ c) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= nd) return;
    const int64_t d = find_ext(ext, V, del_ids[i]);
    if (d < 0 || !((died_bits[d >> 5] >> (d & 31)) & 1u)) return;
    const uint32_t cap = atomicExch(&T.cap[d], 0u);   // a vertex listed twice is dropped once
    if (!cap) return;
    const uint64_t b = T.base[d];
    for (uint32_t q = 0; q < cap / 4; ++q) T.own[b / 4 + q] = kNoOwner;
    atomicAdd(&c->n_casc, (unsigned long long)T.cnt[d]);
    atomicAdd(&c->garbage, (unsigned long long)cap);
    T.cnt[d] = 0;
    T.used[d] = 0;
}
__global__ void __launch_bounds__(256, 4) k_dyn_cascade(Tabs T, uint64_t groups, const uint32_t* __restrict__ died_bits,
                                                        const uint32_t* __restrict__ filter, Ctr* __restrict__ c) {
    if (*(volatile unsigned long long*)&c->n_vdel == 0) return;   // nobody died this cycle (no host sync)
    extern __shared__ uint32_t filt[];
    for (uint32_t t = threadIdx.x; t < kFilterBits / 32; t += blockDim.x) filt[t] = filter[t];
    __syncthreads();
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    uint4* g4 = reinterpret_cast<uint4*>(T.key);
    unsigned long long gone = 0;
    constexpr int U = 4;   // 4 independent 16-byte loads in flight per thread
    uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    auto visit = [&](uint64_t q, uint4 k) {
        uint32_t* kk = reinterpret_cast<uint32_t*>(&k);
        uint32_t hits = 0;
#pragma unroll
        for (int e = 0; e < 4; ++e)
            if (kk[e] < kKTomb && died_of(died_bits, filt, kk[e])) { kk[e] = kKTomb; ++hits; }
        if (!hits) return;
        const uint32_t o = T.own[q];
        if (o == kNoOwner) return;   // garbage: stale keys of a moved or dropped table
        g4[q] = k;
        atomicSub(&T.cnt[o], hits);
        gone += hits;
    };
    for (; g + (U - 1) * stride < groups; g += U * stride) {
        uint4 k[U];
#pragma unroll
        for (int u = 0; u < U; ++u) k[u] = __ldcs(g4 + g + u * stride);
#pragma unroll
        for (int u = 0; u < U; ++u) visit(g + u * stride, k[u]);
    }
    for (; g < groups; g += stride) visit(g, g4[g]);
    gone = warp_sum<unsigned long long>(gone);
    if ((threadIdx.x & 31) == 0 && gone) atomicAdd(&c->n_casc, gone);
}

// create: flat edge list -> packed keys (an endpoint that is no vertex -> bad)
__global__ void k_dyn_expand_flat(const uint64_t* __restrict__ src, const uint64_t* __restrict__ dst,
                                  const float* __restrict__ w, uint64_t n, const uint64_t* __restrict__ ext, uint64_t V,
                                  uint64_t* __restrict__ keys, uint32_t* __restrict__ vals, float* __restrict__ witem,
                                  Ctr* __restrict__ c) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const int64_t s = find_ext(ext, V, src[i]), d = find_ext(ext, V, dst[i]);
    if (s < 0 || d < 0) { atomicOr(&c->bad, 1ull); keys[i] = V * V; }
    else keys[i] = (uint64_t)s * V + (uint64_t)d;
    vals[i] = (uint32_t)i;
    witem[i] = w ? w[i] : 1.0f;
}
__global__ void k_dyn_check_ids(const uint64_t* __restrict__ ext, uint64_t V, Ctr* __restrict__ c) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i > 0 && i < V && ext[i] <= ext[i - 1]) atomicOr(&c->bad, 1ull);
}
__global__ void k_dyn_sub_base(const uint64_t* __restrict__ ids, uint64_t n, uint64_t base, uint64_t* __restrict__ k,
                               uint32_t* __restrict__ v) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) { k[i] = ids[i] - base; v[i] = 0; }
}
__global__ void k_dyn_fill_u32(uint32_t* p, uint64_t n, uint32_t v) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) p[i] = v;
}

// export: every live key as a sort key s * V + d (thread per vertex, warp-aggregated output)
__global__ void k_dyn_compact(Tabs T, uint64_t V, uint64_t* __restrict__ ok, uint32_t* __restrict__ oi,
                              float* __restrict__ ow, Ctr* __restrict__ c) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t u0 = blockIdx.x * (uint64_t)blockDim.x; u0 < V; u0 += stride) {
        const uint64_t u = u0 + threadIdx.x;
        const uint32_t n = u < V ? T.cnt[u] : 0u;
        const uint32_t lane = threadIdx.x & 31;
        uint32_t inc = n;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
            if ((int)lane >= o) inc += y;
        }
        const uint32_t tot = __shfl_sync(0xffffffffu, inc, 31);
        unsigned long long base = 0;
        if (lane == 0 && tot) base = atomicAdd(&c->n_out, (unsigned long long)tot);
        base = __shfl_sync(0xffffffffu, base, 0) + inc - n;
        if (!n) continue;
        const uint64_t b = T.base[u];
        const uint32_t cap = T.cap[u];
        for (uint32_t j = 0; j < cap; ++j) {
            const uint32_t k = T.key[b + j];
            if (k < kKTomb) {
                ok[base] = u * V + k;
                oi[base] = (uint32_t)base;
                ow[base] = T.val[b + j];
                ++base;
            }
        }
    }
}

// ---- reads on the tables in place (Table 1's BFS / PageRank / SSSP)
__global__ void k_dyn_bfs_expand(Tabs T, const uint32_t* __restrict__ front, uint64_t nf, int32_t* __restrict__ level,
                                 int32_t depth, uint32_t* __restrict__ next, unsigned long long* __restrict__ n_next) {
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t f = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; f < nf; f += nw) {
        const uint32_t u = front[f], cap = T.cap[u];
        const uint64_t b = T.base[u];
        for (uint32_t j = lane_id(); j < cap; j += 32) {
            const uint32_t v = T.key[b + j];
            bool claim = false;
            if (v < kKTomb && level[v] < 0) claim = atomicCAS(&level[v], -1, depth + 1) == -1;
            const uint32_t m = __ballot_sync(__activemask(), claim);
            if (claim) {
                const uint32_t leader = __ffs(m) - 1;
                unsigned long long o = 0;
                if (lane_id() == leader) o = atomicAdd(n_next, (unsigned long long)__popc(m));
                o = __shfl_sync(m, o, leader);
                next[o + __popc(m & lanemask_lt())] = v;
            }
        }
    }
}
__global__ void k_dyn_pr_dangling(const uint32_t* __restrict__ cnt, const uint32_t* __restrict__ live,
                                  const double* __restrict__ pr, uint64_t V, double* __restrict__ out) {
    double acc = 0;
    for (uint64_t u = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; u < V; u += (uint64_t)gridDim.x * blockDim.x)
        if (live[u] && cnt[u] == 0) acc += pr[u];
    acc = warp_sum(acc);
    if (lane_id() == 0 && acc != 0.0) atomicAdd(out, acc);
}
__global__ void k_dyn_pr_push(Tabs T, const double* __restrict__ pr, uint64_t V, double* __restrict__ nxt) {
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t u = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; u < V; u += nw) {
        const uint32_t n = T.cnt[u];
        if (!n) continue;
        const uint32_t cap = T.cap[u];
        const uint64_t b = T.base[u];
        const double cu = pr[u] / (double)n;
        for (uint32_t j = lane_id(); j < cap; j += 32) {
            const uint32_t v = T.key[b + j];
            if (v < kKTomb) atomicAdd(&nxt[v], cu);
        }
    }
}
__global__ void k_dyn_check_w(Tabs T, uint64_t V, Ctr* __restrict__ c) {
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    bool bad = false;
    for (uint64_t u = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; u < V; u += nw) {
        const uint32_t cap = T.cap[u];
        const uint64_t b = T.base[u];
        for (uint32_t j = lane_id(); j < cap; j += 32)
            if (T.key[b + j] < kKTomb) { const float x = T.val[b + j]; bad |= !(x >= 0.0f); }
    }
    if (__any_sync(0xffffffffu, bad) && lane_id() == 0) atomicOr(&c->bad_w, 1ull);
}
__global__ void k_dyn_sssp_relax(Tabs T, const uint32_t* __restrict__ front, uint64_t nf, unsigned long long* dist,
                                 uint32_t* __restrict__ stamp, uint32_t round, uint32_t* __restrict__ next,
                                 unsigned long long* __restrict__ n_next) {
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t f = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; f < nf; f += nw) {
        const uint32_t u = front[f], cap = T.cap[u];
        const uint64_t b = T.base[u];
        const double du = __longlong_as_double((long long)ld_volatile(reinterpret_cast<const uint64_t*>(dist + u)));
        for (uint32_t j = lane_id(); j < cap; j += 32) {
            const uint32_t v = T.key[b + j];
            bool push = false;
            if (v < kKTomb) {
                const double nd = du + (double)T.val[b + j];
                const unsigned long long nb = (unsigned long long)__double_as_longlong(nd);
                if (nb < ld_volatile(reinterpret_cast<const uint64_t*>(dist + v)) && atomicMin(dist + v, nb) > nb)
                    push = atomicExch(stamp + v, round) != round;
            }
            const uint32_t m = __ballot_sync(__activemask(), push);
            if (push) {
                const uint32_t leader = __ffs(m) - 1;
                unsigned long long o = 0;
                if (lane_id() == leader) o = atomicAdd(n_next, (unsigned long long)__popc(m));
                o = __shfl_sync(m, o, leader);
                next[o + __popc(m & lanemask_lt())] = v;
            }
        }
    }
}

__global__ void k_dyn_emit(const uint64_t* __restrict__ sk, const uint32_t* __restrict__ si, const float* __restrict__ cw,
                           uint64_t E, uint64_t V, uint32_t* __restrict__ cols, float* __restrict__ w) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= E) return;
    cols[i] = (uint32_t)(sk[i] % V);
    w[i] = cw[si[i]];
}
__global__ void k_dyn_offsets(const uint64_t* __restrict__ sk, uint64_t E, uint64_t V, int64_t* __restrict__ off) {
    const uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (v > V) return;
    const uint64_t key = v * V;   // sort key s * V + d
    uint64_t lo = 0, hi = E;
    while (lo < hi) {
        const uint64_t m = (lo + hi) >> 1;
        if (sk[m] < key) lo = m + 1; else hi = m;
    }
    off[v] = (int64_t)lo;
}
// dense id + 1 of a live ext id into c->bad (0: none)
__global__ void k_dyn_lookup(const uint64_t* __restrict__ ext, const uint32_t* __restrict__ live, uint64_t V,
                             uint64_t x, Ctr* __restrict__ c) {
    if (threadIdx.x) return;
    const int64_t d = find_ext(ext, V, x);
    c->bad = (d >= 0 && live[d]) ? (unsigned long long)d + 1 : 0;
}
__global__ void k_dyn_live_u8(const uint32_t* __restrict__ live, uint64_t V, uint8_t* __restrict__ out) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < V) out[i] = (uint8_t)live[i];
}

}  // namespace dyn

struct h2tap_dyn {
    h2tap_replica* r = nullptr;   // stream, allocator, radix-sort scratch
    uint64_t V = 0, n_live = 0, xid = 0;   // xid = ext[V - 1] (host copy)
    uint64_t slab_cap = 0, tail = 0, garbage = 0;   // slab slots, allocated slots, garbage slots
    Buf ext, live, base, cap, cnt, used, key, val, own, inc, grow_v, grow_cap, died, big;
    Buf cin, oin, new_ids, del_ids, kill, flag, fpos, keys, vals, keys2, vals2, witem, ctr, xo;
    Buf x_rec, x_ins, x_wts, x_del, live8, fa, fb, lvl, da, db;
    struct Stage {
        Buf rec, ins, wts, del;
        cudaEvent_t ev = nullptr;
        uint64_t bytes = 0;
    } stg[2];
    int stg_next = 0;
    dyn::Ctr* hctr = nullptr;     // pinned host mirror
};

namespace {

dyn::Tabs dyn_tabs(h2tap_dyn* d) {
    return dyn::Tabs{static_cast<uint64_t*>(d->base.p), static_cast<uint32_t*>(d->cap.p),
                     static_cast<uint32_t*>(d->cnt.p), static_cast<uint32_t*>(d->used.p),
                     static_cast<uint32_t*>(d->key.p), static_cast<float*>(d->val.p),
                     static_cast<uint32_t*>(d->own.p)};
}

void dyn_free(h2tap_dyn* d) {
    if (!d) return;
    if (d->r) {
        for (Buf* b : {&d->ext, &d->live, &d->base, &d->cap, &d->cnt, &d->used, &d->key, &d->val, &d->own, &d->inc,
                       &d->grow_v, &d->grow_cap, &d->died, &d->big, &d->cin, &d->oin, &d->new_ids, &d->del_ids,
                       &d->kill, &d->flag, &d->fpos, &d->keys, &d->vals, &d->keys2, &d->vals2, &d->witem, &d->ctr,
                       &d->xo, &d->x_rec, &d->x_ins, &d->x_wts, &d->x_del, &d->live8, &d->fa, &d->fb, &d->lvl,
                       &d->da, &d->db})
            if (b->p) d->r->dfree(b->p);
        for (auto& g : d->stg) {
            for (Buf* b : {&g.rec, &g.ins, &g.wts, &g.del}) if (b->p) d->r->dfree(b->p);
            if (g.ev) cudaEventDestroy(g.ev);
        }
        free_replica(d->r);
    }
    if (d->hctr) cudaFreeHost(d->hctr);
    delete d;
}

dyn::Ctr* dyn_ctr_reset(h2tap_dyn* d) {
    h2tap_replica* r = d->r;
    dyn::Ctr* c = r->get<dyn::Ctr>(d->ctr, 1);
    CK(cudaMemsetAsync(c, 0, sizeof(dyn::Ctr), r->st));
    return c;
}
void dyn_ctr_read(h2tap_dyn* d) {
    CK(cudaMemcpyAsync(d->hctr, d->ctr.p, sizeof(dyn::Ctr), cudaMemcpyDeviceToHost, d->r->st));
    g_d2h += sizeof(dyn::Ctr);
    d->r->sync();
}

// grow the per-vertex arrays to hold n dense ids (contents kept, new entries: no table)
void dyn_reserve_vertices(h2tap_dyn* d, uint64_t n) {
    h2tap_replica* r = d->r;
    if (d->ext.cap >= (n + 16) * 8 && d->live.cap >= (n + 16) * 4) return;
    const uint64_t want = std::max<uint64_t>(n, 2 * d->V) + 1024;
    auto regrow = [&](Buf& b, size_t el) {
        Buf b2;
        r->get<uint8_t>(b2, want * el);
        CK(cudaMemsetAsync(b2.p, 0, (want + 16) * el, r->st));
        if (d->V) CK(cudaMemcpyAsync(b2.p, b.p, d->V * el, cudaMemcpyDeviceToDevice, r->st));
        r->release(b);
        b = b2;
    };
    regrow(d->ext, 8);
    regrow(d->live, 4);
    regrow(d->base, 8);
    regrow(d->cap, 4);
    regrow(d->cnt, 4);
    regrow(d->used, 4);
    regrow(d->inc, 4);
}

// rebuild the slab: every table re-sized for load <= 1/2 into a slab with `extra` free slots
void dyn_rebuild(h2tap_dyn* d, uint64_t extra) {
    h2tap_replica* r = d->r;
    cudaStream_t st = r->st;
    const uint64_t V = d->V;
    Buf bc, bb;
    uint64_t* capn = r->get<uint64_t>(bc, V + 1);
    uint64_t* nbase = r->get<uint64_t>(bb, V + 1);
    dyn::k_dyn_caps<<<g1(V + 1), 256, 0, st>>>(static_cast<const uint32_t*>(d->cnt.p), V, capn);
    CKL();
    const uint64_t nt = cdiv(V + 1, kTile);
    uint64_t* stt = r->get<uint64_t>(r->status2, nt);
    unsigned int* sc = reinterpret_cast<unsigned int*>(r->get<uint64_t>(d->xo, 2));
    CK(cudaMemsetAsync(stt, 0, nt * 8, st));
    CK(cudaMemsetAsync(sc, 0, 4, st));
    k_scan_exclusive_u64<<<(unsigned)nt, kThreads, 0, st>>>(capn, nbase, V + 1, stt, sc);
    CKL();
    uint64_t total = 0;
    CK(cudaMemcpyAsync(&total, nbase + V, 8, cudaMemcpyDeviceToHost, st));
    r->sync();
    const uint64_t ncap = ((total + extra) * 5 / 4 + 1023) & ~1023ull;
    Buf k2, v2, o2;
    uint32_t* nk = r->get<uint32_t>(k2, ncap);
    float* nv = r->get<float>(v2, ncap);
    uint32_t* no = r->get<uint32_t>(o2, ncap / 4);
    CK(cudaMemsetAsync(nk, 0xFF, (ncap + 16) * 4, st));
    CK(cudaMemsetAsync(no, 0xFF, (ncap / 4 + 16) * 4, st));
    if (V) {
        const unsigned grid = (unsigned)std::min<uint64_t>(cdiv(V * 32, 256), (uint64_t)r->n_sm * 16);
        dyn::k_dyn_rebuild<<<grid, 256, 0, st>>>(dyn_tabs(d), V, capn, nbase, nk, nv, no);
        CKL();
    }
    r->release(d->key);
    r->release(d->val);
    r->release(d->own);
    d->own = o2;
    r->release(bc);
    r->release(bb);
    d->key = k2;
    d->val = v2;
    d->slab_cap = ncap;
    d->tail = total;
    d->garbage = 0;
}

// sort (key, item) items and upsert the latest item of every key; tables grow first
void dyn_upsert_items(h2tap_dyn* d, uint64_t n, dyn::Ctr* c) {
    h2tap_replica* r = d->r;
    cudaStream_t st = r->st;
    if (!n) return;
    uint64_t* k = static_cast<uint64_t*>(d->keys.p);
    uint32_t* v = static_cast<uint32_t*>(d->vals.p);
    uint64_t* k2 = static_cast<uint64_t*>(d->keys2.p);
    uint32_t* v2 = static_cast<uint32_t*>(d->vals2.p);
    radix_sort(r, k, v, k2, v2, n, bits_for(d->V * d->V));
    uint32_t* grow_v = r->get<uint32_t>(d->grow_v, n);
    uint32_t* grow_cap = r->get<uint32_t>(d->grow_cap, n);
    for (int attempt = 0;; ++attempt) {
        CK(cudaMemsetAsync(&c->n_grow, 0, 24, st));   // n_grow, grow_slots, alloc_tail
        dyn::k_dyn_inc<<<g1(n), 256, 0, st>>>(k, n, d->V, static_cast<uint32_t*>(d->inc.p));
        CKL();
        dyn::k_dyn_plan<<<g1(n), 256, 0, st>>>(k, n, d->V, dyn_tabs(d), static_cast<uint32_t*>(d->inc.p), grow_v,
                                               grow_cap, c);
        CKL();
        dyn_ctr_read(d);
        const uint64_t ng = d->hctr->n_grow, slots = d->hctr->grow_slots;
        if (d->tail + slots <= d->slab_cap) {
            if (ng) {
                CK(cudaMemsetAsync(static_cast<uint32_t*>(d->key.p) + d->tail, 0xFF, slots * 4, st));
                const unsigned grid = (unsigned)std::min<uint64_t>(cdiv(ng * 32, 256), (uint64_t)r->n_sm * 16);
                dyn::k_dyn_grow<<<grid, 256, 0, st>>>(grow_v, grow_cap, dyn_tabs(d), d->tail, c);
                CKL();
                d->tail += slots;
            }
            break;
        }
        if (attempt) { set_err("slab rebuild did not make room"); throw Fail{H2TAP_E_CUDA}; }
        // out of slab: rebuild (garbage dropped, room for this cycle's growth), then plan again
        dyn_rebuild(d, slots + d->slab_cap / 4);
    }
    dyn::k_dyn_upsert<<<g1(n), 256, 0, st>>>(k, v, n, static_cast<float*>(d->witem.p), d->V, dyn_tabs(d), c);
    CKL();
}

void dyn_item_bufs(h2tap_dyn* d, uint64_t n) {
    h2tap_replica* r = d->r;
    r->get<uint64_t>(d->keys, n);
    r->get<uint64_t>(d->keys2, n);
    r->get<uint32_t>(d->vals, n);
    r->get<uint32_t>(d->vals2, n);
    r->get<float>(d->witem, n);
}

h2tap_status dyn_apply(h2tap_dyn* d, const h2tap_record_batch* b, h2tap_apply_stats* stats) {
    h2tap_replica* r = d->r;
    cudaStream_t st = r->st;
    g_launches = g_h2d = g_d2h = 0;
    CK(cudaEventRecord(r->ev[0], st));
    const uint64_t nr = b->n_records;
    const DeltaRec* rec = reinterpret_cast<const DeltaRec*>(b->records);
    const uint64_t* ins = b->inserts;
    const float* wts = b->weights;
    const uint64_t* del = b->deletes;
    if (nr && !rec) { set_err("records is NULL"); return H2TAP_E_INVAL; }
    if (b->weights64) { set_err("the dynamic replica takes f32 weights (weights64 is for the CSR replica)"); return H2TAP_E_INVAL; }
    if ((b->n_inserts && (!ins || !wts)) || (b->n_deletes && !del)) { set_err("null inserts/weights/deletes"); return H2TAP_E_INVAL; }
    for (auto& g : d->stg)  // a batch staged by h2tap_dyn_stage: its copy is ordered first
        if (nr && b->on_device && b->records == g.rec.p) {
            CK(cudaStreamWaitEvent(st, g.ev, 0));
            g_h2d += g.bytes;
            g.bytes = 0;
        }
    if (!b->on_device) {
        DeltaRec* xr = r->get<DeltaRec>(d->x_rec, nr);
        uint64_t* xi = r->get<uint64_t>(d->x_ins, b->n_inserts);
        float* xw = r->get<float>(d->x_wts, b->n_inserts);
        uint64_t* xd = r->get<uint64_t>(d->x_del, b->n_deletes);
        copy_in(r, xr, rec, nr, 0);
        copy_in(r, xi, ins, b->n_inserts, 0);
        copy_in(r, xw, wts, b->n_inserts, 0);
        copy_in(r, xd, del, b->n_deletes, 0);
        rec = xr; ins = xi; wts = xw; del = xd;
    }
    // ---- lines 1-9: classify records
    const uint64_t xid = d->xid;
    dyn::Ctr* c = dyn_ctr_reset(d);
    if (b->n_inserts >= (1ull << 32) || b->n_deletes >= (1ull << 32)) {
        set_err("inserts / deletes arrays of 2^32 or more entries");
        return H2TAP_E_CAPACITY;
    }
    uint64_t* cnt = r->get<uint64_t>(d->cin, nr + 1);
    uint64_t* oin = r->get<uint64_t>(d->oin, nr + 1);   // packed exclusive offsets (ins << 32 | del)
    uint64_t* odel = oin;
    uint64_t* new_ids = r->get<uint64_t>(d->new_ids, nr);
    uint64_t* del_ids = r->get<uint64_t>(d->del_ids, nr);
    dyn::k_dyn_rec<<<g1(nr + 1), 256, 0, st>>>(rec, nr, b->n_inserts, b->n_deletes, xid, d->V ? 1 : 0, cnt,
                                              new_ids, del_ids, c);
    CKL();
    {
        const uint64_t n = nr + 1, nt = cdiv(n, kTile);
        uint64_t* stt = r->get<uint64_t>(r->status2, nt);
        unsigned int* sc = reinterpret_cast<unsigned int*>(r->get<uint64_t>(d->xo, 2));
        CK(cudaMemsetAsync(stt, 0, nt * 8, st));
        CK(cudaMemsetAsync(sc, 0, 4, st));
        k_scan_exclusive_u64<<<(unsigned)nt, kThreads, 0, st>>>(cnt, oin, n, stt, sc);
        CKL();
    }
    uint64_t packed_tot = 0, tot[2];
    CK(cudaMemcpyAsync(&packed_tot, oin + nr, 8, cudaMemcpyDeviceToHost, st));
    g_d2h += 8;
    dyn_ctr_read(d);
    const dyn::Ctr h0 = *d->hctr;
    // The packed scan is carry-free only while every prefix fits its field: deletes in the
    // low 32 bits, inserts in bits 32..61 (the look-back status word keeps its flag in bits
    // 62-63 and masks values to 62 bits, dev_common.cuh), hence sum_ins < 2^30.  Nothing
    // has read the packed offsets yet, so refusing here leaves the replica unchanged.
    if (!(h0.bad & (REC_BAD_FLAG | REC_BAD_SLICE)) && (h0.sum_ins >= (1ull << 30) || h0.sum_del >= (1ull << 32))) {
        set_err("%llu inserted / %llu deleted edge items in one cycle (limits 2^30 - 1 / 2^32 - 1)",
                (unsigned long long)h0.sum_ins, (unsigned long long)h0.sum_del);
        return H2TAP_E_CAPACITY;
    }
    if (d->n_live + h0.sum_ins >= 0xFFFFFFFFull) {  // the materialised CSR keys edges by u32 position
        set_err("live edges (%llu) + inserted items (%llu) would reach 2^32 - 1",
                (unsigned long long)d->n_live, (unsigned long long)h0.sum_ins);
        return H2TAP_E_CAPACITY;
    }
    tot[0] = packed_tot >> 32;
    tot[1] = packed_tot & 0xffffffffu;
    if (h0.bad & REC_BAD_FLAG) { set_err("delta record flag other than 0/1"); return H2TAP_E_INVAL; }
    if (h0.bad & REC_BAD_SLICE) { set_err("delta record slice outside the inserts/weights/deletes arrays"); return H2TAP_E_INVAL; }
    const uint64_t n_ins = tot[0];
    // ---- line 10: new nodes (ascending, after every old id; D3)
    uint64_t n_vins = 0;
    const uint64_t u = h0.n_new_ids;
    if (u) {
        const uint64_t base = d->V ? xid + 1 : 0;
        dyn_item_bufs(d, std::max<uint64_t>(u, 1));
        uint64_t* k = static_cast<uint64_t*>(d->keys.p);
        uint32_t* v = static_cast<uint32_t*>(d->vals.p);
        uint64_t* k2 = static_cast<uint64_t*>(d->keys2.p);
        uint32_t* v2 = static_cast<uint32_t*>(d->vals2.p);
        // key = id - base (fits the bits of max_new - base)
        dyn::k_dyn_sub_base<<<g1(u), 256, 0, st>>>(new_ids, u, base, k, v);
        CKL();
        radix_sort(r, k, v, k2, v2, u, bits_for(h0.max_new - base));
        uint8_t* kill = r->get<uint8_t>(d->kill, u);
        CK(cudaMemsetAsync(kill, 0, u, st));
        if (h0.n_del_ids) {
            dyn::k_dyn_kill<<<g1(h0.n_del_ids), 256, 0, st>>>(del_ids, h0.n_del_ids, k, u, base, kill);
            CKL();
        }
        uint64_t* flag = r->get<uint64_t>(d->flag, u + 1);
        uint64_t* pos = r->get<uint64_t>(d->fpos, u + 1);
        dyn::k_dyn_heads<<<g1(u + 1), 256, 0, st>>>(k, u, kill, flag);
        CKL();
        const uint64_t nt = cdiv(u + 1, kTile);
        uint64_t* stt = r->get<uint64_t>(r->status2, nt);
        unsigned int* sc = reinterpret_cast<unsigned int*>(r->get<uint64_t>(d->xo, 2));
        CK(cudaMemsetAsync(stt, 0, nt * 8, st));
        CK(cudaMemsetAsync(sc, 0, 4, st));
        k_scan_exclusive_u64<<<(unsigned)nt, kThreads, 0, st>>>(flag, pos, u + 1, stt, sc);
        CKL();
        CK(cudaMemcpyAsync(&n_vins, pos + u, 8, cudaMemcpyDeviceToHost, st));
        g_d2h += 8;
        dyn_reserve_vertices(d, d->V + u);
        dyn::k_dyn_append<<<g1(u), 256, 0, st>>>(k, u, flag, pos, base, static_cast<uint64_t*>(d->ext.p) + d->V,
                                                 static_cast<uint32_t*>(d->live.p) + d->V, c);
        CKL();
        r->sync();
        if (d->V + n_vins >= 0xFFFFFFFFull) { set_err("more than 2^32 - 2 dense vertex ids"); return H2TAP_E_CAPACITY; }
        d->V += n_vins;
    }
    const uint64_t* ext = static_cast<const uint64_t*>(d->ext.p);
    uint32_t* live = static_cast<uint32_t*>(d->live.p);
    const unsigned wgrid = (unsigned)r->n_sm * 4;   // warp passes over the queued large records
    // ---- lines 6 + 10: one insert batch (D1, D2)
    if (n_ins) {
        dyn_item_bufs(d, n_ins);
        uint64_t* big = r->get<uint64_t>(d->big, nr);
        unsigned long long* nbig = &c->n_big_ins;
        dyn::k_dyn_expand_ins<0><<<g1(nr), 256, 0, st>>>(rec, nr, oin, ins, wts, ext, live, d->V,
                                                        static_cast<uint64_t*>(d->keys.p), static_cast<uint32_t*>(d->vals.p),
                                                        static_cast<float*>(d->witem.p), big, nbig, c);
        CKL();
        dyn::k_dyn_expand_ins<1><<<wgrid, 256, 0, st>>>(rec, nr, oin, ins, wts, ext, live, d->V,
                                                       static_cast<uint64_t*>(d->keys.p), static_cast<uint32_t*>(d->vals.p),
                                                       static_cast<float*>(d->witem.p), big, nbig, c);
        CKL();
        dyn_upsert_items(d, n_ins, c);
    }
    // ---- line 7: delete batch
    if (tot[1]) {
        uint64_t* big = r->get<uint64_t>(d->big, nr);
        dyn::k_dyn_delete<0><<<g1(nr), 256, 0, st>>>(rec, nr, odel, del, ext, d->V, dyn_tabs(d), big, &c->n_big_del, c);
        CKL();
        dyn::k_dyn_delete<1><<<wgrid, 256, 0, st>>>(rec, nr, odel, del, ext, d->V, dyn_tabs(d), big, &c->n_big_del, c);
        CKL();
    }
    // ---- line 11: node deletes + cascade
    bool casc_timed = false;
    if (h0.n_del_ids) {
        const uint64_t nwd = (d->V + 31) / 32, nwf = dyn::kFilterBits / 32;
        uint32_t* died = r->get<uint32_t>(d->died, nwd + nwf);
        uint32_t* filter = died + nwd;
        CK(cudaMemsetAsync(died, 0, (nwd + nwf) * 4, st));
        dyn::k_dyn_node_del<<<g1(h0.n_del_ids), 256, 0, st>>>(del_ids, h0.n_del_ids, ext, d->V, live, died, filter, c);
        CKL();
        dyn::k_dyn_drop_dead<<<g1(h0.n_del_ids), 256, 0, st>>>(del_ids, h0.n_del_ids, ext, d->V, died, dyn_tabs(d), c);
        CKL();
        if (d->tail) {
            constexpr int smem = dyn::kFilterBits / 8;
            CK(cudaFuncSetAttribute(dyn::k_dyn_cascade, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
            const uint64_t groups = d->tail / 4;
            const unsigned grid = (unsigned)std::min<uint64_t>(g1(groups), (uint64_t)r->n_sm * 4);  // 4 CTAs/SM
            CK(cudaEventRecord(r->ev[2], st));
            dyn::k_dyn_cascade<<<grid, 256, smem, st>>>(dyn_tabs(d), groups, died, filter, c);
            CKL();
            CK(cudaEventRecord(r->ev[3], st));
            casc_timed = true;
        }
    }
    CK(cudaEventRecord(r->ev[1], st));
    dyn_ctr_read(d);
    const dyn::Ctr& h = *d->hctr;
    d->n_live = d->n_live + h.n_new - h.n_del - h.n_casc;
    d->garbage += h.garbage;
    if (n_vins) d->xid = h.last_ext;
    if (stats) {
        std::memset(stats, 0, sizeof(*stats));
        stats->n_visible = n_ins + tot[1] + u + h0.n_del_ids;
        stats->n_gated = h.n_gated;
        stats->n_new = h.n_new;
        stats->n_upd = h.n_upd;
        stats->n_del = h.n_del;
        stats->n_casc = h.n_casc;
        stats->n_vertex_inserted = n_vins;
        stats->n_vertex_deleted = h.n_vdel;
        stats->ms_total = ev_ms(r->ev[0], r->ev[1]);
        if (casc_timed && h.n_vdel) {   // the cascade pass: its launch time and the table bytes it streams
            stats->ms_merge = ev_ms(r->ev[2], r->ev[3]);
            stats->bytes_merge = d->tail * 4;   // the linear pass reads every allocated slot once
        }
        // algorithmic bytes: records + slices read, one probe (4-byte key + 4-byte weight) per item
        stats->bytes_alg = nr * sizeof(DeltaRec) + n_ins * 12 + tot[1] * 8 + (n_ins + tot[1]) * 8;
        stats->n_launches = g_launches;
        stats->h2d_bytes = g_h2d;
        stats->d2h_bytes = g_d2h;
    }
    return H2TAP_OK;
}

// the CSR of the tables (rows = dense ids, columns ascending) into caller-owned scratch Bufs
h2tap_status dyn_materialise(h2tap_dyn* d, Buf& bo, Buf& bc, Buf& bw) {
    h2tap_replica* r = d->r;
    cudaStream_t st = r->st;
    const uint64_t V = d->V, E = d->n_live;
    dyn::Ctr* c = dyn_ctr_reset(d);
    dyn_item_bufs(d, std::max<uint64_t>(E, 1));
    uint64_t* k = static_cast<uint64_t*>(d->keys.p);
    uint32_t* v = static_cast<uint32_t*>(d->vals.p);
    uint64_t* k2 = static_cast<uint64_t*>(d->keys2.p);
    uint32_t* v2 = static_cast<uint32_t*>(d->vals2.p);
    float* cw = static_cast<float*>(d->witem.p);
    if (V) {
        const unsigned grid = (unsigned)std::min<uint64_t>(g1(V), (uint64_t)r->n_sm * 16);
        dyn::k_dyn_compact<<<grid, 256, 0, st>>>(dyn_tabs(d), V, k, v, cw, c);
        CKL();
    }
    radix_sort(r, k, v, k2, v2, E, bits_for(V * V));
    int64_t* o_off = r->get<int64_t>(bo, V + 1);
    uint32_t* o_cols = r->get<uint32_t>(bc, E);
    float* o_w = r->get<float>(bw, E);
    if (E) { dyn::k_dyn_emit<<<g1(E), 256, 0, st>>>(k, v, cw, E, V, o_cols, o_w); CKL(); }
    dyn::k_dyn_offsets<<<g1(V + 1), 256, 0, st>>>(k, E, V, o_off);
    CKL();
    dyn_ctr_read(d);
    if (d->hctr->n_out != E) {
        set_err("tables hold %llu live keys, expected %llu", d->hctr->n_out, (unsigned long long)E);
        return H2TAP_E_CUDA;
    }
    return H2TAP_OK;
}

// dense id of a live vertex (or an error)
h2tap_status dyn_source(h2tap_dyn* d, uint64_t source_ext, uint64_t* out) {
    h2tap_replica* r = d->r;
    dyn::Ctr* c = dyn_ctr_reset(d);
    dyn::k_dyn_lookup<<<1, 32, 0, r->st>>>(static_cast<const uint64_t*>(d->ext.p),
                                           static_cast<const uint32_t*>(d->live.p), d->V, source_ext, c);
    CKL();
    dyn_ctr_read(d);
    if (!d->hctr->bad) { set_err("source %llu is not a live vertex", (unsigned long long)source_ext); return H2TAP_E_INVAL; }
    *out = d->hctr->bad - 1;
    return H2TAP_OK;
}

}  // namespace

extern "C" {

h2tap_status h2tap_dyn_create(const h2tap_config* cfg, size_t n_vertices, const uint64_t* vertex_ids,
                              size_t n_edges, const uint64_t* src, const uint64_t* dst, const float* w,
                              int on_device, h2tap_dyn** out) {
    if (!out) { set_err("out is NULL"); return H2TAP_E_INVAL; }
    *out = nullptr;
    if (n_edges && (!src || !dst)) { set_err("src/dst NULL"); return H2TAP_E_INVAL; }
    if (n_vertices >= 0xFFFFFFFEull || n_edges >= 0xFFFFFFFFull) { set_err("more than 2^32 - 3 vertices or 2^32 - 2 edges"); return H2TAP_E_CAPACITY; }
    if (cfg && (cfg->world > 1 || cfg->id_mode != H2TAP_ID_COMPACT)) {
        set_err("the dynamic replica is single-GPU with fixed dense ids (leave world / id_mode at 0)");
        return H2TAP_E_INVAL;
    }
    h2tap_dyn* d = new (std::nothrow) h2tap_dyn();
    if (!d) { set_err("host allocation failed"); return H2TAP_E_NOMEM; }
    const h2tap_status s = run_guarded(nullptr, [&]() -> h2tap_status {
        g_launches = g_h2d = g_d2h = 0;
        d->r = new_replica(cfg);
        h2tap_replica* r = d->r;
        CK(cudaHostAlloc(reinterpret_cast<void**>(&d->hctr), sizeof(dyn::Ctr), cudaHostAllocDefault));
        for (int e = 0; e < 4; ++e)
            if (!r->ev[e]) CK(cudaEventCreate(&r->ev[e]));
        for (auto& g : d->stg) CK(cudaEventCreateWithFlags(&g.ev, cudaEventDisableTiming));
        dyn_reserve_vertices(d, n_vertices);
        uint64_t* ext = static_cast<uint64_t*>(d->ext.p);
        if (vertex_ids) copy_in(r, ext, vertex_ids, n_vertices, on_device);
        else if (n_vertices) { k_iota_u64<<<g1(n_vertices), 256, 0, r->st>>>(ext, n_vertices); CKL(); }
        if (n_vertices) {
            dyn::k_dyn_fill_u32<<<g1(n_vertices), 256, 0, r->st>>>(static_cast<uint32_t*>(d->live.p), n_vertices, 1);
            CKL();
        }
        dyn::Ctr* c = dyn_ctr_reset(d);
        dyn::k_dyn_check_ids<<<g1(n_vertices), 256, 0, r->st>>>(ext, n_vertices, c);
        CKL();
        dyn_ctr_read(d);
        if (d->hctr->bad) { set_err("vertex ids not strictly increasing"); return H2TAP_E_INVAL; }
        d->V = n_vertices;
        if (n_vertices) {
            CK(cudaMemcpyAsync(&d->xid, ext + n_vertices - 1, 8, cudaMemcpyDeviceToHost, r->st));
            r->sync();
        }
        dyn_rebuild(d, 3 * n_edges);   // an empty slab with room for the edges' tables (load >= 1/4)
        if (n_edges) {
            dyn_item_bufs(d, n_edges);
            const uint64_t *s2 = src, *d2 = dst;
            const float* w2 = w;
            Buf bs, bd, bw;
            if (!on_device) {
                uint64_t* xs = r->get<uint64_t>(bs, n_edges);
                uint64_t* xd = r->get<uint64_t>(bd, n_edges);
                copy_in(r, xs, src, n_edges, 0);
                copy_in(r, xd, dst, n_edges, 0);
                s2 = xs; d2 = xd;
                if (w) { float* xw = r->get<float>(bw, n_edges); copy_in(r, xw, w, n_edges, 0); w2 = xw; }
            }
            dyn::k_dyn_expand_flat<<<g1(n_edges), 256, 0, r->st>>>(s2, d2, w2, n_edges, ext, d->V,
                                                                   static_cast<uint64_t*>(d->keys.p),
                                                                   static_cast<uint32_t*>(d->vals.p),
                                                                   static_cast<float*>(d->witem.p), c);
            CKL();
            dyn_ctr_read(d);
            r->release(bs); r->release(bd); r->release(bw);
            if (d->hctr->bad) { set_err("edge endpoint is not a vertex"); return H2TAP_E_INVAL; }
            dyn_upsert_items(d, n_edges, c);
            dyn_ctr_read(d);
            d->n_live = d->hctr->n_new;
            d->garbage = d->hctr->garbage;
        }
        r->sync();
        return H2TAP_OK;
    });
    if (s != H2TAP_OK) {
        try { dyn_free(d); } catch (...) {}
        return s;
    }
    *out = d;
    return H2TAP_OK;
}

h2tap_status h2tap_dyn_apply_records(h2tap_dyn* d, const h2tap_record_batch* batch, h2tap_apply_stats* stats) {
    if (!d || !batch) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(d->r, [&]() { return dyn_apply(d, batch, stats); });
}

h2tap_status h2tap_dyn_stage(h2tap_dyn* d, const h2tap_record_batch* host, h2tap_record_batch* staged) {
    if (!d || !host || !staged) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (host->on_device) { set_err("h2tap_dyn_stage takes a host batch"); return H2TAP_E_INVAL; }
    if (host->weights64) { set_err("the dynamic replica takes f32 weights"); return H2TAP_E_INVAL; }
    if ((host->n_records && !host->records) || (host->n_inserts && (!host->inserts || !host->weights)) ||
        (host->n_deletes && !host->deletes)) {
        set_err("null records/inserts/weights/deletes");
        return H2TAP_E_INVAL;
    }
    return run_guarded(d->r, [&]() -> h2tap_status {
        h2tap_replica* r = d->r;
        CK(cudaSetDevice(r->cfg.device));
        auto& g = d->stg[d->stg_next];
        d->stg_next ^= 1;
        CK(cudaEventSynchronize(g.ev));   // the slot's previous copy is done before a regrow
        DeltaRec* xr = r->get<DeltaRec>(g.rec, host->n_records);
        uint64_t* xi = r->get<uint64_t>(g.ins, host->n_inserts);
        float* xw = r->get<float>(g.wts, host->n_inserts);
        uint64_t* xd = r->get<uint64_t>(g.del, host->n_deletes);
        CK(cudaStreamSynchronize(r->st));   // slot buffers (re)allocated on the replica stream are ready
        cudaStream_t cs = r->st_copy;
        uint64_t bytes = 0;
        auto cp = [&](void* dst, const void* src, uint64_t nb) {
            if (!nb) return;
            CK(cudaMemcpyAsync(dst, src, nb, cudaMemcpyHostToDevice, cs));
            bytes += nb;
        };
        cp(xr, host->records, host->n_records * sizeof(DeltaRec));
        cp(xi, host->inserts, host->n_inserts * 8);
        cp(xw, host->weights, host->n_inserts * 4);
        cp(xd, host->deletes, host->n_deletes * 8);
        CK(cudaEventRecord(g.ev, cs));
        g.bytes = bytes;
        *staged = *host;
        staged->on_device = 1;
        staged->records = reinterpret_cast<const h2tap_delta_record*>(xr);
        staged->inserts = xi; staged->weights = xw; staged->deletes = xd;
        return H2TAP_OK;
    });
}

h2tap_status h2tap_dyn_info(const h2tap_dyn* d, uint64_t* n_vertices, uint64_t* n_edges, uint64_t* table_slots) {
    if (!d) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (n_vertices) *n_vertices = d->V;
    if (n_edges) *n_edges = d->n_live;
    if (table_slots) *table_slots = d->tail - d->garbage;
    return H2TAP_OK;
}

h2tap_status h2tap_dyn_export(h2tap_dyn* d, int64_t* offsets, uint32_t* cols, float* w, uint64_t* ext_ids,
                              uint8_t* live) {
    if (!d) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(d->r, [&]() -> h2tap_status {
        h2tap_replica* r = d->r;
        cudaStream_t st = r->st;
        const uint64_t V = d->V, E = d->n_live;
        Buf bo, bc, bw, bl;
        const h2tap_status s = dyn_materialise(d, bo, bc, bw);
        if (s != H2TAP_OK) return s;
        uint8_t* o_live = r->get<uint8_t>(bl, V);
        if (V) { dyn::k_dyn_live_u8<<<g1(V), 256, 0, st>>>(static_cast<uint32_t*>(d->live.p), V, o_live); CKL(); }
        if (offsets) CK(cudaMemcpyAsync(offsets, bo.p, (V + 1) * 8, cudaMemcpyDefault, st));
        if (cols && E) CK(cudaMemcpyAsync(cols, bc.p, E * 4, cudaMemcpyDefault, st));
        if (w && E) CK(cudaMemcpyAsync(w, bw.p, E * 4, cudaMemcpyDefault, st));
        if (ext_ids && V) CK(cudaMemcpyAsync(ext_ids, d->ext.p, V * 8, cudaMemcpyDefault, st));
        if (live && V) CK(cudaMemcpyAsync(live, o_live, V, cudaMemcpyDefault, st));
        r->sync();
        r->release(bo); r->release(bc); r->release(bw); r->release(bl);
        return H2TAP_OK;
    });
}

h2tap_status h2tap_dyn_bfs(h2tap_dyn* d, uint64_t source_ext, int32_t* level_out) {
    if (!d || !level_out) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(d->r, [&]() -> h2tap_status {
        h2tap_replica* r = d->r;
        cudaStream_t st = r->st;
        const uint64_t V = d->V;
        uint64_t src = 0;
        const h2tap_status e = dyn_source(d, source_ext, &src);
        if (e != H2TAP_OK) return e;
        int32_t* level = r->get<int32_t>(d->lvl, V);
        uint32_t* fa = r->get<uint32_t>(d->fa, V);
        uint32_t* fb = r->get<uint32_t>(d->fb, V);
        unsigned long long* cnt = r->get<unsigned long long>(r->misc, 1);
        k_fill_i32<<<g1(V), 256, 0, st>>>(level, V, -1);
        CKL();
        int32_t zero = 0;
        uint32_t s32 = (uint32_t)src;
        CK(cudaMemcpyAsync(level + src, &zero, 4, cudaMemcpyHostToDevice, st));
        CK(cudaMemcpyAsync(fa, &s32, 4, cudaMemcpyHostToDevice, st));
        uint64_t nf = 1;
        for (int32_t depth = 0; nf; ++depth) {   // level-synchronous, the tables read in place
            CK(cudaMemsetAsync(cnt, 0, 8, st));
            const unsigned grid = (unsigned)std::min<uint64_t>(cdiv(nf * 32, 256), (uint64_t)r->n_sm * 32);
            dyn::k_dyn_bfs_expand<<<grid, 256, 0, st>>>(dyn_tabs(d), fa, nf, level, depth, fb, cnt);
            CKL();
            unsigned long long h = 0;
            CK(cudaMemcpyAsync(&h, cnt, 8, cudaMemcpyDeviceToHost, st));
            r->sync();
            nf = h;
            std::swap(fa, fb);
        }
        CK(cudaMemcpyAsync(level_out, level, V * 4, cudaMemcpyDefault, st));
        r->sync();
        return H2TAP_OK;
    });
}

h2tap_status h2tap_dyn_pagerank(h2tap_dyn* d, double damping, int iterations, double* rank_out) {
    if (!d || !rank_out || iterations < 0) { set_err("bad argument"); return H2TAP_E_INVAL; }
    return run_guarded(d->r, [&]() -> h2tap_status {
        h2tap_replica* r = d->r;
        cudaStream_t st = r->st;
        const uint64_t V = d->V;
        if (V == 0) return H2TAP_OK;
        // the graph is the live vertices (dead ones keep an empty table and rank 0, D3)
        uint8_t* l8 = r->get<uint8_t>(d->live8, V);
        dyn::k_dyn_live_u8<<<g1(V), 256, 0, st>>>(static_cast<const uint32_t*>(d->live.p), V, l8);
        CKL();
        unsigned long long* c = r->get<unsigned long long>(r->misc, 2);
        CK(cudaMemsetAsync(c, 0, 16, st));
        k_count_u8<<<(unsigned)std::min<uint64_t>(g1(V), (uint64_t)r->n_sm * 8), 256, 0, st>>>(l8, V, c);
        CKL();
        unsigned long long nl = 0;
        CK(cudaMemcpyAsync(&nl, c, 8, cudaMemcpyDeviceToHost, st));
        r->sync();
        double* a = r->get<double>(d->da, V);
        double* b = r->get<double>(d->db, V);
        double* ds = reinterpret_cast<double*>(c + 1);
        if (nl == 0) {
            CK(cudaMemsetAsync(a, 0, V * 8, st));
        } else {
            k_pr_init<<<g1(V), 256, 0, st>>>(a, V, l8, nl);
            CKL();
            const unsigned gs = (unsigned)std::min<uint64_t>(g1(V), (uint64_t)r->n_sm * 8);
            const unsigned gw = (unsigned)std::min<uint64_t>(cdiv(V * 32, 256), (uint64_t)r->n_sm * 32);
            for (int it = 0; it < iterations; ++it) {
                CK(cudaMemsetAsync(ds, 0, 8, st));
                CK(cudaMemsetAsync(b, 0, V * 8, st));
                dyn::k_dyn_pr_dangling<<<gs, 256, 0, st>>>(static_cast<const uint32_t*>(d->cnt.p),
                                                           static_cast<const uint32_t*>(d->live.p), a, V, ds);
                dyn::k_dyn_pr_push<<<gw, 256, 0, st>>>(dyn_tabs(d), a, V, b);
                k_pr_finish<<<g1(V), 256, 0, st>>>(b, V, damping, ds, l8, nl);
                CKL();
                std::swap(a, b);
            }
        }
        CK(cudaMemcpyAsync(rank_out, a, V * 8, cudaMemcpyDefault, st));
        r->sync();
        return H2TAP_OK;
    });
}

h2tap_status h2tap_dyn_sssp(h2tap_dyn* d, uint64_t source_ext, double* dist_out) {
    if (!d || !dist_out) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(d->r, [&]() -> h2tap_status {
        h2tap_replica* r = d->r;
        cudaStream_t st = r->st;
        const uint64_t V = d->V;
        uint64_t src = 0;
        const h2tap_status e = dyn_source(d, source_ext, &src);
        if (e != H2TAP_OK) return e;
        dyn::Ctr* c = dyn_ctr_reset(d);
        dyn::k_dyn_check_w<<<(unsigned)std::min<uint64_t>(cdiv(V * 32, 256), (uint64_t)r->n_sm * 16), 256, 0, st>>>(
            dyn_tabs(d), V, c);
        CKL();
        dyn_ctr_read(d);
        if (d->hctr->bad_w) { set_err("h2tap_dyn_sssp: negative or NaN edge weight"); return H2TAP_E_INVAL; }
        double* dist = r->get<double>(d->da, V);
        uint32_t* stamp = reinterpret_cast<uint32_t*>(r->get<double>(d->db, V));
        uint32_t* fa = r->get<uint32_t>(d->fa, V);
        uint32_t* fb = r->get<uint32_t>(d->fb, V);
        unsigned long long* cnt = r->get<unsigned long long>(r->misc, 1);
        k_fill_u64<<<g1(V), 256, 0, st>>>(reinterpret_cast<uint64_t*>(dist), V, 0x7FF0000000000000ull);  // +inf
        CKL();
        CK(cudaMemsetAsync(stamp, 0, V * 4, st));
        const double zero = 0.0;
        const uint32_t s32 = (uint32_t)src;
        CK(cudaMemcpyAsync(dist + src, &zero, 8, cudaMemcpyHostToDevice, st));
        CK(cudaMemcpyAsync(fa, &s32, 4, cudaMemcpyHostToDevice, st));
        uint64_t nf = 1;
        for (uint32_t round = 1; nf; ++round) {
            CK(cudaMemsetAsync(cnt, 0, 8, st));
            const unsigned grid = (unsigned)std::min<uint64_t>(cdiv(nf * 32, 256), (uint64_t)r->n_sm * 32);
            dyn::k_dyn_sssp_relax<<<grid, 256, 0, st>>>(dyn_tabs(d), fa, nf, reinterpret_cast<unsigned long long*>(dist),
                                                        stamp, round, fb, cnt);
            CKL();
            unsigned long long h = 0;
            CK(cudaMemcpyAsync(&h, cnt, 8, cudaMemcpyDeviceToHost, st));
            r->sync();
            nf = h;
            std::swap(fa, fb);
        }
        CK(cudaMemcpyAsync(dist_out, dist, V * 8, cudaMemcpyDefault, st));
        r->sync();
        return H2TAP_OK;
    });
}

void h2tap_dyn_destroy(h2tap_dyn* d) {
    try { dyn_free(d); } catch (...) {}
}

}  // extern "C"
