// dyn.cuh - the dynamic replica: Algorithm 1 (§5.4 "Dynamic
// Data Structures") ingesting one cycle's delta records into a GPU hash-table
// graph, included by h2tap.cu (shares its allocator, stream, radix sort and record layout).
//
// Storage: one open-addressing table over packed edge keys
//   key = src_dense << 32 | dst_dense  (u64; EMPTY = ~0, TOMB = ~0 - 1), value f32
// linear probing from fmix64(key), load (live + tombstones) <= 0.7 (re-hashed into a table of
// twice the needed size when a cycle would pass it); inserts only ever claim EMPTY slots, so a
// CAS on the key word is the whole synchronisation.  Vertices: ext ids ascending (new IDs are
// > xid, Alg. 1 line 5/8, so they append) and a u32 liveness word per dense id (D3: dense ids
// never move, dead ones keep an empty row).
//
// One cycle (h2tap_dyn_apply_records), all on the replica stream:
//   k_dyn_rec        classify records (lines 2-9): deletion / new-node queues, per-record
//                    insert / delete item counts (+ record validation)
//   scan             item offsets, inserts and deletes packed in one u64 (k_scan_exclusive_u64)
//   new nodes        radix sort of the new IDs, k_dyn_kill (created and deleted in the same
//                    cycle: D3), k_dyn_heads + scan + k_dyn_append (line 10)
//   k_dyn_expand_ins thread per record (warp per large record): resolve endpoints, gate (D2), pack keys
//   radix sort       (key, item) - stable, so the last item of a key is the latest (D1)
//   k_dyn_upsert     last item of each key: CAS-insert or overwrite (lines 6, 10)
//   k_dyn_delete     thread per record (warp per large record): probe + CAS to TOMB (line 7)
//   k_dyn_node_del   liveness off (line 11) + k_dyn_cascade over the table if any died
// Export materialises the CSR: k_dyn_compact (warp-aggregated) + radix sort + k_dyn_emit +
// k_dyn_offsets.  The cost of a cycle is O(batch) plus O(table) only for node deletes.

namespace dyn {

constexpr uint64_t kEmpty = ~0ull, kTomb = ~0ull - 1;
constexpr uint32_t kFilterBits = 1u << 18;   // cascade filter: 32 KB of shared memory

struct Ctr {
    unsigned long long n_new_ids, n_del_ids, bad, max_new, n_new, n_upd, n_del, n_casc, n_gated, n_vdel, n_out, last_ext, n_big_ins, n_big_del, sum_ins, sum_del;
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

// insert-only probe into EMPTY slots; keys are unique within a launch
__device__ __forceinline__ bool table_put(uint64_t* hk, float* hv, uint64_t mask, uint64_t k, float w) {
    uint64_t h = hmix(k) & mask;
    while (true) {
        uint64_t cur = *((volatile uint64_t*)&hk[h]);
        if (cur == k) { hv[h] = w; return false; }
        if (cur == kEmpty) {
            cur = atomicCAS((unsigned long long*)&hk[h], (unsigned long long)kEmpty, (unsigned long long)k);
            if (cur == kEmpty || cur == k) { hv[h] = w; return cur == kEmpty; }
        }
        h = (h + 1) & mask;
    }
}

__global__ void k_dyn_upsert(const uint64_t* __restrict__ sk, const uint32_t* __restrict__ sv, uint64_t n,
                             const float* __restrict__ witem, uint64_t V, uint64_t* hk, float* hv, uint64_t mask,
                             Ctr* __restrict__ c) {
    const uint64_t key_bad = V * V;
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    bool nw = false, up = false;
    if (i < n) {
        const uint64_t k = sk[i];
        if (k < key_bad && (i + 1 == n || sk[i + 1] != k)) {   // D1: the latest item of its key
            const uint64_t s = k / V;
            nw = table_put(hk, hv, mask, s << 32 | (k - s * V), witem[sv[i]]);
            up = !nw;
        }
    }
    wadd(&c->n_new, nw);
    wadd(&c->n_upd, up);
}

__device__ __forceinline__ bool del_item(int64_t s, uint64_t x, const uint64_t* __restrict__ ext, uint64_t V,
                                         uint64_t* hk, uint64_t mask) {
    const int64_t d = find_ext(ext, V, x);
    if (d < 0) return false;
    const uint64_t k = (uint64_t)s << 32 | (uint64_t)d;
    uint64_t h = hmix(k) & mask;
    while (true) {
        const uint64_t cur = *((volatile uint64_t*)&hk[h]);
        if (cur == k)
            return atomicCAS((unsigned long long*)&hk[h], (unsigned long long)k, (unsigned long long)kTomb) == k;
        if (cur == kEmpty) return false;
        h = (h + 1) & mask;
    }
}
// line 7: the records' deleted edges to TOMB; passes as in k_dyn_expand_ins
template <int kPass>
__global__ void __launch_bounds__(256) k_dyn_delete(const DeltaRec* __restrict__ rec, uint64_t nr,
        const uint64_t* __restrict__ off, const uint64_t* __restrict__ del, const uint64_t* __restrict__ ext,
        uint64_t V, uint64_t* hk, uint64_t mask, uint64_t* __restrict__ big, unsigned long long* __restrict__ n_big,
        Ctr* __restrict__ c) {
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
                    for (uint64_t j = 0; j < n; ++j) hits += del_item(s, del[r.del_off + j], ext, V, hk, mask);
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
            for (uint64_t j = lane; j < n; j += 32) hits += del_item(s, del[dO + j], ext, V, hk, mask);
        }
    }
    hits = warp_sum<unsigned long long>(hits);
    if ((threadIdx.x & 31) == 0 && hits) atomicAdd(&c->n_del, hits);
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

// every table key had two live endpoints before this cycle's node deletes, so a key is
// removed iff an endpoint died this cycle (bitmap, V/8 bytes, L2-resident); 2 slots/thread
// a 32 KB filter (bit v mod 2^18 of every dead vertex) in shared memory screens the keys;
// the exact bitmap is read only on a filter hit
__device__ __forceinline__ bool died_of(const uint32_t* __restrict__ b, const uint32_t* __restrict__ filt, uint64_t k) {
    const uint64_t s = k >> 32, d = k & 0xffffffffu;
    const uint32_t fs = (uint32_t)s & (kFilterBits - 1), fd = (uint32_t)d & (kFilterBits - 1);
    if ((((filt[fs >> 5] >> (fs & 31)) | (filt[fd >> 5] >> (fd & 31))) & 1u) == 0) return false;
    return ((__ldg(b + (s >> 5)) >> (s & 31)) | (__ldg(b + (d >> 5)) >> (d & 31))) & 1u;
}
__global__ void __launch_bounds__(256, 4) k_dyn_cascade(uint64_t* __restrict__ hk, uint64_t cap,
        const uint32_t* __restrict__ died_bits, const uint32_t* __restrict__ filter, Ctr* __restrict__ c) {
    if (*(volatile unsigned long long*)&c->n_vdel == 0) return;   // nobody died this cycle (no host sync)
    extern __shared__ uint32_t filt[];
    for (uint32_t t = threadIdx.x; t < kFilterBits / 32; t += blockDim.x) filt[t] = filter[t];
    __syncthreads();
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x, half = cap >> 1;
    ulonglong2* h2 = reinterpret_cast<ulonglong2*>(hk);
    unsigned long long gone = 0;
    constexpr int U = 4;   // 4 independent 16-byte loads in flight per thread
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    for (; i + (U - 1) * stride < half; i += U * stride) {
        ulonglong2 k[U];
#pragma unroll
        for (int u = 0; u < U; ++u) k[u] = __ldcs(h2 + i + u * stride);
#pragma unroll
        for (int u = 0; u < U; ++u) {
            bool w = false;
            if (k[u].x < kTomb && died_of(died_bits, filt, k[u].x)) { k[u].x = kTomb; w = true; ++gone; }
            if (k[u].y < kTomb && died_of(died_bits, filt, k[u].y)) { k[u].y = kTomb; w = true; ++gone; }
            if (w) h2[i + u * stride] = k[u];
        }
    }
    for (; i < half; i += stride) {
        ulonglong2 k = h2[i];
        bool w = false;
        if (k.x < kTomb && died_of(died_bits, filt, k.x)) { k.x = kTomb; w = true; ++gone; }
        if (k.y < kTomb && died_of(died_bits, filt, k.y)) { k.y = kTomb; w = true; ++gone; }
        if (w) h2[i] = k;
    }
    gone = warp_sum<unsigned long long>(gone);
    if ((threadIdx.x & 31) == 0 && gone) atomicAdd(&c->n_casc, gone);
}

__global__ void k_dyn_rehash(const uint64_t* __restrict__ ok, const float* __restrict__ ov, uint64_t ocap,
                             uint64_t* hk, float* hv, uint64_t mask) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < ocap; i += stride) {
        const uint64_t k = ok[i];
        if (k < kTomb) table_put(hk, hv, mask, k, ov[i]);
    }
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

// export
__global__ void k_dyn_compact(const uint64_t* __restrict__ hk, const float* __restrict__ hv, uint64_t cap,
                              uint64_t V, uint64_t* __restrict__ ok, uint32_t* __restrict__ oi, float* __restrict__ ow,
                              Ctr* __restrict__ c) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const unsigned lane = threadIdx.x & 31;
    for (uint64_t i0 = blockIdx.x * (uint64_t)blockDim.x; i0 < cap; i0 += stride) {
        const uint64_t i = i0 + threadIdx.x;
        const uint64_t k = i < cap ? hk[i] : kEmpty;
        const bool keep = k < kTomb;
        const unsigned m = __ballot_sync(0xffffffffu, keep);
        unsigned long long base = 0;
        if (lane == 0 && m) base = atomicAdd(&c->n_out, (unsigned long long)__popc(m));
        base = __shfl_sync(0xffffffffu, base, 0);
        if (keep) {
            const uint64_t p = base + __popc(m & ((1u << lane) - 1));
            ok[p] = (k >> 32) * V + (k & 0xffffffffu);   // sort key
            oi[p] = (uint32_t)p;
            ow[p] = hv[i];
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
    uint64_t V = 0, n_live = 0, n_tomb = 0, cap = 0, xid = 0;   // xid = ext[V - 1] (host copy)
    Buf ext, live, hk, hv, died, big;
    Buf cin, oin, new_ids, del_ids, kill, flag, fpos, keys, vals, keys2, vals2, witem, ctr, xo;
    Buf x_rec, x_ins, x_wts, x_del;
    dyn::Ctr* hctr = nullptr;     // pinned host mirror
};

namespace {

void dyn_free(h2tap_dyn* d) {
    if (!d) return;
    if (d->r) {
        for (Buf* b : {&d->ext, &d->live, &d->died, &d->big, &d->hk, &d->hv, &d->cin, &d->oin, &d->new_ids,
                       &d->del_ids, &d->kill, &d->flag, &d->fpos, &d->keys, &d->vals, &d->keys2, &d->vals2,
                       &d->witem, &d->ctr, &d->xo, &d->x_rec, &d->x_ins, &d->x_wts, &d->x_del})
            if (b->p) d->r->dfree(b->p);
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

// grow ext / live to hold n dense ids (contents kept)
void dyn_reserve_vertices(h2tap_dyn* d, uint64_t n) {
    h2tap_replica* r = d->r;
    if (d->ext.cap >= (n + 16) * 8 && d->live.cap >= (n + 16) * 4) return;
    const uint64_t want = std::max<uint64_t>(n, 2 * d->V) + 1024;
    Buf e2, l2;
    r->get<uint64_t>(e2, want);
    r->get<uint32_t>(l2, want);
    if (d->V) {
        CK(cudaMemcpyAsync(e2.p, d->ext.p, d->V * 8, cudaMemcpyDeviceToDevice, r->st));
        CK(cudaMemcpyAsync(l2.p, d->live.p, d->V * 4, cudaMemcpyDeviceToDevice, r->st));
    }
    r->release(d->ext);
    r->release(d->live);
    d->ext = e2;
    d->live = l2;
}

uint64_t pow2_at_least(uint64_t x) {
    uint64_t c = 1024;
    while (c < x) c <<= 1;
    return c;
}

// make room for `incoming` more keys at load <= 0.7 (tombstones count as used); a re-hash
// sizes for load <= 0.7 as well, so after it the load is 0.35-0.7 (the cascade pass of a
// node delete streams the whole table: a denser table is a shorter pass)
void dyn_reserve_table(h2tap_dyn* d, uint64_t incoming) {
    h2tap_replica* r = d->r;
    if (d->cap && 10 * (d->n_live + d->n_tomb + incoming) <= 7 * d->cap) return;
    const uint64_t nc = pow2_at_least((10 * (d->n_live + incoming)) / 7 + 1);
    Buf k2, v2;
    uint64_t* nk = r->get<uint64_t>(k2, nc);
    float* nv = r->get<float>(v2, nc);
    CK(cudaMemsetAsync(nk, 0xFF, nc * 8, r->st));
    if (d->cap && d->n_live) {
        const unsigned grid = (unsigned)std::min<uint64_t>(g1(d->cap), (uint64_t)r->n_sm * 8);
        dyn::k_dyn_rehash<<<grid, 256, 0, r->st>>>(static_cast<uint64_t*>(d->hk.p), static_cast<float*>(d->hv.p),
                                                   d->cap, nk, nv, nc - 1);
        CKL();
    }
    r->release(d->hk);
    r->release(d->hv);
    d->hk = k2;
    d->hv = v2;
    d->cap = nc;
    d->n_tomb = 0;
}

// sort (keys, item) items and upsert the latest item of every key; n items, keys < V' << 32
void dyn_upsert_items(h2tap_dyn* d, uint64_t n, dyn::Ctr* c) {
    h2tap_replica* r = d->r;
    if (!n) return;
    uint64_t* k = static_cast<uint64_t*>(d->keys.p);
    uint32_t* v = static_cast<uint32_t*>(d->vals.p);
    uint64_t* k2 = static_cast<uint64_t*>(d->keys2.p);
    uint32_t* v2 = static_cast<uint32_t*>(d->vals2.p);
    radix_sort(r, k, v, k2, v2, n, bits_for(d->V * d->V));
    dyn::k_dyn_upsert<<<g1(n), 256, 0, r->st>>>(k, v, n, static_cast<float*>(d->witem.p), d->V,
                                                static_cast<uint64_t*>(d->hk.p), static_cast<float*>(d->hv.p),
                                                d->cap - 1, c);
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
        dyn_reserve_table(d, n_ins);
        dyn_upsert_items(d, n_ins, c);
    }
    // ---- line 7: delete batch
    if (tot[1] && d->cap) {
        uint64_t* big = r->get<uint64_t>(d->big, nr);
        uint64_t* hk = static_cast<uint64_t*>(d->hk.p);
        dyn::k_dyn_delete<0><<<g1(nr), 256, 0, st>>>(rec, nr, odel, del, ext, d->V, hk, d->cap - 1, big, &c->n_big_del, c);
        CKL();
        dyn::k_dyn_delete<1><<<wgrid, 256, 0, st>>>(rec, nr, odel, del, ext, d->V, hk, d->cap - 1, big, &c->n_big_del, c);
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
        if (d->cap) {
            constexpr int smem = dyn::kFilterBits / 8;
            CK(cudaFuncSetAttribute(dyn::k_dyn_cascade, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
            const unsigned grid = (unsigned)std::min<uint64_t>(g1(d->cap / 2), (uint64_t)r->n_sm * 4);  // 4 CTAs/SM
            CK(cudaEventRecord(r->ev[2], st));
            dyn::k_dyn_cascade<<<grid, 256, smem, st>>>(static_cast<uint64_t*>(d->hk.p), d->cap, died, filter, c);
            CKL();
            CK(cudaEventRecord(r->ev[3], st));
            casc_timed = true;
        }
    }
    CK(cudaEventRecord(r->ev[1], st));
    dyn_ctr_read(d);
    const dyn::Ctr& h = *d->hctr;
    d->n_live = d->n_live + h.n_new - h.n_del - h.n_casc;
    d->n_tomb += h.n_del + h.n_casc;
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
            stats->bytes_merge = d->cap * 8;
        }
        // algorithmic bytes: records + slices read, one 12-byte slot touch per item
        stats->bytes_alg = nr * sizeof(DeltaRec) + n_ins * 12 + tot[1] * 8 + (n_ins + tot[1]) * 12;
        stats->n_launches = g_launches;
        stats->h2d_bytes = g_h2d;
        stats->d2h_bytes = g_d2h;
    }
    return H2TAP_OK;
}

// the CSR of the table (rows = dense ids, columns ascending) into caller-owned scratch Bufs
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
    if (d->cap) {
        const unsigned grid = (unsigned)std::min<uint64_t>(g1(d->cap), (uint64_t)r->n_sm * 8);
        dyn::k_dyn_compact<<<grid, 256, 0, st>>>(static_cast<uint64_t*>(d->hk.p), static_cast<float*>(d->hv.p),
                                                 d->cap, V, k, v, cw, c);
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
        set_err("table holds %llu live keys, expected %llu", d->hctr->n_out, (unsigned long long)E);
        return H2TAP_E_CUDA;
    }
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
    if (n_vertices >= 0xFFFFFFFFull || n_edges >= 0xFFFFFFFFull) { set_err("more than 2^32 - 2 vertices or edges"); return H2TAP_E_CAPACITY; }
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
        if (!r->ev[0]) CK(cudaEventCreate(&r->ev[0]));
        for (int e = 1; e < 4; ++e)
            if (!r->ev[e]) CK(cudaEventCreate(&r->ev[e]));
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
        dyn_reserve_table(d, n_edges);
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

h2tap_status h2tap_dyn_info(const h2tap_dyn* d, uint64_t* n_vertices, uint64_t* n_edges, uint64_t* table_slots) {
    if (!d) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (n_vertices) *n_vertices = d->V;
    if (n_edges) *n_edges = d->n_live;
    if (table_slots) *table_slots = d->cap;
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
        const uint64_t* ext = static_cast<const uint64_t*>(d->ext.p);
        // source: dense id of a live vertex (host binary search over a copy is avoided:
        // one device lookup through the counters block)
        dyn::Ctr* c = dyn_ctr_reset(d);
        dyn::k_dyn_lookup<<<1, 32, 0, st>>>(ext, static_cast<const uint32_t*>(d->live.p), V, source_ext, c);
        CKL();
        dyn_ctr_read(d);
        if (!d->hctr->bad) { set_err("BFS source %llu is not a live vertex", (unsigned long long)source_ext); return H2TAP_E_INVAL; }
        const uint64_t src = d->hctr->bad - 1;
        Buf bo, bc, bw, bl, fa_, fb_;
        const h2tap_status s = dyn_materialise(d, bo, bc, bw);
        if (s != H2TAP_OK) return s;
        int32_t* level = r->get<int32_t>(bl, V);
        uint32_t* fa = r->get<uint32_t>(fa_, V);
        uint32_t* fb = r->get<uint32_t>(fb_, V);
        unsigned long long* cnt = r->get<unsigned long long>(r->misc, 1);
        k_fill_i32<<<g1(V), 256, 0, st>>>(level, V, -1);
        CKL();
        int32_t zero = 0;
        uint32_t s32 = (uint32_t)src;
        CK(cudaMemcpyAsync(level + src, &zero, 4, cudaMemcpyHostToDevice, st));
        CK(cudaMemcpyAsync(fa, &s32, 4, cudaMemcpyHostToDevice, st));
        uint64_t nf = 1;
        for (int32_t depth = 0; nf; ++depth) {   // the CSR path's level-synchronous expansion
            CK(cudaMemsetAsync(cnt, 0, 8, st));
            const unsigned grid = (unsigned)std::min<uint64_t>(cdiv(nf * 32, 256), 148 * 32);
            k_bfs_expand<<<grid, 256, 0, st>>>(static_cast<const int64_t*>(bo.p), static_cast<const uint32_t*>(bc.p),
                                               fa, nf, level, depth, fb, cnt);
            CKL();
            unsigned long long h = 0;
            CK(cudaMemcpyAsync(&h, cnt, 8, cudaMemcpyDeviceToHost, st));
            r->sync();
            nf = h;
            std::swap(fa, fb);
        }
        CK(cudaMemcpyAsync(level_out, level, V * 4, cudaMemcpyDefault, st));
        r->sync();
        for (Buf* b : {&bo, &bc, &bw, &bl, &fa_, &fb_}) r->release(*b);
        return H2TAP_OK;
    });
}

void h2tap_dyn_destroy(h2tap_dyn* d) {
    try { dyn_free(d); } catch (...) {}
}

}  // extern "C"
