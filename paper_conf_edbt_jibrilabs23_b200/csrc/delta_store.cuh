// delta_store.cuh - the paper's append-only delta store (§5.1, Fig. 2) as a
// native host component with a device mirror, and the propagation cycle that scans it
// (§5.2-§5.3), included by h2tap.cu.
//
// Host side (what committing transactions touch): a delta table of fixed-size chunks of
// 48-byte delta records (a linked list of chunks in the paper; here a fixed table of chunk
// pointers, so a reader never races a growing list) plus the inserts / weights / deletes
// arrays, chunked the same way, with the paper's 8-byte weights.  Appends are append-only
// and thread-safe: one short critical section reserves the record slot and the payload
// ranges in the same order (so payload offsets grow with the record index), the payload
// and the record are written outside it, and records are published in index order.
// Chunks live in pinned memory so the copies to the GPU are DMA.
//
// Device side: a mirror of the still-unconsumed tail of the store.  A cycle
// (h2tap_delta_apply_store) scans [cursor, end): `end` stops before the trailing 1024-record
// blocks whose every record has ts > snapshot_ts (they are invisible, so the scan
// can leave them to the next cycle); their copy to the mirror starts on the store's copy
// stream while this cycle is applied (read-ahead).  The scan itself is the records path:
// k_rec_count / k_rec_expand with the visibility bound (valid and ts <= snapshot_ts), then
// the flat pipeline.  When the cycle succeeded, k_rec_consume marks every record it used
// invalid in the mirror (each delta is used once, "by the end of the delta store
// scan") and finds the first record still pending; host chunks wholly before it
// are released and the mirror is compacted.  On any error nothing is marked.

struct h2tap_delta_store {
    static constexpr uint64_t kMaxChunks = 1u << 16, kBlock = 1024;
    int device = 0;
    uint64_t crec = 0, cpay = 0;  // records / payload elements per chunk (powers of two)
    std::mutex mu;                 // reservation + chunk allocation
    std::atomic<DeltaRec*> rch[kMaxChunks];
    std::atomic<std::atomic<uint64_t>*> bmin[kMaxChunks];  // per 1024-record block: min ts
    std::atomic<uint64_t*> ich[kMaxChunks];
    std::atomic<double*> wch[kMaxChunks];
    std::atomic<uint64_t*> dch[kMaxChunks];
    uint64_t n_res = 0, ins_res = 0, del_res = 0;  // reserved (under mu)
    std::atomic<uint64_t> n_pub{0}, pub_ins{0}, pub_del{0};
    // consumption and mirror state (the propagating thread only)
    uint64_t cursor = 0, cur_ins = 0, cur_del = 0;  // first record that may still be valid
    uint64_t snap = 0;                                // snapshot of the last successful scan
    uint64_t mbase = 0, mlen = 0, mcap = 0;           // mirror holds records [mbase, mbase + mlen)
    uint64_t ibase = 0, ilen = 0, icap = 0, wcap = 0, dbase = 0, dlen = 0, dcap = 0;
    DeltaRec* m_rec = nullptr, *m_rec2 = nullptr;
    uint64_t *m_ins = nullptr, *m_del = nullptr, *m_ins2 = nullptr, *m_del2 = nullptr;
    double* m_w = nullptr, *m_w2 = nullptr;
    uint64_t freed_r = 0, freed_i = 0, freed_d = 0;   // host chunks released below these
    cudaStream_t cs = nullptr;
    cudaEvent_t ev = nullptr;
    std::mutex free_mu;                 // recycled pinned chunks by size class:
    std::vector<void*> free_chunks[3];  // records, 8-byte payload, (unused)
    int chunk_class(size_t bytes) const { return bytes == crec * sizeof(DeltaRec) ? 0 : 1; }
    h2tap_delta_store() {
        for (uint64_t i = 0; i < kMaxChunks; ++i) { rch[i] = nullptr; bmin[i] = nullptr; ich[i] = nullptr; wch[i] = nullptr; dch[i] = nullptr; }
    }
};

namespace {

// the mirror's compaction: up to four arrays (records, inserts, weights, deletes) moved to
// their twin buffers in one launch, 8-byte words, grid-stride
struct DsMove {
    const uint64_t* src[4];
    uint64_t* dst[4];
    uint64_t words[4];
};
__global__ void k_ds_move(DsMove m) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
#pragma unroll
    for (int k = 0; k < 4; ++k)
        for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m.words[k]; i += stride)
            m.dst[k][i] = __ldcs(m.src[k] + i);
}

// pinned chunks are recycled (cudaHostAlloc / cudaFreeHost cost milliseconds and synchronise):
// a released chunk goes to its size class's free list and the next reservation takes it
template <typename T>
T* host_chunk(h2tap_delta_store* s, uint64_t n) {
    void* p = nullptr;
    {
        std::lock_guard<std::mutex> g(s->free_mu);
        std::vector<void*>& f = s->free_chunks[s->chunk_class(n * sizeof(T))];
        if (!f.empty()) { p = f.back(); f.pop_back(); }
    }
    if (!p) CK(cudaHostAlloc(&p, n * sizeof(T), cudaHostAllocPortable));
    return static_cast<T*>(p);
}
void release_chunk(h2tap_delta_store* s, void* p, size_t bytes) {
    if (!p) return;
    std::lock_guard<std::mutex> g(s->free_mu);
    s->free_chunks[s->chunk_class(bytes)].push_back(p);
}

// under s->mu: chunks for records [r0, r1) and payload [i0, i1), [d0, d1)
void ds_reserve_chunks(h2tap_delta_store* s, uint64_t r0, uint64_t r1, uint64_t i0, uint64_t i1, uint64_t d0,
                       uint64_t d1) {
    if ((r1 + s->crec - 1) / s->crec > s->kMaxChunks || (i1 + s->cpay - 1) / s->cpay > s->kMaxChunks ||
        (d1 + s->cpay - 1) / s->cpay > s->kMaxChunks) {
        set_err("delta store full (%llu chunks)", (unsigned long long)s->kMaxChunks);
        throw Fail{H2TAP_E_CAPACITY};
    }
    for (uint64_t c = r0 / s->crec; c * s->crec < r1; ++c)
        if (!s->rch[c].load()) {
            const uint64_t nb = s->crec / s->kBlock;
            auto* bm = new std::atomic<uint64_t>[nb];
            for (uint64_t b = 0; b < nb; ++b) bm[b] = ~0ull;
            s->bmin[c].store(bm);
            s->rch[c].store(host_chunk<DeltaRec>(s, s->crec));
        }
    for (uint64_t c = i0 / s->cpay; c * s->cpay < i1; ++c)
        if (!s->ich[c].load()) { s->ich[c].store(host_chunk<uint64_t>(s, s->cpay)); s->wch[c].store(host_chunk<double>(s, s->cpay)); }
    for (uint64_t c = d0 / s->cpay; c * s->cpay < d1; ++c)
        if (!s->dch[c].load()) s->dch[c].store(host_chunk<uint64_t>(s, s->cpay));
}

// copy n elements starting at absolute position a of a chunked host array into dst
template <typename T, typename A>
void ds_gather(const h2tap_delta_store* s, const A* chunks, uint64_t csize, uint64_t a, uint64_t n, T* dst, bool h2d,
               cudaStream_t cs) {
    while (n) {
        const uint64_t c = a / csize, o = a % csize, k = std::min(n, csize - o);
        const T* src = chunks[c].load() + o;
        if (h2d) CK(cudaMemcpyAsync(dst, src, k * sizeof(T), cudaMemcpyHostToDevice, cs));
        else std::memcpy(dst, src, k * sizeof(T));
        dst += k; a += k; n -= k;
    }
}
template <typename T, typename A>
void ds_scatter(h2tap_delta_store* s, A* chunks, uint64_t csize, uint64_t a, uint64_t n, const T* src) {
    while (n) {
        const uint64_t c = a / csize, o = a % csize, k = std::min(n, csize - o);
        std::memcpy(chunks[c].load() + o, src, k * sizeof(T));
        src += k; a += k; n -= k;
    }
}

void ds_publish(h2tap_delta_store* s, uint64_t first, uint64_t n, uint64_t ins_end, uint64_t del_end) {
    while (s->n_pub.load(std::memory_order_acquire) != first) std::this_thread::yield();  // in index order
    s->pub_ins.store(ins_end, std::memory_order_relaxed);
    s->pub_del.store(del_end, std::memory_order_relaxed);
    s->n_pub.store(first + n, std::memory_order_release);
}

void ds_note_ts(h2tap_delta_store* s, uint64_t idx, uint64_t ts) {
    std::atomic<uint64_t>& m = s->bmin[idx / s->crec].load()[(idx % s->crec) / s->kBlock];
    uint64_t cur = m.load(std::memory_order_relaxed);
    while (ts < cur && !m.compare_exchange_weak(cur, ts, std::memory_order_relaxed)) {}
}

// device mirror array + its compaction twin (the window moves between the two): grown 2x, rarely
template <typename T>
void ds_grow(T*& p, T*& p2, uint64_t& cap, uint64_t keep, uint64_t need) {
    if (need <= cap) return;
    const uint64_t nc = std::max<uint64_t>(2 * need, 1024);
    T* q = nullptr;
    CK(cudaMalloc(&q, nc * sizeof(T)));
    if (keep) CK(cudaMemcpy(q, p, keep * sizeof(T), cudaMemcpyDeviceToDevice));
    if (p) CK(cudaFree(p));
    if (p2) CK(cudaFree(p2));
    p = q;
    CK(cudaMalloc(&p2, nc * sizeof(T)));
    cap = nc;
}

// mirror records [mbase + mlen, upto) and their payload (async on s->cs); returns bytes
uint64_t ds_mirror(h2tap_delta_store* s, uint64_t upto, uint64_t ins_upto, uint64_t del_upto) {
    uint64_t bytes = 0;
    const uint64_t r0 = s->mbase + s->mlen, i0 = s->ibase + s->ilen, d0 = s->dbase + s->dlen;
    if (upto > r0) {
        ds_gather(s, s->rch, s->crec, r0, upto - r0, s->m_rec + s->mlen, true, s->cs);
        bytes += (upto - r0) * sizeof(DeltaRec);
        s->mlen = upto - s->mbase;
    }
    if (ins_upto > i0) {
        ds_gather(s, s->ich, s->cpay, i0, ins_upto - i0, s->m_ins + s->ilen, true, s->cs);
        ds_gather(s, s->wch, s->cpay, i0, ins_upto - i0, s->m_w + s->ilen, true, s->cs);
        bytes += (ins_upto - i0) * 16;
        s->ilen = ins_upto - s->ibase;
    }
    if (del_upto > d0) {
        ds_gather(s, s->dch, s->cpay, d0, del_upto - d0, s->m_del + s->dlen, true, s->cs);
        bytes += (del_upto - d0) * 8;
        s->dlen = del_upto - s->dbase;
    }
    return bytes;
}

// the payload positions at record boundary i (cursor <= i <= n_pub)
void ds_pos(const h2tap_delta_store* s, uint64_t i, uint64_t n_pub, uint64_t pins, uint64_t pdel, uint64_t* io,
            uint64_t* dq) {
    if (i >= n_pub) { *io = pins; *dq = pdel; return; }
    const DeltaRec& r = s->rch[i / s->crec].load()[i % s->crec];
    *io = r.ins_off;
    *dq = r.del_off;
}

void ds_release_below(h2tap_delta_store* s, uint64_t rec_lo, uint64_t ins_lo, uint64_t del_lo) {
    for (; (s->freed_r + 1) * s->crec <= rec_lo; ++s->freed_r) {
        release_chunk(s, s->rch[s->freed_r].exchange(nullptr), s->crec * sizeof(DeltaRec));
        delete[] s->bmin[s->freed_r].exchange(nullptr);
    }
    for (; (s->freed_i + 1) * s->cpay <= ins_lo; ++s->freed_i) {
        release_chunk(s, s->ich[s->freed_i].exchange(nullptr), s->cpay * 8);
        release_chunk(s, s->wch[s->freed_i].exchange(nullptr), s->cpay * 8);
    }
    for (; (s->freed_d + 1) * s->cpay <= del_lo; ++s->freed_d)
        release_chunk(s, s->dch[s->freed_d].exchange(nullptr), s->cpay * 8);
}

}  // namespace

extern "C" {

h2tap_status h2tap_ds_create(int device, size_t chunk_records, h2tap_delta_store** out) {
    if (!out) { set_err("null argument"); return H2TAP_E_INVAL; }
    *out = nullptr;
    uint64_t cr = 1024;
    while (cr < chunk_records) cr <<= 1;
    if (cr > (1u << 24)) { set_err("chunk_records > 2^24"); return H2TAP_E_INVAL; }
    h2tap_delta_store* s = new (std::nothrow) h2tap_delta_store();
    if (!s) { set_err("host allocation failed"); return H2TAP_E_NOMEM; }
    s->device = device;
    s->crec = cr;
    s->cpay = cr * 4;
    h2tap_status st = run_guarded(nullptr, [&]() -> h2tap_status {
        CK(cudaSetDevice(device));
        CK(cudaStreamCreateWithFlags(&s->cs, cudaStreamNonBlocking));
        CK(cudaEventCreateWithFlags(&s->ev, cudaEventDisableTiming));
        return H2TAP_OK;
    });
    if (st != H2TAP_OK) { delete s; return st; }
    *out = s;
    return H2TAP_OK;
}

h2tap_status h2tap_ds_append(h2tap_delta_store* s, uint64_t ts, uint64_t node, int inserted, int deleted,
                             const uint64_t* inserts, const double* weights, uint32_t n_ins, const uint64_t* deletes,
                             uint32_t n_del) {
    if (!s || (n_ins && (!inserts || !weights)) || (n_del && !deletes)) { set_err("null argument"); return H2TAP_E_INVAL; }
    if ((inserted != 0 && inserted != 1) || (deleted != 0 && deleted != 1)) { set_err("flags must be 0/1"); return H2TAP_E_INVAL; }
    return run_guarded(nullptr, [&]() -> h2tap_status {
        uint64_t idx, io, dq;
        {
            std::lock_guard<std::mutex> g(s->mu);
            ds_reserve_chunks(s, s->n_res, s->n_res + 1, s->ins_res, s->ins_res + n_ins, s->del_res, s->del_res + n_del);
            idx = s->n_res++;
            io = s->ins_res; s->ins_res += n_ins;
            dq = s->del_res; s->del_res += n_del;
        }
        ds_scatter(s, s->ich, s->cpay, io, n_ins, inserts);
        ds_scatter(s, s->wch, s->cpay, io, n_ins, weights);
        ds_scatter(s, s->dch, s->cpay, dq, n_del, deletes);
        DeltaRec r{};
        r.ts = ts; r.node = node; r.ins_off = io; r.del_off = dq; r.ins_cnt = n_ins; r.del_cnt = n_del;
        r.valid = 1; r.deleted = (uint8_t)deleted; r.inserted = (uint8_t)inserted;
        s->rch[idx / s->crec].load()[idx % s->crec] = r;
        ds_note_ts(s, idx, ts);
        ds_publish(s, idx, 1, io + n_ins, dq + n_del);
        return H2TAP_OK;
    });
}

h2tap_status h2tap_ds_append_records(h2tap_delta_store* s, const h2tap_delta_record* recs, size_t n,
                                     const uint64_t* inserts, const double* weights, size_t n_ins,
                                     const uint64_t* deletes, size_t n_del) {
    if (!s || (n && !recs) || (n_ins && (!inserts || !weights)) || (n_del && !deletes)) {
        set_err("null argument");
        return H2TAP_E_INVAL;
    }
    const DeltaRec* in = reinterpret_cast<const DeltaRec*>(recs);
    for (size_t i = 0; i < n; ++i) {
        const DeltaRec& r = in[i];
        if (r.valid != 1 || r.deleted > 1 || r.inserted > 1) { set_err("record %zu: valid must be 1, flags 0/1", i); return H2TAP_E_INVAL; }
        if (r.ins_off > n_ins || r.ins_cnt > n_ins - r.ins_off || r.del_off > n_del || r.del_cnt > n_del - r.del_off) {
            set_err("record %zu: slice outside the given arrays", i);
            return H2TAP_E_INVAL;
        }
    }
    return run_guarded(nullptr, [&]() -> h2tap_status {
        uint64_t si = 0, sd = 0;   // the records' slices (a caller array may hold unused entries)
        for (size_t i = 0; i < n; ++i) { si += in[i].ins_cnt; sd += in[i].del_cnt; }
        uint64_t idx, io, dq;
        {
            std::lock_guard<std::mutex> g(s->mu);
            ds_reserve_chunks(s, s->n_res, s->n_res + n, s->ins_res, s->ins_res + si, s->del_res, s->del_res + sd);
            idx = s->n_res; s->n_res += n;
            io = s->ins_res; s->ins_res += si;
            dq = s->del_res; s->del_res += sd;
        }
        n_ins = si;   // what is copied below
        n_del = sd;
        // The store keeps every record's slices in record order (payload offsets grow with the
        // record index; an empty slice sits at the running position): a caller layout that is
        // already back to back goes in with one copy per array, any other is gathered per record.
        bool packed = true;
        for (uint64_t i = 0, pi = 0, pd = 0; i < n && packed; ++i) {
            packed = (in[i].ins_cnt == 0 || in[i].ins_off == pi) && (in[i].del_cnt == 0 || in[i].del_off == pd);
            pi += in[i].ins_cnt;
            pd += in[i].del_cnt;
        }
        if (packed) {
            ds_scatter(s, s->ich, s->cpay, io, n_ins, inserts);
            ds_scatter(s, s->wch, s->cpay, io, n_ins, weights);
            ds_scatter(s, s->dch, s->cpay, dq, n_del, deletes);
        } else {
            for (uint64_t i = 0, pi = io, pd = dq; i < n; ++i) {
                ds_scatter(s, s->ich, s->cpay, pi, in[i].ins_cnt, inserts + in[i].ins_off);
                ds_scatter(s, s->wch, s->cpay, pi, in[i].ins_cnt, weights + in[i].ins_off);
                ds_scatter(s, s->dch, s->cpay, pd, in[i].del_cnt, deletes + in[i].del_off);
                pi += in[i].ins_cnt;
                pd += in[i].del_cnt;
            }
        }
        const uint64_t bs = 1u << 14;
        std::vector<DeltaRec> tmp(std::min<uint64_t>(n, bs));
        uint64_t pi = io, pd = dq;   // running positions (the records' slices, in record order)
        for (uint64_t a = 0; a < n; a += bs) {
            const uint64_t k = std::min<uint64_t>(bs, n - a);
            uint64_t mn = ~0ull;
            for (uint64_t i = 0; i < k; ++i) {
                tmp[i] = in[a + i];
                tmp[i].ins_off = pi;
                tmp[i].del_off = pd;
                pi += tmp[i].ins_cnt;
                pd += tmp[i].del_cnt;
            }
            ds_scatter(s, s->rch, s->crec, idx + a, k, tmp.data());
            for (uint64_t i = 0; i < k; ++i) {
                mn = std::min(mn, tmp[i].ts);
                if (((idx + a + i + 1) % s->kBlock) == 0 || i + 1 == k) { ds_note_ts(s, idx + a + i, mn); mn = ~0ull; }
            }
        }
        ds_publish(s, idx, n, io + si, dq + sd);
        return H2TAP_OK;
    });
}

h2tap_status h2tap_ds_info(const h2tap_delta_store* s, uint64_t* n_records, uint64_t* first_pending,
                           uint64_t* n_mirrored, uint64_t* host_bytes, uint64_t* device_bytes) {
    if (!s) { set_err("null store"); return H2TAP_E_INVAL; }
    if (n_records) *n_records = s->n_pub.load();
    if (first_pending) *first_pending = s->cursor;
    if (n_mirrored) *n_mirrored = s->mbase + s->mlen;
    if (host_bytes) {
        uint64_t b = 0;
        for (uint64_t c = 0; c < s->kMaxChunks; ++c) {
            if (s->rch[c].load()) b += s->crec * sizeof(DeltaRec);
            if (s->ich[c].load()) b += s->cpay * 16;
            if (s->dch[c].load()) b += s->cpay * 8;
        }
        *host_bytes = b;
    }
    if (device_bytes) *device_bytes = s->mcap * sizeof(DeltaRec) + s->icap * 8 + s->wcap * 8 + s->dcap * 8;
    return H2TAP_OK;
}

/* records [first, first + n) of the live window [first_pending, n_records) with their
 * current validity flags and absolute payload offsets (tests, checkpoints) */
h2tap_status h2tap_ds_export(h2tap_delta_store* s, uint64_t first, size_t n, h2tap_delta_record* out) {
    if (!s || (n && !out)) { set_err("null argument"); return H2TAP_E_INVAL; }
    const uint64_t np = s->n_pub.load();
    if (first < s->cursor || first + n > np) { set_err("range outside the live window"); return H2TAP_E_INVAL; }
    return run_guarded(nullptr, [&]() -> h2tap_status {
        DeltaRec* o = reinterpret_cast<DeltaRec*>(out);
        const uint64_t mend = s->mbase + s->mlen;
        uint64_t a = first, k = n;
        if (a < mend && k) {   // mirrored: the device copy holds the current flags
            const uint64_t m = std::min<uint64_t>(k, mend - a);
            CK(cudaSetDevice(s->device));
            CK(cudaStreamSynchronize(s->cs));
            CK(cudaMemcpy(o, s->m_rec + (a - s->mbase), m * sizeof(DeltaRec), cudaMemcpyDeviceToHost));
            o += m; a += m; k -= m;
        }
        if (k) ds_gather(s, s->rch, s->crec, a, k, o, false, nullptr);
        return H2TAP_OK;
    });
}

h2tap_status h2tap_ds_join(h2tap_delta_store* s, void* stream) {
    if (!s) { set_err("null argument"); return H2TAP_E_INVAL; }
    try {
        CK(cudaSetDevice(s->device));
        CK(cudaEventRecord(s->ev, s->cs));
        CK(cudaStreamWaitEvent(static_cast<cudaStream_t>(stream), s->ev, 0));
    } catch (const Fail& e) {
        return e.st;
    }
    return H2TAP_OK;
}

void h2tap_ds_destroy(h2tap_delta_store* s) {
    if (!s) return;
    cudaSetDevice(s->device);
    if (s->cs) cudaStreamSynchronize(s->cs);
    for (uint64_t c = 0; c < s->kMaxChunks; ++c) {
        if (DeltaRec* p = s->rch[c].load()) cudaFreeHost(p);
        delete[] s->bmin[c].load();
        if (uint64_t* p = s->ich[c].load()) cudaFreeHost(p);
        if (double* p = s->wch[c].load()) cudaFreeHost(p);
        if (uint64_t* p = s->dch[c].load()) cudaFreeHost(p);
    }
    for (auto& f : s->free_chunks)
        for (void* p : f) cudaFreeHost(p);
    for (void* p : {(void*)s->m_rec, (void*)s->m_ins, (void*)s->m_w, (void*)s->m_del, (void*)s->m_rec2,
                    (void*)s->m_ins2, (void*)s->m_w2, (void*)s->m_del2})
        if (p) cudaFree(p);
    if (s->ev) cudaEventDestroy(s->ev);
    if (s->cs) cudaStreamDestroy(s->cs);
    delete s;
}

/* One propagation cycle from the store (see the file comment). */
h2tap_status h2tap_delta_apply_store(h2tap_replica* r, h2tap_delta_store* s, uint64_t snapshot_ts,
                                     h2tap_apply_stats* stats) {
    if (!r || !s) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (s->device != r->cfg.device) { set_err("store and replica on different devices"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        if (snapshot_ts < r->snap) {
            set_err("snapshot_ts %llu < current %llu", (unsigned long long)snapshot_ts, (unsigned long long)r->snap);
            return H2TAP_E_SNAPSHOT_REGRESSION;
        }
        g_ht.init();
        g_ht.mark("entry");
        CK(cudaSetDevice(r->cfg.device));
        cudaStream_t st = r->st;
        g_launches = g_h2d = g_d2h = 0;
        if (!r->ev[7]) CK(cudaEventCreate(&r->ev[7]));
        CK(cudaEventRecord(r->ev[7], st));
        const uint64_t np = s->n_pub.load(std::memory_order_acquire);
        const uint64_t pins = s->pub_ins.load(), pdel = s->pub_del.load();
        // the scan's end: trailing whole blocks whose every record is invisible stay for later
        uint64_t end = np;
        while (end > s->cursor) {  // (a block's min covers every record noted in it: conservative)
            const uint64_t b0 = ((end - 1) / s->kBlock) * s->kBlock;
            if (b0 < s->cursor) break;
            if (s->bmin[b0 / s->crec].load()[(b0 % s->crec) / s->kBlock].load() <= snapshot_ts) break;
            end = b0;
        }
        g_ht.mark("visible_end");
        uint64_t ie, de;  // payload positions at the scan's end
        ds_pos(s, end, np, pins, pdel, &ie, &de);
        // mirror capacity for everything published (read-ahead included), then the copies the
        // scan needs; the replica stream waits for them
        if (np - s->mbase > s->mcap || pins - s->ibase > s->icap || pins - s->ibase > s->wcap ||
            pdel - s->dbase > s->dcap) {
            CK(cudaStreamSynchronize(s->cs));  // earlier copies are done before a regrow
            CK(cudaStreamSynchronize(st));
            ds_grow(s->m_rec, s->m_rec2, s->mcap, s->mlen, np - s->mbase);
            ds_grow(s->m_ins, s->m_ins2, s->icap, s->ilen, pins - s->ibase);
            ds_grow(s->m_w, s->m_w2, s->wcap, s->ilen, pins - s->ibase);
            ds_grow(s->m_del, s->m_del2, s->dcap, s->dlen, pdel - s->dbase);
        }
        g_ht.mark("grow");
        uint64_t h2d = ds_mirror(s, end, ie, de);
        CK(cudaEventRecord(s->ev, s->cs));
        CK(cudaStreamWaitEvent(st, s->ev, 0));
        g_ht.mark("mirror");
        const uint64_t nr = end - s->cursor;
        DeltaRec* rec = s->m_rec + (s->cursor - s->mbase);
        // read-ahead: the copies of the not-yet-needed deltas are issued while the scan kernels run
        // and overlap the rest of the cycle (the mirror's capacity was reserved above)
        uint64_t ra = 0;
        // consumed records -> invalid, enqueued behind the cycle's last kernel so that the
        // first still-pending record comes back with the cycle's own read-back (Counters);
        // the kernel marks nothing when the cycle's status carries an error
        bool consumed = false;
        const std::function<void()> consume = [&] {
            if (nr) {
                k_rec_consume<<<g1(nr), 256, 0, st>>>(rec, nr, snapshot_ts, r->dctr(), ST_NOT_OWNED | ST_CREATE_ENDPOINT);
                CK(cudaGetLastError());
            }
            consumed = true;
        };
        h2tap_status rc = apply_records_dev(r, rec, nr, s->m_ins, nullptr, s->m_w, ie - s->ibase, s->m_del,
                                            de - s->dbase, snapshot_ts, s->ibase, s->dbase, snapshot_ts, stats,
                                            [&] { ra = ds_mirror(s, np, pins, pdel); }, &consume);
        g_ht.mark("apply");
        h2d += ra;
        if (stats) stats->h2d_bytes += h2d;
        if (rc != H2TAP_OK) return rc;
        unsigned long long first = r->hc->first_pend;
        if (!consumed) {  // the cycle ended before its final read-back (nothing visible): mark here
            k_init_counters<<<1, 32, 0, st>>>(r->dctr());
            consume();
            r->read_counters();
            first = r->hc->first_pend;
        }
        g_ht.mark("consume");
        if (stats) stats->n_launches += nr ? 1 : 0;
        const uint64_t cur = s->cursor + std::min<uint64_t>(first, nr);
        uint64_t ci, cd;
        ds_pos(s, cur, np, pins, pdel, &ci, &cd);
        s->cursor = cur; s->cur_ins = ci; s->cur_del = cd;
        s->snap = snapshot_ts;
        ds_release_below(s, cur, ci, cd);
        // move the mirror window to the twin buffers: what is still pending starts at slot 0 again
        const uint64_t rs = cur - s->mbase, is = ci - s->ibase, dsh = cd - s->dbase;
        if (rs) {
            CK(cudaEventRecord(s->ev, st));  // the consume kernel ran on the replica stream
            CK(cudaStreamWaitEvent(s->cs, s->ev, 0));
            DsMove mv{};
            int k = 0;
            auto seg = [&](auto*& p, auto*& p2, uint64_t by, uint64_t len) {
                if (len > by) {
                    mv.src[k] = reinterpret_cast<const uint64_t*>(p + by);
                    mv.dst[k] = reinterpret_cast<uint64_t*>(p2);
                    mv.words[k] = (len - by) * sizeof(*p) / 8;
                    ++k;
                }
                std::swap(p, p2);
            };
            seg(s->m_rec, s->m_rec2, rs, s->mlen);
            seg(s->m_ins, s->m_ins2, is, s->ilen);
            seg(s->m_w, s->m_w2, is, s->ilen);
            seg(s->m_del, s->m_del2, dsh, s->dlen);
            if (k) {
                k_ds_move<<<(unsigned)(r->n_sm * 4), 256, 0, s->cs>>>(mv);
                CK(cudaGetLastError());
            }
            s->mbase = cur; s->mlen -= rs;
            s->ibase = ci; s->ilen -= is;
            s->dbase = cd; s->dlen -= dsh;
        }
        g_ht.mark("release+move");
        g_ht.dump("store cycle");
        return H2TAP_OK;
    });
}

}  // extern "C"
