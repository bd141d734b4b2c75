// Collective mode of a sharded replica: the library owns an NCCL
// communicator (h2tap_config.nccl_unique_id) and every multi-GPU call is collective - all
// ranks call it with their own arguments and it returns the same status everywhere.
//
// h2tap_delta_apply on such a replica takes this rank's slice of the global batch
// (rank-major arrival order, reading A5) and runs the exchange step a8 inside:
//   1. k_validate + k_route_count on the slice; ONE ncclAllGather of the rows
//      {status, slice size, counts[world]} -> host (round trip 1): the agreed validity,
//      the global seq base of this slice, the world x world count matrix C;
//   2. k_route_pack: 40-byte route records grouped by destination (sizes known from C);
//   3. the records move with grouped ncclSend / ncclRecv (an all-to-all over NVLink /
//      NVSwitch; splits from C);
//   4. two-phase apply: the cycle runs on what arrived, result left in the back buffers;
//      ONE ncclAllGather of {prepare status, new shard edge count} -> host (round trip 2);
//      every rank commits (the swap) or every rank aborts; the shard's global edge base
//      comes from the same gather.
// h2tap_bfs / h2tap_pagerank / h2tap_sssp on such a replica run the per-shard kernels and
// combine the shards with ncclAllReduce (MAX of the u8 frontier marks per level, SUM of the
// PageRank contributions and dangling mass, MIN of the relaxed fp64 distances).
//
// NCCL is loaded at run time (dlopen "libnccl.so.2": the process's NCCL - torch's when torch
// is loaded), so a replica without a communicator never needs it.
#include <dlfcn.h>
#include <nccl.h>

namespace coll {

struct Api {
    ncclResult_t (*GetUniqueId)(ncclUniqueId*);
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int);
    ncclResult_t (*CommDestroy)(ncclComm_t);
    ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t);
    ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t);
    ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
    ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
    ncclResult_t (*GroupStart)();
    ncclResult_t (*GroupEnd)();
    const char* (*GetErrorString)(ncclResult_t);
};

const Api* api() {
    static std::mutex mu;
    static Api a{};
    static int state = 0;  // 0 untried, 1 loaded, -1 unavailable
    std::lock_guard<std::mutex> lk(mu);
    if (state == 0) {
        void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        state = -1;
        if (h) {
            bool ok = true;
            auto sym = [&](auto& fn, const char* name) {
                fn = reinterpret_cast<std::remove_reference_t<decltype(fn)>>(dlsym(h, name));
                ok = ok && fn != nullptr;
            };
            sym(a.GetUniqueId, "ncclGetUniqueId");
            sym(a.CommInitRank, "ncclCommInitRank");
            sym(a.CommDestroy, "ncclCommDestroy");
            sym(a.AllGather, "ncclAllGather");
            sym(a.AllReduce, "ncclAllReduce");
            sym(a.Send, "ncclSend");
            sym(a.Recv, "ncclRecv");
            sym(a.GroupStart, "ncclGroupStart");
            sym(a.GroupEnd, "ncclGroupEnd");
            sym(a.GetErrorString, "ncclGetErrorString");
            if (ok) state = 1;
        }
    }
    if (state != 1) {
        set_err("collective mode: NCCL (libnccl.so.2) could not be loaded");
        return nullptr;
    }
    return &a;
}

#define NCK(call)                                                                              \
    do {                                                                                       \
        ncclResult_t e_ = (call);                                                              \
        if (e_ != ncclSuccess) {                                                               \
            set_err("NCCL %s: %s (%s:%d)", #call, coll::api()->GetErrorString(e_), __FILE__, __LINE__); \
            throw Fail{H2TAP_E_NCCL};                                                          \
        }                                                                                      \
    } while (0)

// {status, n, counts[P]} of this rank's slice, assembled on the device
__global__ void k_coll_row(const unsigned long long* __restrict__ st, uint64_t n, const unsigned long long* __restrict__ cnt,
                           int P, unsigned long long* __restrict__ row) {
    for (int i = threadIdx.x; i < P + 2; i += blockDim.x)
        row[i] = i == 0 ? *st : (i == 1 ? (unsigned long long)n : cnt[i - 2]);
}

// communicator of a new collective-mode replica (every rank calls create)
void init_comm(h2tap_replica* r) {
    const Api* A = api();
    if (!A) throw Fail{H2TAP_E_INVAL};
    ncclUniqueId id;
    std::memcpy(&id, r->cfg.nccl_unique_id, sizeof id);
    ncclComm_t c = nullptr;
    NCK(A->CommInitRank(&c, r->cfg.world, id, r->cfg.rank));
    r->comm = c;
    r->cfg.nccl_unique_id = nullptr;  // not retained
}

void destroy_comm(h2tap_replica* r) {
    if (r->comm && api()) api()->CommDestroy(static_cast<ncclComm_t>(r->comm));
    r->comm = nullptr;
}

// one collective apply (steps 1-4 above); `b` host or device
h2tap_status apply(h2tap_replica* r, const h2tap_batch* b, uint64_t S, h2tap_apply_stats* stats) {
    const Api* A = api();
    if (!A) return H2TAP_E_INVAL;
    ncclComm_t comm = static_cast<ncclComm_t>(r->comm);
    cudaStream_t st = r->st;
    const int P = r->cfg.world, me = r->cfg.rank;
    const uint64_t n = b->n;
    // the slice on the device (route packing reads device memory)
    h2tap_batch d = *b;
    if (n && !b->on_device) {
        d.kind = r->get<uint8_t>(r->Wk, n);
        d.src = r->get<uint64_t>(r->Ws, n);
        d.dst = r->get<uint64_t>(r->Wd, n);
        d.weight = r->get<float>(r->Ww, n);
        d.ts = r->get<uint64_t>(r->Wt, n);
        copy_in(r, const_cast<uint8_t*>(d.kind), b->kind, n, 0);
        copy_in(r, const_cast<uint64_t*>(d.src), b->src, n, 0);
        if (b->dst) copy_in(r, const_cast<uint64_t*>(d.dst), b->dst, n, 0);
        else CK(cudaMemsetAsync(const_cast<uint64_t*>(d.dst), 0, n * 8, st));
        if (b->weight) copy_in(r, const_cast<float*>(d.weight), b->weight, n, 0);
        else CK(cudaMemsetAsync(const_cast<float*>(d.weight), 0, n * 4, st));
        copy_in(r, const_cast<uint64_t*>(d.ts), b->ts, n, 0);
        d.on_device = 1;
    } else if (n && (!d.dst || !d.weight)) {
        if (!d.dst) { d.dst = r->get<uint64_t>(r->Wd, n); CK(cudaMemsetAsync(const_cast<uint64_t*>(d.dst), 0, n * 8, st)); }
        if (!d.weight) { d.weight = r->get<float>(r->Ww, n); CK(cudaMemsetAsync(const_cast<float*>(d.weight), 0, n * 4, st)); }
    }
    // 1. validity + counts -> all-gather -> host
    const uint64_t* bounds = static_cast<const uint64_t*>(r->bounds_dev.p);
    unsigned long long* w = r->get<unsigned long long>(r->coll, 2 * (size_t)(P + 2) * (P + 1) + 64);
    unsigned long long* vst = w;             // validate status word
    unsigned long long* cnt = w + 1;         // counts[P]
    unsigned long long* row = cnt + P;       // {status, n, counts[P]}
    unsigned long long* all = row + P + 2;   // P rows
    CK(cudaMemsetAsync(w, 0, (size_t)(1 + P) * 8, st));
    if (n) {
        const unsigned g = (unsigned)std::min<uint64_t>(cdiv(n, 256), 148 * 8);
        k_validate<<<g, 256, 0, st>>>(d.kind, d.ts, n, r->snap, vst);
        CKL();
        k_route_count<<<g, 256, (P + 1) * 4, st>>>(d.kind, d.src, n, bounds, P, cnt);
        CKL();
    }
    k_coll_row<<<1, 64, 0, st>>>(vst, n, cnt, P, row);
    CKL();
    NCK(A->AllGather(row, all, (size_t)P + 2, ncclUint64, comm, st));
    std::vector<unsigned long long> M((size_t)P * (P + 2));
    CK(cudaMemcpyAsync(M.data(), all, M.size() * 8, cudaMemcpyDeviceToHost, st));
    r->sync();                                                    // round trip 1
    unsigned long long bad = 0;
    for (int p = 0; p < P; ++p) bad |= M[(size_t)p * (P + 2)];
    if (bad & ST_BAD_KIND) { set_err("collective apply: a rank's slice has an unknown op kind"); return H2TAP_E_INVAL; }
    if (bad & ST_STALE) { set_err("collective apply: a rank's slice has an op with ts <= snapshot (reading A7)"); return H2TAP_E_STALE_TS; }
    if (S < r->snap) { set_err("snapshot_ts regression"); return H2TAP_E_SNAPSHOT_REGRESSION; }
    auto C = [&](int s, int dd) -> uint64_t { return M[(size_t)s * (P + 2) + 2 + dd]; };
    uint64_t seq0 = r->coll_seq, total = 0, n_send = 0, n_recv = 0;
    for (int p = 0; p < P; ++p) {
        const uint64_t sz = M[(size_t)p * (P + 2) + 1];
        if (p < me) seq0 += sz;
        total += sz;
        n_send += C(me, p);
        n_recv += C(p, me);
    }
    // 2. pack by destination
    RouteRec* sendb = r->get<RouteRec>(r->coll_send, n_send);
    RouteRec* recvb = r->get<RouteRec>(r->coll_recv, n_recv);
    uint64_t route_bytes = 0;
    if (n) {
        const uint64_t nt = cdiv(n, kTile);
        uint64_t* stt = r->get<uint64_t>(r->status, nt);
        unsigned int* ctr = r->get<unsigned int>(r->rs_ctr, P);
        CK(cudaMemsetAsync(ctr, 0, P * 4, st));
        uint64_t base = 0;
        for (int p = 0; p < P; ++p) {
            if (C(me, p)) {
                CK(cudaMemsetAsync(stt, 0, nt * 8, st));
                k_route_pack<<<(unsigned)nt, kThreads, 0, st>>>(d.kind, d.src, d.dst, d.weight, d.ts, n, seq0, bounds, P, p,
                                                                sendb + base, stt, ctr + p);
                CKL();
            }
            base += C(me, p);
        }
    }
    // 3. all-to-all of the records
    {
        uint64_t so = 0, ro = 0;
        NCK(A->GroupStart());
        for (int p = 0; p < P; ++p) {
            const uint64_t ns = C(me, p), nr = C(p, me);
            if (ns) NCK(A->Send(sendb + so, ns * sizeof(RouteRec), ncclUint8, p, comm, st));
            if (nr) NCK(A->Recv(recvb + ro, nr * sizeof(RouteRec), ncclUint8, p, comm, st));
            if (p != me) route_bytes += ns * sizeof(RouteRec);
            so += ns;
            ro += nr;
        }
        NCK(A->GroupEnd());
    }
    // 4. prepare, agree, commit or abort everywhere
    h2tap_status ps;
    r->defer_commit = true;
    try {
        BatchIn in{n_recv, 1, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, 0, recvb};
        ps = apply_core(r, in, S, false, stats);
    } catch (const Fail& e) {
        ps = e.st;
    }
    r->defer_commit = false;
    if (ps != H2TAP_OK) r->prep.on = false;
    if (r->poisoned) throw Fail{H2TAP_E_POISONED};
    {
        long long mine[2] = {(long long)ps, (long long)(ps == H2TAP_OK ? r->prep.E : 0)};
        long long* rowd = reinterpret_cast<long long*>(all + (size_t)P * (P + 2));
        long long* alld = rowd + 2;
        CK(cudaMemcpyAsync(rowd, mine, 16, cudaMemcpyHostToDevice, st));
        NCK(A->AllGather(rowd, alld, 2, ncclInt64, comm, st));
        std::vector<long long> G(2 * (size_t)P);
        CK(cudaMemcpyAsync(G.data(), alld, G.size() * 8, cudaMemcpyDeviceToHost, st));
        r->sync();                                                // round trip 2
        long long agreed = 0;
        uint64_t ebase = 0;
        for (int p = 0; p < P; ++p) {
            agreed = std::min(agreed, G[2 * (size_t)p]);
            if (p < me) ebase += (uint64_t)G[2 * (size_t)p + 1];
        }
        if (agreed != 0) {
            r->prep.on = false;  // abort (nothing was swapped)
            if (ps == H2TAP_OK) set_err("collective apply: another rank failed to prepare; every rank aborted");
            return (h2tap_status)agreed;
        }
        r->commit();
        r->edge_base = ebase;
    }
    r->coll_seq += total;
    r->last_route_bytes = route_bytes;
    if (stats) {
        stats->n_launches += (n ? 2 : 0) + 1;
        stats->h2d_bytes += b->on_device ? 16 : 16 + n * 29;
        stats->d2h_bytes += M.size() * 8 + 16 * (uint64_t)P;
    }
    return H2TAP_OK;
}

// global vertex count (every shard keeps the whole ID map)
uint64_t lookup_src(h2tap_replica* r, uint64_t source_ext, const char* who) {
    const uint64_t k = dense_of(r, source_ext);
    if (k >= r->V) {
        set_err("%s source %llu is not a live vertex", who, (unsigned long long)source_ext);
        throw Fail{H2TAP_E_INVAL};
    }
    return k;
}

h2tap_status bfs(h2tap_replica* r, uint64_t source_ext, int32_t* level_out, int on_device) {
    const Api* A = api();
    if (!A) return H2TAP_E_INVAL;
    ncclComm_t comm = static_cast<ncclComm_t>(r->comm);
    cudaStream_t st = r->st;
    const uint64_t V = r->V, src = lookup_src(r, source_ext, "BFS");
    const ShardView s = shard_view(r);
    int32_t* level = on_device ? level_out : r->get<int32_t>(r->pr_a, V);
    uint8_t* mark = r->get<uint8_t>(r->bfs_a, V);
    unsigned long long* c = r->get<unsigned long long>(r->misc, 1);
    k_fill_i32<<<g1(V), 256, 0, st>>>(level, V, -1);
    CKL();
    const int32_t zero = 0;
    CK(cudaMemcpyAsync(level + src, &zero, 4, cudaMemcpyHostToDevice, st));
    for (int32_t depth = 0;; ++depth) {
        CK(cudaMemsetAsync(mark, 0, V, st));
        if (s.Vr) { k_shard_bfs_expand<<<warp_grid(r, s.Vr), 256, 0, st>>>(s.off, s.cols, s.Vr, s.row_lo, level, depth, mark); CKL(); }
        NCK(A->AllReduce(mark, mark, V, ncclUint8, ncclMax, comm, st));
        CK(cudaMemsetAsync(c, 0, 8, st));
        k_shard_bfs_settle<<<g1(V), 256, 0, st>>>(level, mark, V, depth, c);
        CKL();
        unsigned long long h = 0;
        CK(cudaMemcpyAsync(&h, c, 8, cudaMemcpyDeviceToHost, st));
        r->sync();
        if (h == 0) break;  // identical on every rank (the marks were reduced)
    }
    if (!on_device) CK(cudaMemcpyAsync(level_out, level, V * 4, cudaMemcpyDeviceToHost, st));
    r->sync();
    return H2TAP_OK;
}

h2tap_status pagerank(h2tap_replica* r, double damping, int iterations, double* rank_out, int on_device) {
    const Api* A = api();
    if (!A) return H2TAP_E_INVAL;
    ncclComm_t comm = static_cast<ncclComm_t>(r->comm);
    cudaStream_t st = r->st;
    const uint64_t V = r->V;
    if (V == 0) return H2TAP_OK;
    const ShardView s = shard_view(r);
    double* a = r->get<double>(r->pr_a, V);
    double* acc = r->get<double>(r->pr_b, V);
    double* dang = r->get<double>(r->misc, 1);
    k_pr_init<<<g1(V), 256, 0, st>>>(a, V, nullptr, V);
    CKL();
    for (int it = 0; it < iterations; ++it) {
        CK(cudaMemsetAsync(acc, 0, V * 8, st));
        CK(cudaMemsetAsync(dang, 0, 8, st));
        if (s.Vr) { k_shard_pr_push<<<warp_grid(r, s.Vr), 256, 0, st>>>(s.off, s.cols, s.Vr, s.row_lo, a, acc, dang); CKL(); }
        NCK(A->GroupStart());
        NCK(A->AllReduce(acc, acc, V, ncclFloat64, ncclSum, comm, st));
        NCK(A->AllReduce(dang, dang, 1, ncclFloat64, ncclSum, comm, st));
        NCK(A->GroupEnd());
        k_shard_pr_finish<<<g1(V), 256, 0, st>>>(acc, V, damping, dang);
        CKL();
        std::swap(a, acc);
    }
    CK(cudaMemcpyAsync(rank_out, a, V * 8, on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, st));
    r->sync();
    return H2TAP_OK;
}

h2tap_status sssp(h2tap_replica* r, uint64_t source_ext, double* dist_out, int on_device) {
    const Api* A = api();
    if (!A) return H2TAP_E_INVAL;
    ncclComm_t comm = static_cast<ncclComm_t>(r->comm);
    cudaStream_t st = r->st;
    const ShardView s = shard_view(r);
    const uint64_t V = r->V, E = r->E;
    unsigned long long* c = r->get<unsigned long long>(r->misc, 2);
    CK(cudaMemsetAsync(c, 0, 16, st));
    if (E) {
        k_sssp_check_w<<<(unsigned)std::min<uint64_t>(cdiv(E, 256 * 8), (uint64_t)r->n_sm * 8), 256, 0, st>>>(
            s.w, E, reinterpret_cast<unsigned int*>(c));
        CKL();
    }
    NCK(A->AllReduce(c, c, 1, ncclUint64, ncclMax, comm, st));  // any shard's bad weight fails all
    unsigned long long hb = 0;
    CK(cudaMemcpyAsync(&hb, c, 8, cudaMemcpyDeviceToHost, st));
    r->sync();
    if (hb) { set_err("h2tap_sssp: negative or NaN edge weight"); return H2TAP_E_INVAL; }
    const uint64_t src = lookup_src(r, source_ext, "SSSP");
    double* dist = on_device ? dist_out : r->get<double>(r->pr_a, V);
    double* nd = r->get<double>(r->pr_b, V);
    uint8_t* frontier = r->get<uint8_t>(r->bfs_a, V);
    k_fill_u64<<<g1(V), 256, 0, st>>>(reinterpret_cast<uint64_t*>(dist), V, 0x7FF0000000000000ull);  // +inf
    CKL();
    CK(cudaMemsetAsync(frontier, 0, V, st));
    const double zero = 0.0;
    const uint8_t one = 1;
    CK(cudaMemcpyAsync(dist + src, &zero, 8, cudaMemcpyHostToDevice, st));
    CK(cudaMemcpyAsync(frontier + src, &one, 1, cudaMemcpyHostToDevice, st));
    for (;;) {
        CK(cudaMemcpyAsync(nd, dist, V * 8, cudaMemcpyDeviceToDevice, st));
        if (s.Vr) {
            k_shard_sssp_relax<<<warp_grid(r, s.Vr), 256, 0, st>>>(s.off, s.cols, s.w, s.Vr, s.row_lo, frontier, dist,
                                                                 reinterpret_cast<unsigned long long*>(nd));
            CKL();
        }
        NCK(A->AllReduce(nd, nd, V, ncclFloat64, ncclMin, comm, st));
        CK(cudaMemsetAsync(c, 0, 8, st));
        k_shard_sssp_settle<<<g1(V), 256, 0, st>>>(dist, nd, frontier, V, c);
        CKL();
        unsigned long long h = 0;
        CK(cudaMemcpyAsync(&h, c, 8, cudaMemcpyDeviceToHost, st));
        r->sync();
        if (h == 0) break;
    }
    if (!on_device) CK(cudaMemcpyAsync(dist_out, dist, V * 8, cudaMemcpyDeviceToHost, st));
    r->sync();
    return H2TAP_OK;
}

}  // namespace coll
