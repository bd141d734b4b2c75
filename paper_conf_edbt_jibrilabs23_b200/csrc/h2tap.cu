// h2tap.cu - host orchestrator and C ABI of libh2tap.so (include/h2tap.h).
//
// One propagation cycle (h2tap_delta_apply) runs these device steps on the
// replica's stream:
//   a1 k_partition         validate, number, split pending / node ops / edge ops
//   a2 node ops            radix sort by (v, ts, seq), k_node_segments, k_node_lists,
//                          remap tables (k_remap_tables) + k_node_place (ID-map compaction)
//   a3 edge ops            k_edge_prep (lookup, gating, packed key), onesweep radix
//                          sort, k_reduce_classify (latest-commit-wins + outcome lists)
//   a6 k_merge             global merge path into the back buffer
//   a4/a5 k_offsets_*      new row offsets
//   a7 swap                front <-> back at snapshot_ts (host pointer flip)
// Host syncs read small counters between steps (sizes of the next launches).
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include <cstdarg>
#include <cstdlib>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <functional>
#include <atomic>
#include <mutex>
#include <new>
#include <thread>
#include <string>
#include <vector>

#include "../../include/h2tap.h"
#include "kernels.cuh"
#include "radix_sort.cuh"

using namespace h2tap;

namespace {

thread_local std::string g_err;

void set_err(const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
}

struct Fail {
    h2tap_status st;
};

#define CK(call)                                                                          \
    do {                                                                                  \
        cudaError_t e_ = (call);                                                          \
        if (e_ != cudaSuccess) {                                                          \
            set_err("%s:%d %s: %s", __FILE__, __LINE__, #call, cudaGetErrorString(e_));    \
            throw Fail{e_ == cudaErrorMemoryAllocation ? H2TAP_E_NOMEM : H2TAP_E_CUDA};    \
        }                                                                                 \
    } while (0)
thread_local uint64_t g_launches = 0, g_h2d = 0, g_d2h = 0;  // per-call accounting
#define CKL()          \
    do {               \
        ++g_launches;  \
        CK(cudaGetLastError()); \
    } while (0)

struct Buf {
    void* p = nullptr;
    size_t cap = 0;
};

inline uint64_t cdiv(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

// Opt-in step trace (H2TAP_TRACE=1): events recorded on the replica's stream at every
// step boundary, printed as device-time deltas at the end of each apply.
struct Trace {
    bool on = false;
    int n = 0;
    const char* name[48];
    cudaEvent_t ev[48];
    void init() {
        const char* e = getenv("H2TAP_TRACE");
        on = e && *e && *e != '0';
        if (on && !ev[0]) for (auto& x : ev) cudaEventCreate(&x);
        n = 0;
    }
    void mark(const char* nm, cudaStream_t st) {
        if (!on || n >= 48) return;
        name[n] = nm;
        cudaEventRecord(ev[n++], st);
    }
    void dump() {
        if (!on || n < 2) return;
        cudaEventSynchronize(ev[n - 1]);
        fprintf(stderr, "[h2tap trace]");
        for (int i = 1; i < n; ++i) {
            float ms = 0;
            cudaEventElapsedTime(&ms, ev[i - 1], ev[i]);
            fprintf(stderr, " %s=%.1fus", name[i], ms * 1e3f);
        }
        float tot = 0;
        cudaEventElapsedTime(&tot, ev[0], ev[n - 1]);
        fprintf(stderr, " | total=%.1fus\n", tot * 1e3f);
    }
    Trace() { for (auto& x : ev) x = nullptr; }
};
thread_local Trace g_tr;
#define TR(nm) (g_tr.mark(nm, st), nvtxMarkA("h2tap " nm))
// host-side timestamps of the same opt-in trace (host stalls vs device time)
struct HostTrace {
    bool on = false;
    int n = 0;
    const char* name[32];
    std::chrono::steady_clock::time_point t[32];
    void init() { const char* e = getenv("H2TAP_TRACE"); on = e && *e && *e != '0'; n = 0; }
    void mark(const char* nm) { if (on && n < 32) { name[n] = nm; t[n++] = std::chrono::steady_clock::now(); } }
    void dump(const char* what) {
        if (!on || n < 2) return;
        fprintf(stderr, "[h2tap host %s]", what);
        for (int i = 1; i < n; ++i)
            fprintf(stderr, " %s=%.1fus", name[i], std::chrono::duration<double, std::micro>(t[i] - t[i - 1]).count());
        fprintf(stderr, " | total=%.1fus\n", std::chrono::duration<double, std::micro>(t[n - 1] - t[0]).count());
    }
};
thread_local HostTrace g_ht;
inline int bits_for(uint64_t range) { return range == 0 ? 0 : 64 - __builtin_clzll(range); }

// NVTX ranges (host timeline of nsys / ncu --nvtx): one per cycle and one per step of the path;
// header-only NVTX 3, a no-op unless a tool is attached
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

}  // namespace

struct h2tap_replica {
    h2tap_config cfg{};
    cudaStream_t st = nullptr, st2 = nullptr;  // st2: side stream (cascade pass)
    cudaStream_t st_copy = nullptr;            // host->device staging of the next batch
    struct Stage {
        Buf k, s, d, w, t;
        cudaEvent_t ev = nullptr;    // its H2D copy is complete
        cudaEvent_t done = nullptr;  // the cycle that read it has finished (the slot may be refilled)
        uint64_t bytes = 0;  // staged H2D bytes not yet accounted to an apply
    } stg[2];
    int stg_next = 0;
    cudaEvent_t evA = nullptr, evB = nullptr, evC = nullptr, evD = nullptr, evS = nullptr;
    cudaEvent_t evE0 = nullptr, evE1 = nullptr;  // node mode: early endpoint lookups (side stream)
    Buf epre;
    uint64_t V = 0, E = 0, snap = 0, next_seq = 0, n_pend = 0;
    // sharding: V = global live vertices (the replicated ID map), the CSR holds the Vr rows
    // of the owned external-ID range starting at global dense id row_lo
    bool sharded = false;
    OwnRange own{0, ~0ull};
    Buf bounds_dev;  // world + 1 split points (device) for routing
    uint64_t row_lo = 0, Vr = 0;
    bool identity = true, poisoned = false;
    int n_sm = 148;
    int cur = 0, ext_cur = 0, pcur = 0;
    Buf off[2], cols[2], w[2], ext[2], fence[2];
    Buf pk[2], ps[2], pd[2], pw[2], pt[2], pq[2];
    // scratch
    Buf Wk, Ws, Wd, Ww, Wt, Wq, idx_p, idx_n, idx_e, status;
    Buf keyA, keyB, valA, valB, hist, dbase, rs_status, rs_ctr, rs_coop;
    Buf nv, nv_ext, dropped, ins_q, ins_oldpos, hd_rows, hd_bits;
    Buf op_flags, op_ou, op_ow;
    Buf ins_pos, ins_row, ins_col, ins_w, del_pos, upd_pos, upd_w, KR, cls_cat, cls_pos, cls_w;
    Buf misc, nsorted, part, opart, deg, tsum, remap_shift, remap32, casc_wrel, tile_emit, tile_base, del_row, casc_mask, status2, bfs_a, bfs_b, pr_a, pr_b;
    Buf xrec, xins, xwts, xdel, xcnt, xoff, xbig, xnbig;  // delta-record input (h2tap_delta_apply_records)
    bool tomb = false;  // tombstone-row mode (reading A23)
    // a finished cycle waiting for the swap (two-phase apply of a sharded replica: every
    // rank prepares, the ranks agree on the status, then all commit or all abort)
    struct Prep {
        bool on = false, node_mode = false, identity = true;
        int nb = 0, pn = 0, ext_new = 0;
        uint64_t V = 0, E = 0, row_lo = 0, Vr = 0, n_pend = 0, n = 0, S = 0;
    } prep;
    bool defer_commit = false;  // apply_core leaves the result prepared instead of swapping
    // asynchronous apply (h2tap_delta_apply_async): the cycle is enqueued and the call returns;
    // the counters that size the next cycle (V, E, row range, identity) are read when the next
    // cycle's first read-back has passed them (or at h2tap_replica_sync / any read call)
    bool async_req = false;
    bool last_node_mode = false;  // the previous cycle had node ops (speculation predictor)
    struct Inflight {
        bool on = false, node_mode = false, csr_changed = false;
        cudaEvent_t ev[8];
        uint64_t n = 0, n_node = 0, n_edge = 0, n_pend_new = 0, V = 0, Vr = 0, E = 0, row_lo = 0;
        uint64_t launches = 0, h2d = 0, d2h = 0;
    } infl;
    bool fin_ready = false;       // stats of a finalised asynchronous cycle, not yet handed out
    h2tap_apply_stats fin_stats{};
    Counters* hcf = nullptr;      // mapped host slot of an asynchronous cycle's final counters
    Counters* hcf_dev = nullptr;
    cudaEvent_t evx[8]{};         // the other event set (alternates with ev across async cycles)
    void commit() {             // a7: the pointer flip
        cur = prep.nb;
        if (prep.node_mode) {
            ext_cur = prep.ext_new;
            identity = prep.identity;
            idmap_swapped();
        }
        V = prep.V;
        E = prep.E;
        row_lo = prep.row_lo;
        Vr = prep.Vr;
        pcur = prep.pn;
        n_pend = prep.n_pend;
        next_seq += prep.n;
        snap = prep.S;
        prep.on = false;
    }
    // collective mode (library-owned NCCL communicator, csrc/collective.cuh)
    void* comm = nullptr;                 // ncclComm_t
    Buf coll, coll_send, coll_recv;       // gather words, route records out / in
    uint64_t coll_seq = 0;                // global arrival number of the next slice base
    uint64_t edge_base = 0;               // first global edge of this shard
    uint64_t last_route_bytes = 0;        // records sent to other ranks by the last apply
    Buf idsame;         // 2 words: back ID-map buffer == front on [0, [0]); [1] = [0] after the swap
    Buf casc_status;    // look-back words of the cascade scan (runs beside the edge-op phase)
    Buf live[2];        // tombstone mode: u8 liveness per dense id, double-buffered with ext
    Buf ctr;
    Counters* hc = nullptr;      // pinned, device-mapped host mirror
    Counters* hc_dev = nullptr;  // its device address: a kernel writes it (no copy engine)
    unsigned long long* hx = nullptr;      // mapped host words of the record pre-pass read-back
    unsigned long long* hx_dev = nullptr;
    cudaEvent_t ev[8]{};

    void* dalloc(size_t bytes) {
        void* p = nullptr;
        if (cfg.alloc.alloc) {
            p = cfg.alloc.alloc(cfg.alloc.ctx, bytes, (void*)st);
            if (!p) { set_err("allocator returned NULL for %zu bytes", bytes); throw Fail{H2TAP_E_NOMEM}; }
        } else {
            cudaError_t e = cudaMallocAsync(&p, bytes, st);
            if (e != cudaSuccess) {
                cudaGetLastError();
                set_err("cudaMallocAsync(%zu): %s", bytes, cudaGetErrorString(e));
                throw Fail{H2TAP_E_NOMEM};
            }
        }
        return p;
    }
    void dfree(void* p) {
        if (!p) return;
        if (cfg.alloc.alloc) { if (cfg.alloc.free) cfg.alloc.free(cfg.alloc.ctx, p, (void*)st); }
        else cudaFreeAsync(p, st);
    }
    // grow-only buffer; 16 elements of slack so 128-bit loads may run past the end
    template <typename T>
    T* get(Buf& b, uint64_t count) {
        size_t need = (size_t)(count + 16) * sizeof(T);
        if (b.cap < need) {
            if (b.p) dfree(b.p);
            b.p = nullptr;
            b.cap = 0;
            size_t nc = need + need / 8;
            b.p = dalloc(nc);
            b.cap = nc;
            // defined contents once: 128-bit loads and sector probes may read the slack past
            // the live elements (masked off, never used) - compute-sanitizer initcheck clean
            CK(cudaMemsetAsync(b.p, 0, nc, st));
        }
        return static_cast<T*>(b.p);
    }
    void release(Buf& b) { dfree(b.p); b.p = nullptr; b.cap = 0; }
    // the two ID-map buffers traded places: they now hold consecutive snapshots
    void idmap_swapped() {
        k_idmap_commit<<<1, 1, 0, st>>>(get<unsigned long long>(idsame, 2));
        CK(cudaGetLastError());
    }
    void sync() { CK(cudaStreamSynchronize(st)); }
    bool identity_pending = false;  // identity flag of the ext buffer being built
    bool identity_of(int which) const { return which == ext_cur ? identity : identity_pending; }
    void read_counters() {
        // a one-warp kernel stores the counters into the mapped host mirror: the read-back
        // never queues on a copy engine behind a staged batch's H2D copy
        g_d2h += sizeof(Counters);
        k_store_counters<<<1, 32, 0, st>>>(static_cast<const Counters*>(ctr.p), hc_dev);
        CK(cudaGetLastError());
        sync();
    }
    Counters* dctr() { return static_cast<Counters*>(ctr.p); }
    template <typename T>
    void zero(Buf& b, uint64_t count) { CK(cudaMemsetAsync(b.p, 0, count * sizeof(T), st)); }
};

namespace coll {  // csrc/collective.cuh
void init_comm(h2tap_replica* r);
void destroy_comm(h2tap_replica* r);
h2tap_status apply(h2tap_replica* r, const h2tap_batch* b, uint64_t S, h2tap_apply_stats* stats);
h2tap_status bfs(h2tap_replica* r, uint64_t source_ext, int32_t* level_out, int on_device);
h2tap_status pagerank(h2tap_replica* r, double damping, int iterations, double* rank_out, int on_device);
h2tap_status sssp(h2tap_replica* r, uint64_t source_ext, double* dist_out, int on_device);
}  // namespace coll

namespace {

// ---------------------------------------------------------------- sort ----
// Stable LSD sort of (keys, vals)[0, n) on the low `bits` bits; result in (k, v).
// n_dev (nullable): the actual count is in device memory and n is an upper bound.
// Cooperative single-launch sort (rs_coop) when every tile fits on the GPU at once; returns
// false (nothing launched) when it does not.
template <int ITEMS>
bool radix_sort_coop(h2tap_replica* r, uint64_t*& k, uint32_t*& v, uint64_t*& k2, uint32_t*& v2, uint64_t n,
                     int passes, const unsigned long long* n_dev) {
    constexpr int tile = kRsThreads * ITEMS, smem = tile * 12;
    static int occ = -1;  // per process: one device type
    if (occ < 0) {
        CK(cudaFuncSetAttribute(rs_coop<ITEMS>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, rs_coop<ITEMS>, kRsThreads, smem));
    }
    const uint64_t T = cdiv(n, tile);
    if (T > (uint64_t)occ * r->n_sm) return false;
    uint32_t* cnt = r->get<uint32_t>(r->rs_coop, T * 256 + 256 + 32);
    uint32_t* tot = cnt + T * 256;
    unsigned int* bar = tot + 256;
    CK(cudaMemsetAsync(bar, 0, 4, r->st));
    void* args[] = {&k, &v, &k2, &v2, &n, &n_dev, &passes, &cnt, &tot, &bar};
    CK(cudaLaunchCooperativeKernel((void*)rs_coop<ITEMS>, dim3((unsigned)T), dim3(kRsThreads), args, smem, r->st));
    CKL();
    if (passes & 1) {
        std::swap(k, k2);
        std::swap(v, v2);
    }
    return true;
}

void radix_sort(h2tap_replica* r, uint64_t*& k, uint32_t*& v, uint64_t*& k2, uint32_t*& v2, uint64_t n, int bits,
                const unsigned long long* n_dev = nullptr) {
    if (n <= 1 || bits <= 0) return;
    const int passes = (bits + 7) / 8;
    if (passes <= kRsMaxPasses) {
#ifndef H2TAP_RS_TINY
#define H2TAP_RS_TINY (1u << 15)  // rs_coop tile: 512 keys up to here
#endif
#ifndef H2TAP_RS_SMALL
#define H2TAP_RS_SMALL (1u << 18)
#endif
        if (n <= H2TAP_RS_TINY ? radix_sort_coop<2>(r, k, v, k2, v2, n, passes, n_dev)
            : n <= H2TAP_RS_SMALL ? radix_sort_coop<4>(r, k, v, k2, v2, n, passes, n_dev)
                                  : radix_sort_coop<12>(r, k, v, k2, v2, n, passes, n_dev))
            return;
    }
    const uint64_t ntiles = cdiv(n, kRsTile);
    uint32_t* hist = r->get<uint32_t>(r->hist, kRsMaxPasses * 256);
    uint64_t* dbase = r->get<uint64_t>(r->dbase, kRsMaxPasses * 256 + kRsMaxPasses);
    uint32_t* skip = reinterpret_cast<uint32_t*>(dbase + kRsMaxPasses * 256);
    uint64_t* st = r->get<uint64_t>(r->rs_status, (uint64_t)passes * ntiles * 256);
    uint32_t* ctr = r->get<uint32_t>(r->rs_ctr, kRsMaxPasses);
    CK(cudaMemsetAsync(hist, 0, kRsMaxPasses * 256 * sizeof(uint32_t), r->st));
    CK(cudaMemsetAsync(st, 0, (size_t)passes * ntiles * 256 * sizeof(uint64_t), r->st));
    CK(cudaMemsetAsync(ctr, 0, kRsMaxPasses * sizeof(uint32_t), r->st));
    int grid = (int)std::min<uint64_t>(cdiv(n, 256 * 8), 148 * 8);
    rs_histogram<<<grid, 256, 0, r->st>>>(k, n, n_dev, passes, hist);
    CKL();
    rs_digit_base<<<passes, 256, 0, r->st>>>(hist, dbase, n, n_dev, skip);
    CKL();
    CK(cudaFuncSetAttribute(rs_onesweep, cudaFuncAttributeMaxDynamicSharedMemorySize, kRsSmem));  // per device
    for (int p = 0; p < passes; ++p) {
        rs_onesweep<<<(unsigned)ntiles, kRsThreads, kRsSmem, r->st>>>(k, v, k2, v2, n, n_dev, 8 * p, dbase + p * 256,
                                                              st + (uint64_t)p * ntiles * 256, ctr + p, skip + p);
        CKL();
        std::swap(k, k2);
        std::swap(v, v2);
    }
}

struct BatchIn {
    uint64_t n;
    int on_device;
    const uint64_t* seq;  // NULL -> next_seq + i
    const uint8_t* kind;  // NULL -> all EDGE_INSERT (create)
    const uint64_t* src;
    const uint64_t* dst;
    const float* w;
    const uint64_t* ts;   // NULL -> all create_ts (create)
    uint64_t fill_ts;
    const RouteRec* recs = nullptr;  // routed records (device) instead of the SoA arrays
    // delta records (device) instead of the SoA arrays: n = their expanded op count
    const DeltaRec* drec = nullptr;
    uint64_t n_drec = 0;
    const uint64_t *drec_off = nullptr, *dins = nullptr, *ddel = nullptr;
    const float* dwts = nullptr;
    const double* dwts64 = nullptr;                  // 8-byte weights (narrowed to f32)
    uint64_t vis_ts = ~0ull, ins_base = 0, del_base = 0;  // delta-store scan: visibility, window bases
    uint64_t pre_h2d = 0, pre_d2h = 0, pre_launches = 0;  // accounting of the record pre-pass
    const std::function<void()>* after_merge_launch = nullptr;  // host work issued behind the merge
    cudaEvent_t input_done = nullptr;  // recorded once no kernel of the cycle reads the input arrays
    const std::function<void()>* before_readback = nullptr;     // kernels enqueued before the final read-back
};

template <typename T>
void copy_in(h2tap_replica* r, T* dst, const T* src, uint64_t n, int on_device) {
    if (n == 0) return;
    if (!on_device) g_h2d += n * sizeof(T);
    CK(cudaMemcpyAsync(dst, src, n * sizeof(T), on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, r->st));
}

__global__ void k_fill_u8(uint8_t* p, uint64_t n, uint8_t v) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) p[i] = v;
}
__global__ void k_fill_u64(uint64_t* p, uint64_t n, uint64_t v) {
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) p[i] = v;
}

inline unsigned g1(uint64_t n, unsigned b = 256) { return (unsigned)std::max<uint64_t>(1, cdiv(n, b)); }

float ev_ms(cudaEvent_t a, cudaEvent_t b) {
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    return ms;
}

uint64_t n_fence(uint64_t V) { return (V + (1u << kFenceShift) - 1) >> kFenceShift; }

void build_fence(h2tap_replica* r, int which, uint64_t V) {
    uint64_t nf = n_fence(V);
    uint64_t* f = r->get<uint64_t>(r->fence[which], nf);
    if (nf && !r->identity_of(which)) {
        k_build_fence<<<g1(nf), 256, 0, r->st>>>(static_cast<const uint64_t*>(r->ext[which].p), V, f);
        CKL();
    }
}

ExtIndex ext_index(h2tap_replica* r) {
    ExtIndex X;
    X.ext = static_cast<const uint64_t*>(r->ext[r->ext_cur].p);
    X.fence = static_cast<const uint64_t*>(r->fence[r->ext_cur].p);
    X.V = r->V;
    X.nf = n_fence(r->V);
    X.identity = r->identity;
    X.live = r->tomb ? static_cast<const uint8_t*>(r->live[r->ext_cur].p) : nullptr;
    return X;
}

#ifndef H2TAP_MERGE_CTAS
#define H2TAP_MERGE_CTAS 0
#endif
#ifndef H2TAP_IDMAP_KEEP
#define H2TAP_IDMAP_KEEP 1  // node mode: leave the ID-map prefix both buffers already share
#endif
#ifndef H2TAP_EDGE_PRE
#define H2TAP_EDGE_PRE 1  // node mode: edge endpoints looked up in the old ID map early, on the side stream
#endif
#ifndef H2TAP_CASC_TMA
#define H2TAP_CASC_TMA 1  // cascade column pass streamed by TMA, one small CTA per SM
#endif
#ifndef H2TAP_CC_CTAS
#define H2TAP_CC_CTAS 8  // TMA cascade pass: CTAs per 8 SMs (fewer leave HBM headroom to the edge-op kernels)
#endif
#ifndef H2TAP_CASC_CTAS
#define H2TAP_CASC_CTAS 4
#endif
constexpr int kCascCtasPerSm = H2TAP_CASC_CTAS;  // cascade pass beside the edge-op phase

// An asynchronous cycle's end: the sizes of the new replica from its final counters (the
// stream has passed their store), its stats kept for h2tap_delta_apply_async /
// h2tap_replica_sync.  The counter-independent part of the swap happened at enqueue time.
void finalize_inflight(h2tap_replica* r) {
    h2tap_replica::Inflight& f = r->infl;
    const Counters& fc = *r->hcf;
    r->V = fc.Vn;
    r->E = fc.En;
    r->Vr = fc.Vr_new;
    if (f.node_mode) r->identity = fc.new_identity == 1;
    h2tap_apply_stats& st = r->fin_stats;
    memset(&st, 0, sizeof st);
    st.n_visible = f.n_node + f.n_edge;
    st.n_deferred = f.n_pend_new;
    st.n_gated = fc.n_gated;
    st.n_new = fc.n_ins;
    st.n_del = fc.n_del;
    st.n_upd = fc.n_upd;
    st.n_casc = fc.n_casc;
    st.n_vertex_inserted = fc.n_inserted;
    st.n_vertex_deleted = fc.n_killed;
    st.ms_ingest = ev_ms(f.ev[0], f.ev[1]);
    st.ms_nodeops = ev_ms(f.ev[1], f.ev[2]);
    st.ms_sort_reduce = ev_ms(f.ev[2], f.ev[3]);
    st.ms_merge = ev_ms(f.ev[6], f.ev[4]);
    st.ms_degree_scan = ev_ms(f.ev[3], f.ev[6]) + ev_ms(f.ev[4], f.ev[5]);
    st.ms_total = ev_ms(f.ev[0], f.ev[5]);
    uint64_t b = 8 * (f.Vr + 1) + 8 * f.E + 8 * (fc.Vr_new + 1) + 8 * fc.En + 29 * f.n;
    if (f.node_mode) b += 16 * (f.V - fc.idmap_keep) + 4 * f.E + 4 * f.V;
    st.bytes_alg = b;
    uint64_t bm = 0;
    if (f.csr_changed && f.E + fc.n_ins) {
        bm = 8 * f.E + 8 * fc.En + 20 * fc.n_ins + 8 * fc.n_del + 12 * fc.n_upd;
        if (f.node_mode) bm += f.E / 8;
    }
    st.bytes_merge = bm;
    st.n_launches = f.launches;
    st.h2d_bytes = f.h2d;
    st.d2h_bytes = f.d2h;
    r->fin_ready = true;
    f.on = false;
}
// every call that reads the replica's sizes or contents first completes an asynchronous cycle
void ensure_final(const h2tap_replica* rc) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !r->infl.on) return;
    CK(cudaStreamSynchronize(r->st));
    finalize_inflight(r);
}

// One propagation cycle.  Nothing visible changes until the final swap.
h2tap_status apply_core(h2tap_replica* r, const BatchIn& in, uint64_t S, bool create, h2tap_apply_stats* stats) {
    cudaStream_t st = r->st;
    const uint64_t n = in.n, np = r->n_pend, m = np + n;
    if (r->prep.on) { set_err("a prepared cycle must be committed or aborted first"); return H2TAP_E_INVAL; }
    if (m >= 0xFFFFFFFFull) { set_err("batch + pending = %llu ops exceeds 2^32-1", (unsigned long long)m); return H2TAP_E_CAPACITY; }
    NvtxRange nv_cycle(create ? "h2tap create" : "h2tap cycle");
    g_launches = in.pre_launches;
    g_h2d = in.pre_h2d;
    g_d2h = in.pre_d2h;
    g_tr.init();
    g_ht.mark("core_start");
    const bool async = r->async_req && !create && !r->sharded && !r->defer_commit && !g_tr.on;
    for (int i = 0; i < 8; ++i)
        if (!r->ev[i]) CK(cudaEventCreate(&r->ev[i]));
    if (async || r->infl.on) {  // the in-flight cycle keeps its event set until it is finalised
        for (int i = 0; i < 8; ++i)
            if (!r->evx[i]) CK(cudaEventCreate(&r->evx[i]));
        std::swap(r->ev, r->evx);
    }
    CK(cudaStreamWaitEvent(st, r->evB, 0));  // a cascade pass of an earlier (failed) cycle is done
    CK(cudaStreamWaitEvent(st, r->evD, 0));  // and so is its merge partition (side stream)
    CK(cudaEventRecord(r->ev[0], st));
    TR("start");

    // ---- a1: assemble work ops (pending ++ batch) and partition
    uint8_t* Wk = r->get<uint8_t>(r->Wk, m);
    uint64_t* Ws = r->get<uint64_t>(r->Ws, m);
    uint64_t* Wd = r->get<uint64_t>(r->Wd, m);
    float* Ww = r->get<float>(r->Ww, m);
    uint64_t* Wt = r->get<uint64_t>(r->Wt, m);
    uint64_t* Wq = r->get<uint64_t>(r->Wq, m);
    const int pc = r->pcur;
    if (np) {
        CK(cudaMemcpyAsync(Wk, r->pk[pc].p, np, cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(Ws, r->ps[pc].p, np * 8, cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(Wd, r->pd[pc].p, np * 8, cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(Ww, r->pw[pc].p, np * 4, cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(Wt, r->pt[pc].p, np * 8, cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(Wq, r->pq[pc].p, np * 8, cudaMemcpyDeviceToDevice, st));
    }
    // a device-resident batch with nothing pending is read in place (no staging copy)
    const bool direct_in = n && !np && in.on_device && !in.recs && !in.drec && in.kind && in.dst && in.w && in.ts;
    if (direct_in) {
        if (in.seq) CK(cudaMemcpyAsync(Wq, in.seq, n * 8, cudaMemcpyDeviceToDevice, st));
        else { k_fill_seq<<<g1(n), 256, 0, st>>>(Wq, 0, n, r->next_seq); CKL(); }
    } else if (n && in.recs) {
        k_unpack_recs<<<g1(n), 256, 0, st>>>(in.recs, n, Wk + np, Ws + np, Wd + np, Ww + np, Wt + np, Wq + np);
        CKL();
    } else if (n && in.drec) {
        uint32_t* bigq = r->get<uint32_t>(r->xbig, in.n_drec);
        unsigned long long* nbig = reinterpret_cast<unsigned long long*>(r->get<uint64_t>(r->xnbig, 1));
        CK(cudaMemsetAsync(nbig, 0, 8, st));
        k_rec_expand<0><<<g1(in.n_drec), 256, 0, st>>>(in.drec, in.n_drec, in.drec_off, in.dins, in.dwts, in.ddel,
                                                      Wk + np, Ws + np, Wd + np, Ww + np, Wt + np, in.dwts64,
                                                      in.vis_ts, in.ins_base, in.del_base, bigq, nbig);
        CKL();
        k_rec_expand<1><<<(unsigned)r->n_sm * 8, 256, 0, st>>>(in.drec, in.n_drec, in.drec_off, in.dins, in.dwts,
                                                               in.ddel, Wk + np, Ws + np, Wd + np, Ww + np, Wt + np,
                                                               in.dwts64, in.vis_ts, in.ins_base, in.del_base, bigq,
                                                               nbig);
        CKL();
        k_fill_seq<<<g1(n), 256, 0, st>>>(Wq, np, n, r->next_seq);
        CKL();
    } else if (n) {
        if (in.kind) copy_in(r, Wk + np, in.kind, n, in.on_device);
        else { k_fill_u8<<<g1(n), 256, 0, st>>>(Wk + np, n, EDGE_INSERT); CKL(); }
        copy_in(r, Ws + np, in.src, n, in.on_device);
        if (in.dst) copy_in(r, Wd + np, in.dst, n, in.on_device);
        else CK(cudaMemsetAsync(Wd + np, 0, n * 8, st));
        if (in.w) copy_in(r, Ww + np, in.w, n, in.on_device);
        else CK(cudaMemsetAsync(Ww + np, 0, n * 4, st));
        if (in.ts) copy_in(r, Wt + np, in.ts, n, in.on_device);
        else { k_fill_u64<<<g1(n), 256, 0, st>>>(Wt + np, n, in.fill_ts); CKL(); }
        if (in.seq) copy_in(r, Wq + np, in.seq, n, in.on_device);
        else { k_fill_seq<<<g1(n), 256, 0, st>>>(Wq, np, n, r->next_seq); CKL(); }
    }
    const Ops ops = direct_in ? Ops{in.kind, in.src, in.dst, in.w, in.ts, Wq} : Ops{Wk, Ws, Wd, Ww, Wt, Wq};

    r->get<Counters>(r->ctr, 1);
    Counters* dc = r->dctr();
    k_init_counters<<<1, 32, 0, st>>>(dc);
    CKL();

    uint32_t* idx_p = r->get<uint32_t>(r->idx_p, m);
    uint32_t* idx_n = r->get<uint32_t>(r->idx_n, m);
    uint32_t* idx_e = r->get<uint32_t>(r->idx_e, m);
    if (m) {
        uint64_t nt = cdiv(m, kTile);
        uint64_t* stt = r->get<uint64_t>(r->status, 3 * nt);
        CK(cudaMemsetAsync(stt, 0, 3 * nt * 8, st));
        k_partition<<<(unsigned)nt, kThreads, 0, st>>>(ops, m, np, r->snap, S, create ? 0 : 1, idx_p, idx_n, idx_e,
                                                       stt, nt, dc);
        CKL();
    }
    // Speculation: when this replica's last cycles had no node ops (and the ID map is the
    // identity), the edge-op keys and their sort do not depend on anything the read-back below
    // returns - they are launched now, sized by upper bounds with the counts read on the device,
    // so the GPU keeps working while the host waits; a batch that does carry node ops discards
    // them and redoes both in node mode.
#ifndef H2TAP_SPECULATE
#define H2TAP_SPECULATE 1
#endif
    const bool spec = H2TAP_SPECULATE && m && !create && !r->sharded && r->identity && !r->last_node_mode &&
                      !(r->infl.on && r->infl.node_mode);
    uint64_t *sk = nullptr, *sk2 = nullptr;
    uint32_t *sv = nullptr, *sv2 = nullptr;
    // the first read-back: its store is enqueued before the speculative kernels and the host
    // waits for an event behind the store only, not for the stream
    g_d2h += sizeof(Counters);
    k_store_counters<<<1, 32, 0, st>>>(dc, r->hc_dev);
    CKL();
    if (!r->evS) CK(cudaEventCreateWithFlags(&r->evS, cudaEventDisableTiming));
    CK(cudaEventRecord(r->evS, st));
    if (spec) {
        sk = r->get<uint64_t>(r->keyA, m);
        sk2 = r->get<uint64_t>(r->keyB, m);
        sv = r->get<uint32_t>(r->valA, m);
        sv2 = r->get<uint32_t>(r->valB, m);
        const uint64_t Vs = r->V;  // no node ops in flight: the vertex count is final
        const int sbits = std::max(1, bits_for(Vs > 1 ? Vs - 1 : 1));
        PrepArgs pa{};
        pa.ops = ops;
        pa.edge_idx = idx_e;
        pa.n_edge = m;
        pa.count_dev = 1;
        pa.X = ext_index(r);
        pa.bits = sbits;
        pa.own = r->own;
        pa.keys = sk;
        pa.vals = sv;
        pa.recs = r->get<EdgeRec>(r->op_flags, m);
        const uint64_t nts = cdiv(m, (uint64_t)kThreads * 4);
        pa.status = r->get<uint64_t>(r->status2, nts);
        CK(cudaMemsetAsync(pa.status, 0, nts * 8, st));
        pa.n_tiles = nts;
        pa.c = dc;
        k_edge_prep<4><<<(unsigned)nts, kThreads, 0, st>>>(pa);
        CKL();
        radix_sort(r, sk, sv, sk2, sv2, m, 2 * sbits, &dc->n_valid);
    }
    TR("assemble+partition");
    g_ht.mark("a1_issued");
    CK(cudaEventSynchronize(r->evS));
    g_ht.mark("sync1");
    TR("sync1");
    if (r->infl.on) finalize_inflight(r);  // the previous (asynchronous) cycle's counters precede this read-back
    Counters hc = *r->hc;
    g_ht.mark("hc_read");
    if (hc.status & ST_BAD_KIND) { set_err("unknown op kind in batch"); return H2TAP_E_INVAL; }
    if (hc.status & ST_STALE) {
        set_err("op with ts <= current snapshot_ts %llu (reading A7)", (unsigned long long)r->snap);
        return H2TAP_E_STALE_TS;
    }
    const uint64_t n_pend_new = hc.n_pend, n_node = hc.n_node, n_edge = hc.n_edge;
    CK(cudaEventRecord(r->ev[1], st));

    // ---- a2: node ops -> per-vertex timeline, ID-map compaction, remap
    const uint64_t V = r->V, E = r->E, row_lo = r->row_lo, Vr = r->Vr;
    const int ec = r->ext_cur;
    const uint64_t* old_ext = static_cast<const uint64_t*>(r->ext[ec].p);
    // Only the sizes known after a1 (node ops, edge ops, pending) are host values from
    // here on; every later size (unique vertices, dropped/inserted vertices, surviving
    // edge ops, outcome lists, the new V and E) stays in device memory (Counters) and
    // the kernels read it there.  Buffers and grids are sized by upper bounds, so the
    // rest of the cycle runs without a host round trip until the final read-back.
    const bool node_mode = n_node > 0;
    const uint64_t Vn_ub = V + n_node;  // new vertices <= old + inserted
    if (Vn_ub >= 0x7FFFFFFFull) { set_err("vertex count could exceed 2^31-1"); return H2TAP_E_CAPACITY; }
    const uint64_t Vr_new_ub = node_mode ? Vn_ub : Vr;  // rows of the new CSR (shard rows <= all)
    NodeVtx* nv = nullptr;
    uint64_t* nv_ext = nullptr;
    RemapView R{};  // identity unless node ops shift the dense ids
    uint32_t *dropped = nullptr, *ins_q = nullptr, *ins_oldpos = nullptr, *hd_rows = nullptr,
             *hd_bits = nullptr, *node_sorted = nullptr;
    uint64_t* new_ext = nullptr;
    unsigned long long* idsame = nullptr;
    uint32_t* casc_mask = nullptr;
    bool casc_pending = false;  // cascade pass in flight on the side stream
    uint64_t *casc_cnt = nullptr, *casc_pre = nullptr;
    uint16_t* casc_wrel = nullptr;
    const int64_t* old_off_nc = static_cast<const int64_t*>(r->off[r->cur].p);
    const uint32_t* old_cols_nc = static_cast<const uint32_t*>(r->cols[r->cur].p);
    // node mode: the old-map lookups of the edge ops' endpoints, on the side stream beside the
    // node-op phase (k_edge_prep then reads them instead of searching the ID map while the
    // cascade pass streams the columns)
    uint32_t* epre = nullptr;
    if (node_mode && n_edge && !r->identity && H2TAP_EDGE_PRE) {
        epre = r->get<uint32_t>(r->epre, 2 * n_edge);
        if (!r->evE0) CK(cudaEventCreateWithFlags(&r->evE0, cudaEventDisableTiming));
        if (!r->evE1) CK(cudaEventCreateWithFlags(&r->evE1, cudaEventDisableTiming));
        CK(cudaEventRecord(r->evE0, st));
        CK(cudaStreamWaitEvent(r->st2, r->evE0, 0));
        k_edge_oldpos<<<g1(n_edge), 256, 0, r->st2>>>(ops, idx_e, dc, ext_index(r), epre);
        CKL();
        CK(cudaEventRecord(r->evE1, r->st2));
    }
    if (node_mode) {
        uint64_t* kA = r->get<uint64_t>(r->keyA, n_node);
        uint64_t* kB = r->get<uint64_t>(r->keyB, n_node);
        uint32_t* vA = r->get<uint32_t>(r->valA, n_node);
        uint32_t* vB = r->get<uint32_t>(r->valB, n_node);
        // (v, ts, seq) order: the input is in seq order and the sort is stable, so one sort
        // by the packed key (v - v_min, ts - ts_min) when both ranges fit in 64 bits, else
        // stable by ts, then stable by vertex
        const int vb = bits_for(hc.v_max - hc.v_min), tb = bits_for(hc.ts_max - hc.ts_min);
        if (vb + tb <= 64) {
            k_node_keys<<<g1(n_node), 256, 0, st>>>(idx_n, n_node, ops.src, hc.v_min, ops.ts, hc.ts_min, tb, kA, vA);
            CKL();
            radix_sort(r, kA, vA, kB, vB, n_node, vb + tb);
        } else {
            k_keys_from<<<g1(n_node), 256, 0, st>>>(idx_n, n_node, ops.ts, hc.ts_min, kA, vA);
            CKL();
            radix_sort(r, kA, vA, kB, vB, n_node, tb);
            k_keys_from<<<g1(n_node), 256, 0, st>>>(vA, n_node, ops.src, hc.v_min, kB, vB);
            CKL();
            std::swap(kA, kB);
            std::swap(vA, vB);
            radix_sort(r, kA, vA, kB, vB, n_node, vb);
        }
        TR("node_sort");
        node_sorted = r->get<uint32_t>(r->nsorted, n_node);
        CK(cudaMemcpyAsync(node_sorted, vA, n_node * 4, cudaMemcpyDeviceToDevice, st));

        nv = r->get<NodeVtx>(r->nv, n_node);
        nv_ext = r->get<uint64_t>(r->nv_ext, n_node);
        const uint64_t nt = cdiv(n_node, kTile);  // tile bound of the unique-vertex list
        const uint64_t nts = cdiv(n_node, kSegTile);
        uint64_t* stt = r->get<uint64_t>(r->status, 3 * nt + nts);
        CK(cudaMemsetAsync(stt, 0, (3 * nt + nts) * 8, st));
        k_node_segments<<<(unsigned)nts, kThreads, 0, st>>>(ops, node_sorted, n_node, ext_index(r), nv, nv_ext,
                                                            stt + 3 * nt, nts, dc);
        CKL();
        TR("node_segments");
        dropped = r->get<uint32_t>(r->dropped, n_node);
        ins_q = r->get<uint32_t>(r->ins_q, n_node);
        ins_oldpos = r->get<uint32_t>(r->ins_oldpos, n_node);
        hd_rows = r->get<uint32_t>(r->hd_rows, n_node);
        hd_bits = r->get<uint32_t>(r->hd_bits, cdiv(V, 32));  // deleted vertices (set by k_node_lists)
        CK(cudaMemsetAsync(hd_bits, 0, cdiv(V, 32) * 4, st));
        k_node_lists<<<(unsigned)nt, kThreads, 0, st>>>(nv, dropped, ins_q, ins_oldpos, hd_rows, hd_bits, stt, nt, dc,
                                                        r->tomb ? 1 : 0);
        CKL();
        TR("node_lists");
        const uint64_t nblk_c = cdiv(E, kCascBlock);
        casc_mask = r->get<uint32_t>(r->casc_mask, (nblk_c + 2) * (kCascBlock / 32));
        casc_cnt = r->get<uint64_t>(r->tile_emit, nblk_c + 1);
        casc_pre = r->get<uint64_t>(r->tile_base, nblk_c + 1);
        unsigned rg = (unsigned)std::min<uint64_t>(cdiv(n_node * 32, 256), (uint64_t)r->n_sm * 8);
        const uint64_t nst = cdiv(nblk_c + 1, kThreads);
        uint64_t* st2s2 = r->get<uint64_t>(r->casc_status, nst);
        CK(cudaMemsetAsync(st2s2, 0, nst * 8, st));
        casc_wrel = r->get<uint16_t>(r->casc_wrel, (nblk_c + 1) * (kCascBlock / 32));
        // The cascade pass (a4, reading A8: one bit per old element removed by a node delete)
        // streams the old columns (HBM-bound) and nothing before the row pass reads its
        // output, so it starts as soon as the deleted vertices are known and runs on the side
        // stream beside the remap tables and the edge-op phase; the row pass joins it
        // (casc_join) before reading the cascade tables.
#ifndef H2TAP_CASC_MAIN
#define H2TAP_CASC_MAIN 0
#endif
        CK(cudaEventRecord(r->evA, st));
        CK(cudaStreamWaitEvent(r->st2, r->evA, 0));
        cudaStream_t cs = H2TAP_CASC_MAIN ? st : r->st2;
        if (nblk_c) {
            if (H2TAP_CASC_TMA) {
                static bool attr = false;
                if (!attr) { CK(cudaFuncSetAttribute(k_casc_cols_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, kCcSmem)); attr = true; }
                const unsigned gc = (unsigned)std::min<uint64_t>(cdiv(E, kCcChunk), (uint64_t)r->n_sm * H2TAP_CC_CTAS / 8);
                k_casc_cols_tma<<<gc, kCcThreads, kCcSmem, cs>>>(old_cols_nc, E, hd_bits, hd_rows, dc, casc_mask);
            } else {
                const unsigned gc = (unsigned)std::min<uint64_t>(cdiv(nblk_c, 2), (uint64_t)r->n_sm * kCascCtasPerSm);
                k_casc_cols<<<gc, kThreads, 0, cs>>>(old_cols_nc, E, hd_bits, hd_rows, dc, casc_mask);
            }
            CKL();
            k_casc_rows<<<rg, 256, 0, cs>>>(old_off_nc, hd_rows, dc, row_lo, row_lo + Vr, casc_mask);
            CKL();
        }
        k_casc_scan<<<(unsigned)nst, kThreads, 0, cs>>>(casc_mask, nblk_c, casc_pre, casc_wrel, st2s2, &dc->tiles[6]);
        CKL();
        k_copy_u64<<<1, 1, 0, cs>>>(&dc->n_casc, casc_pre + nblk_c);
        CKL();
        CK(cudaEventRecord(r->evB, cs));
        casc_pending = true;
        // ID-map compaction: remap tables (64K-id block shifts, 32-id groups, the
        // unchanged / uniformly shifted id ranges), then the survivors and the inserted
        const size_t ext_cap = r->ext[ec ^ 1].cap;  // a regrow (even at the same address) zeroes it
        new_ext = r->get<uint64_t>(r->ext[ec ^ 1], Vn_ub);
        idsame = r->get<unsigned long long>(r->idsame, 2);
        if (r->ext[ec ^ 1].cap != ext_cap) CK(cudaMemsetAsync(idsame, 0, 16, st));  // fresh back buffer
        const uint64_t nblk = cdiv(V, 1ull << kRemapBlockShift), ng = cdiv(V, 32);
        int32_t* rs = r->get<int32_t>(r->remap_shift, nblk + 8);  // + lohi (6 entries)
        uint2* r32 = r->get<uint2>(r->remap32, ng);
        k_remap_tables<<<g1(std::max(nblk, ng)), 256, 0, st>>>(V, dropped, ins_oldpos, dc, rs, rs + nblk, r32);  // + c->Vn
        CKL();
        R.shift = rs; R.g32 = r32; R.ins_oldpos = ins_oldpos; R.n_vins = &dc->n_inserted; R.lohi = rs + nblk;
        TR("remap_tables");
        // the inserted vertices' ID-map entries now; the survivors' entries are written
        // by k_rows_fused together with the new row offsets
        // (+ the node-op vertices' new ids)
        k_node_place<<<g1(n_node), 256, 0, st>>>(nv, nv_ext, ins_q, ins_oldpos, dropped, dc, new_ext, R);
        CKL();
        TR("nv_newid");
        if (r->sharded) {
            k_row_range_new<<<1, 1, 0, st>>>(dropped, ins_q, nv_ext, row_lo, row_lo + Vr, r->own, dc);
            CKL();
        }
    }
    CK(cudaEventRecord(r->ev[2], st));
    g_ht.mark("idmap");
    TR("idmap+remap");

    // ---- a3: edge ops -> keys, sort, segmented reduce + classify
    const int bits = std::max(1, bits_for(Vn_ub > 1 ? Vn_ub - 1 : 1));  // dense ids < Vn <= Vn_ub
    const int64_t* old_off = static_cast<const int64_t*>(r->off[r->cur].p);
    const uint32_t* old_cols = static_cast<const uint32_t*>(r->cols[r->cur].p);
    const float* old_w = static_cast<const float*>(r->w[r->cur].p);
    uint64_t* ins_pos = r->get<uint64_t>(r->ins_pos, n_edge);
    uint32_t* ins_row = r->get<uint32_t>(r->ins_row, n_edge);
    uint32_t* ins_col = r->get<uint32_t>(r->ins_col, n_edge);
    float* ins_w = r->get<float>(r->ins_w, n_edge);
    uint64_t* del_pos = r->get<uint64_t>(r->del_pos, n_edge);
    uint32_t* del_row = r->get<uint32_t>(r->del_row, n_edge);
    uint64_t* upd_pos = r->get<uint64_t>(r->upd_pos, n_edge);
    float* upd_w = r->get<float>(r->upd_w, n_edge);
    if (n_edge) {
        uint64_t* kA = r->get<uint64_t>(r->keyA, n_edge);
        uint64_t* kB = r->get<uint64_t>(r->keyB, n_edge);
        uint32_t* vA = r->get<uint32_t>(r->valA, n_edge);
        uint32_t* vB = r->get<uint32_t>(r->valB, n_edge);
        const bool spec_ok = spec && !node_mode;  // the speculative keys are this cycle's keys
        PrepArgs pa{};
        pa.ops = ops;
        pa.edge_idx = idx_e;
        pa.n_edge = n_edge;
        pa.X = ext_index(r);
        pa.R = R;
        pa.nv = nv;
        pa.nv_ext = nv_ext;
        pa.node_sorted = node_sorted;
        pa.bits = bits;
        pa.create = create ? 1 : 0;
        pa.own = r->own;
        pa.keys = kA;
        pa.vals = vA;
        pa.recs = r->get<EdgeRec>(r->op_flags, m);
        if (epre) {  // the endpoints' old-map lookups (side stream)
            CK(cudaStreamWaitEvent(st, r->evE1, 0));
            pa.epre = epre;
        }
        const bool lookups_direct = r->identity && !node_mode;  // no searches -> 4 ops per thread
#ifndef H2TAP_EI_DIRECT
#define H2TAP_EI_DIRECT 4
#endif
        const int eitems = lookups_direct ? H2TAP_EI_DIRECT : 1;
        uint64_t nt = cdiv(n_edge, (uint64_t)kThreads * eitems);
        pa.status = r->get<uint64_t>(r->status, 3 * nt);
        CK(cudaMemsetAsync(pa.status, 0, nt * 8, st));
        pa.n_tiles = nt;
        pa.c = dc;
        if (spec_ok) {
            kA = sk; vA = sv;
        } else {
            if (spec) {  // discard the speculative keys: counters and the tile ticket start over
                CK(cudaMemsetAsync(&dc->n_valid, 0, 8, st));
                CK(cudaMemsetAsync(&dc->n_gated, 0, 8, st));
                CK(cudaMemsetAsync(&dc->tiles[3], 0, 4, st));
            }
            if (lookups_direct) k_edge_prep<H2TAP_EI_DIRECT><<<(unsigned)nt, kThreads, 0, st>>>(pa);
            else k_edge_prep<1><<<(unsigned)nt, kThreads, 0, st>>>(pa);
            CKL();
            TR("edge_prep");
            radix_sort(r, kA, vA, kB, vB, n_edge, 2 * bits, &dc->n_valid);
        }
        TR("edge_sort");
        ClassArgs ca{};
        ca.ops = ops;
        ca.keys = kA;
        ca.vals = vA;
        ca.n = n_edge;  // upper bound; the kernel reads n_valid
        ca.bits = bits;
        ca.recs = pa.recs;
        ca.old_off = old_off - row_lo;  // indexed by global dense ids of owned rows
        ca.old_cols = old_cols;
        ca.V_old = V;
        ca.direct = node_mode ? 0 : 1;  // identity remap: the key's row is the old row
        ca.ins_pos = ins_pos; ca.ins_row = ins_row; ca.ins_col = ins_col; ca.ins_w = ins_w;
        ca.del_pos = del_pos;
        ca.del_row = del_row;
        ca.upd_pos = upd_pos; ca.upd_w = upd_w;
#ifndef H2TAP_CLASSIFY_SPLIT
#define H2TAP_CLASSIFY_SPLIT (1u << 16)  // edge ops from which classification and compaction are split
#endif
        ca.c = dc;
        if (n_edge >= H2TAP_CLASSIFY_SPLIT) {
            ca.kcat = r->get<uint8_t>(r->cls_cat, n_edge);
            ca.kpos = r->get<uint64_t>(r->cls_pos, n_edge);
            ca.kw = r->get<float>(r->cls_w, n_edge);
            k_reduce_classify<1><<<(unsigned)cdiv(n_edge, kCTile), kThreads, 0, st>>>(ca);
            CKL();
            const uint64_t nt3 = cdiv(n_edge, kTile);
            ca.status3 = r->get<uint64_t>(r->status2, 3 * nt3);
            CK(cudaMemsetAsync(ca.status3, 0, 3 * nt3 * 8, st));
            ca.n_tiles = nt3;
            k_classify_compact<<<(unsigned)nt3, kThreads, 0, st>>>(ca);
            CKL();
        } else {
            uint64_t nt2 = cdiv(n_edge, kCTile);
            ca.status3 = r->get<uint64_t>(r->status2, 3 * nt2);
            CK(cudaMemsetAsync(ca.status3, 0, 3 * nt2 * 8, st));
            ca.n_tiles = nt2;
            k_reduce_classify<0><<<(unsigned)nt2, kThreads, 0, st>>>(ca);
            CKL();
        }
        TR("classify");
    }
    CK(cudaEventRecord(r->ev[3], st));
    // ---- new pending set (double-buffered so an error above leaves the old one intact): the
    // last reader of the input arrays, so a staged batch's slot may be refilled from here on
    // (the next-but-one batch's H2D copy then overlaps this cycle's merge)
    const int pn = pc ^ 1;
    if (n_pend_new) {
        k_gather_ops<<<g1(n_pend_new), 256, 0, st>>>(
            ops, idx_p, n_pend_new, r->get<uint8_t>(r->pk[pn], n_pend_new), r->get<uint64_t>(r->ps[pn], n_pend_new),
            r->get<uint64_t>(r->pd[pn], n_pend_new), r->get<float>(r->pw[pn], n_pend_new),
            r->get<uint64_t>(r->pt[pn], n_pend_new), r->get<uint64_t>(r->pq[pn], n_pend_new));
        CKL();
    }
    if (in.input_done) CK(cudaEventRecord(in.input_done, st));

    // ---- a6 prerequisite: the merge-path partition depends only on the outcome lists (and the
    // cascade tables, which the side stream already produces), so it runs on the side stream
    // beside the row-offset / ID-map pass of the main stream
    const bool csr_changed = node_mode || n_edge;
    const uint64_t Ecap_ = E + n_edge;
    TilePart* part = nullptr;
    MergeArgs mp{};
    if (csr_changed && Ecap_) {
        mp.E_old = E;
        mp.ins_pos = ins_pos;
        mp.del_pos = del_pos;
        mp.upd_pos = upd_pos;
        mp.n_tiles = cdiv(Ecap_, kMergeTile);  // upper bound; the kernels use E + n_ins
        mp.c = dc;
        if (node_mode) { mp.casc_mask = casc_mask; mp.casc_pre = casc_pre; }
        part = r->get<TilePart>(r->part, mp.n_tiles + 1);
        CK(cudaEventRecord(r->evC, st));
        CK(cudaStreamWaitEvent(r->st2, r->evC, 0));
        k_merge_partition<<<g1(mp.n_tiles + 1), 256, 0, r->st2>>>(mp, part);
        CKL();
        CK(cudaEventRecord(r->evD, r->st2));
    }

    // ---- a6: merge into the back buffer (skipped when no op can change the CSR)
    const int nb = csr_changed ? (r->cur ^ 1) : r->cur;
    int64_t* new_off = nullptr;
    const bool casc = node_mode;
    if (csr_changed) {
    const uint64_t Ecap = E + n_edge;  // >= E + n_ins
    new_off = r->get<int64_t>(r->off[nb], Vr_new_ub + 1);
    uint32_t* new_cols = r->get<uint32_t>(r->cols[nb], Ecap);
    float* new_w = r->get<float>(r->w[nb], Ecap);
    // node mode: survivors' ID map + row offsets before the merge, while the cascade
    // tables written by the cascade pass are still L2-resident (the merge streams the CSR)
    if (node_mode) {
        RowArgs ra{};
        ra.old_off = old_off - row_lo; ra.V_old = V; ra.E_old = E; ra.R = R;
        ra.row_lo = row_lo; ra.row_hi = row_lo + Vr;
        ra.own = r->own; ra.nv_ext = nv_ext;
        ra.casc_mask = casc_mask; ra.casc_pre = casc_pre; ra.casc_wrel = casc_wrel;
        ra.del_pos = del_pos; ra.ins_row = ins_row;
        ra.dropped = dropped; ra.ins_oldpos = ins_oldpos;
        ra.new_off = new_off;
        ra.c = dc;
        ra.old_ext = old_ext; ra.new_ext = new_ext; ra.identity = r->identity ? 1 : 0;
        ra.same = H2TAP_IDMAP_KEEP ? idsame : nullptr;
        uint8_t* new_live = nullptr;
        if (r->tomb) {
            ra.old_live = static_cast<const uint8_t*>(r->live[ec].p);
            ra.new_live = new_live = r->get<uint8_t>(r->live[ec ^ 1], Vn_ub);
        }
        const uint64_t ncta = cdiv(V, kRowTile);
        ra.part = r->get<uint64_t>(r->opart, 2 * (ncta + 1));
        if (V) {
            k_rows_partition<><<<g1(ncta + 1), 256, 0, st>>>(ra);  // reads no cascade table
            CKL();
        }
        if (casc_pending) {  // join the cascade pass (side stream) before its tables are read
            CK(cudaStreamWaitEvent(st, r->evB, 0));
            casc_pending = false;
            TR("casc_join");
        }
        if (V) {
            k_rows_fused<<<(unsigned)ncta, kThreads, 0, st>>>(ra);  // survivors: ID map + row offsets
            CKL();
        } else {
            CK(cudaMemsetAsync(idsame, 0, 16, st));
        }
        // the inserted vertices' rows, the new ID map's fence and the ID-map prefix mark
        uint64_t* f = r->get<uint64_t>(r->fence[ec ^ 1], n_fence(Vn_ub));
        k_rows_finish<<<std::max(g1(n_node), g1(n_fence(Vn_ub))), 256, 0, st>>>(
            nv, ins_q, ra, new_ext, f, idsame, R.lohi, (r->tomb || !H2TAP_IDMAP_KEEP) ? 1 : 0, V ? 1 : 0);
        CKL();
        if (new_live) {  // node-op vertices' final liveness over the carried flags
            k_nv_live<<<g1(n_node), 256, 0, st>>>(nv, dc, R, new_live);
            CKL();
        }
    }
    // ---- a4/a5 without node ops: row offsets (while the outcome lists are L2-resident)
    if (Vr && !node_mode) {
        // new_off[k] = old_off[k] - (deletes before it) + (inserts in earlier rows): two
        // ranks in the sorted outcome lists, one streaming pass over the shard's rows
        RowArgs ra{};
        ra.old_off = old_off - row_lo; ra.V_old = V; ra.E_old = E;
        ra.row_lo = row_lo; ra.row_hi = row_lo + Vr;
        ra.del_pos = del_pos; ra.del_row = del_row; ra.ins_row = ins_row;
        ra.new_off = new_off;
        ra.c = dc;
        const uint64_t ncta = cdiv(V, kOffTile);
        ra.part = r->get<uint64_t>(r->opart, 2 * (ncta + 1));
        k_offsets_bounds<<<(unsigned)std::min<uint64_t>(g1(n_edge + 1), (uint64_t)r->n_sm * 16), 256, 0, st>>>(
            del_row, ins_row, dc, n_edge, ncta, ra.part);
        CKL();
        const uint64_t c_lo = row_lo / kOffTile, c_hi = cdiv(row_lo + Vr, kOffTile);
        k_offsets_direct<<<(unsigned)(c_hi - c_lo), kThreads, 0, st>>>(ra);
        CKL();
    }
    if (Ecap) {
        MergeArgs ma{};
        ma.old_cols = old_cols; ma.old_w = old_w; ma.E_old = E;
        ma.ins_pos = ins_pos; ma.ins_col = ins_col; ma.ins_w = ins_w;
        ma.del_pos = del_pos;
        ma.upd_pos = upd_pos; ma.upd_w = upd_w;
        ma.R = R;
        ma.new_cols = new_cols; ma.new_w = new_w;
        ma.n_tiles = cdiv(Ecap, kMergeTile);  // upper bound; the kernels use E + n_ins
        ma.c = dc;
        if (casc) {
            ma.casc_mask = casc_mask;
            ma.casc_pre = casc_pre;
        }
        CK(cudaStreamWaitEvent(st, r->evD, 0));  // the partition (side stream) is complete
        if (casc_pending) { CK(cudaStreamWaitEvent(st, r->evB, 0)); casc_pending = false; }
        CK(cudaEventRecord(r->ev[6], st));  // merge kernel starts here (after its prerequisites)
        TR("merge_prep+casc_join");
        auto launch = [&](auto kern) {
            int occ = 0;
            CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kMerge3Smem));
            CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kThreads, kMerge3Smem));
            if (H2TAP_MERGE_CTAS > 0) occ = std::min(occ, (int)H2TAP_MERGE_CTAS);
            const uint64_t grid = std::min<uint64_t>(ma.n_tiles, (uint64_t)std::max(1, occ) * r->n_sm);
            kern<<<(unsigned)grid, kThreads, kMerge3Smem, st>>>(ma, part);
        };
        if (node_mode) launch(k_merge3<true, true>);
        else launch(k_merge3<false, false>);
        CKL();
        if (in.after_merge_launch) (*in.after_merge_launch)();
    } else {
        CK(cudaEventRecord(r->ev[6], st));
    }
    CK(cudaEventRecord(r->ev[4], st));
    TR("merge");

    } else {
        CK(cudaEventRecord(r->ev[6], st));
        CK(cudaEventRecord(r->ev[4], st));
    }

    k_finish<<<1, 1, 0, st>>>(dc, V, Vr, E, node_mode ? 1 : 0, r->sharded ? 1 : 0, new_ext, new_off);
    CKL();
    CK(cudaEventRecord(r->ev[5], st));
    TR("offsets+pending");
    if (async) {  // enqueue the final read-back and return; finalize_inflight completes the cycle
        k_store_counters<<<1, 32, 0, st>>>(dc, r->hcf_dev);
        CKL();
        h2tap_replica::Inflight& f = r->infl;
        f.on = true;
        for (int i = 0; i < 8; ++i) f.ev[i] = r->ev[i];
        f.node_mode = node_mode; f.csr_changed = csr_changed;
        f.n = n; f.n_node = n_node; f.n_edge = n_edge; f.n_pend_new = n_pend_new;
        f.V = V; f.Vr = Vr; f.E = E; f.row_lo = row_lo;
        f.launches = g_launches; f.h2d = g_h2d; f.d2h = g_d2h + sizeof(Counters);
        // the part of the swap that needs no counter (what the next cycle reads first)
        r->cur = nb;
        if (node_mode) { r->ext_cur = ec ^ 1; r->idmap_swapped(); }
        r->pcur = pc ^ 1;
        r->n_pend = n_pend_new;
        r->next_seq += n;
        r->snap = S;
        r->last_node_mode = node_mode;
        if (stats) memset(stats, 0, sizeof *stats);
        return H2TAP_OK;
    }
    if (in.before_readback) (*in.before_readback)();
    g_ht.mark("issued");
    r->read_counters();  // the one read-back of the cycle's device-side sizes
    TR("end");
    g_ht.mark("core_end");
    g_tr.dump();
    const Counters& fc = *r->hc;
    if (create && (fc.status & ST_CREATE_ENDPOINT)) {
        set_err("create: edge endpoint not in the vertex set");
        return H2TAP_E_INVAL;
    }
    if (fc.status & ST_NOT_OWNED) {
        set_err("sharded replica: edge op whose source is owned by another shard");
        return H2TAP_E_INVAL;
    }
    const uint64_t Vn = fc.Vn, Vr_new = fc.Vr_new, En = fc.En;
    const uint64_t row_lo_new = (node_mode && r->sharded) ? fc.row_lo_new : row_lo;
    const uint64_t n_ins = fc.n_ins, n_del = fc.n_del, n_upd = fc.n_upd, n_casc = fc.n_casc;

    // ---- a7: swap at snapshot_ts (nothing above touched the front state).  Two-phase
    // (h2tap_delta_*_prepare): the new state waits in the back buffers for commit/abort.
    h2tap_replica::Prep& pr = r->prep;
    pr.nb = nb; pr.pn = pn; pr.node_mode = node_mode; pr.ext_new = ec ^ 1;
    pr.identity = fc.new_identity == 1;
    pr.V = Vn; pr.E = En; pr.row_lo = row_lo_new; pr.Vr = Vr_new; pr.n_pend = n_pend_new; pr.n = n; pr.S = S;
    pr.on = true;
    if (!r->defer_commit) r->commit();
    r->last_node_mode = node_mode;
    if (stats) {
        memset(stats, 0, sizeof *stats);
        stats->n_visible = n_node + n_edge;
        stats->n_deferred = n_pend_new;
        stats->n_gated = fc.n_gated;
        stats->n_new = n_ins;
        stats->n_del = n_del;
        stats->n_upd = n_upd;
        stats->n_casc = n_casc;
        stats->n_vertex_inserted = fc.n_inserted;
        stats->n_vertex_deleted = fc.n_killed;  // live before the cycle, dead after it (both ID modes)
        stats->ms_ingest = ev_ms(r->ev[0], r->ev[1]);
        stats->ms_nodeops = ev_ms(r->ev[1], r->ev[2]);
        stats->ms_sort_reduce = ev_ms(r->ev[2], r->ev[3]);
        // merge = the merge kernel alone; its prerequisites (remap tables, merge-path
        // partition, cascade-pass join) and the offsets/pending epilogue are "degree_scan"
        stats->ms_merge = ev_ms(r->ev[6], r->ev[4]);
        stats->ms_degree_scan = ev_ms(r->ev[3], r->ev[6]) + ev_ms(r->ev[4], r->ev[5]);
        stats->ms_total = ev_ms(r->ev[0], r->ev[5]);
        uint64_t b = 8 * (Vr + 1) + 8 * E + 8 * (Vr_new + 1) + 8 * En + 29 * n;
        if (node_mode) b += 16 * (V - fc.idmap_keep) + 4 * E + 4 * V;
        stats->bytes_alg = b;
        // merge launch: stream old cols+weights, write new ones, read the outcome lists
        // (+ remap table and cascade bitmap when node ops changed the ID map)
        uint64_t bm = 0;
        if (csr_changed && E + n_ins) {
            bm = 8 * E + 8 * En + 20 * n_ins + 8 * n_del + 12 * n_upd;
            if (node_mode) bm += E / 8;                                  // cascade mask
        }
        stats->bytes_merge = bm;
        stats->n_launches = g_launches;
        stats->h2d_bytes = g_h2d;
        stats->d2h_bytes = g_d2h;
    }
    return H2TAP_OK;
}

template <typename F>
h2tap_status run_guarded(h2tap_replica* r, F&& f) {
    if (r && r->poisoned) { set_err("replica poisoned by an earlier CUDA error"); return H2TAP_E_POISONED; }
    try {
        return f();
    } catch (const Fail& e) {
        if (r && e.st == H2TAP_E_CUDA) {
            cudaError_t s = cudaDeviceSynchronize();
            if (s != cudaSuccess) r->poisoned = true;
            cudaGetLastError();
        }
        return e.st;
    } catch (const std::bad_alloc&) {
        set_err("host allocation failed");
        return H2TAP_E_NOMEM;
    } catch (...) {
        set_err("unexpected C++ exception");
        return H2TAP_E_CUDA;
    }
}

h2tap_replica* new_replica(const h2tap_config* cfg) {
    h2tap_replica* r = new h2tap_replica();
    if (cfg) r->cfg = *cfg;
    else { r->cfg.world = 1; }
    if (r->cfg.world <= 0) r->cfg.world = 1;
    if (r->cfg.id_mode != H2TAP_ID_COMPACT && r->cfg.id_mode != H2TAP_ID_TOMBSTONE) {
        set_err("id_mode must be H2TAP_ID_COMPACT or H2TAP_ID_TOMBSTONE");
        throw Fail{H2TAP_E_INVAL};
    }
    r->tomb = r->cfg.id_mode == H2TAP_ID_TOMBSTONE;
    if (r->tomb && r->cfg.world > 1) {
        set_err("tombstone-row mode is single-replica only in this build");
        throw Fail{H2TAP_E_INVAL};
    }
    static const uint64_t kOneShard[2] = {0, ~0ull};
    if (r->cfg.nccl_unique_id && r->cfg.world == 1 && !r->cfg.shard_bounds) r->cfg.shard_bounds = kOneShard;
    if (r->cfg.world > 1 || r->cfg.nccl_unique_id) {
        if (!r->cfg.shard_bounds || r->cfg.rank < 0 || r->cfg.rank >= r->cfg.world) {
            set_err("sharded replica needs shard_bounds[world+1] and 0 <= rank < world");
            throw Fail{H2TAP_E_INVAL};
        }
        if (r->cfg.world > 4096) { set_err("world > 4096"); throw Fail{H2TAP_E_INVAL}; }
        for (int p = 0; p < r->cfg.world; ++p)
            if (r->cfg.shard_bounds[p] > r->cfg.shard_bounds[p + 1]) {
                set_err("shard_bounds must be non-decreasing");
                throw Fail{H2TAP_E_INVAL};
            }
        r->sharded = true;
        uint64_t* bd = r->get<uint64_t>(r->bounds_dev, r->cfg.world + 1);
        CK(cudaMemcpy(bd, r->cfg.shard_bounds, (r->cfg.world + 1) * 8, cudaMemcpyHostToDevice));
        r->own.lo = r->cfg.shard_bounds[r->cfg.rank];
        r->own.hi = (r->cfg.rank == r->cfg.world - 1) ? ~0ull : r->cfg.shard_bounds[r->cfg.rank + 1];
        r->cfg.shard_bounds = nullptr;  // not retained
    }
    CK(cudaSetDevice(r->cfg.device));
    if (r->cfg.nccl_unique_id) coll::init_comm(r);  // collective: every rank creates its shard
    CK(cudaDeviceGetAttribute(&r->n_sm, cudaDevAttrMultiProcessorCount, r->cfg.device));
    r->st = static_cast<cudaStream_t>(r->cfg.stream);
    {   // side stream at the lowest priority: its streaming work fills gaps left by the
        // latency-bound main-stream kernels instead of delaying them
        int lo = 0, hi = 0;
        CK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
        CK(cudaStreamCreateWithPriority(&r->st2, cudaStreamNonBlocking, lo));
        CK(cudaStreamCreateWithFlags(&r->st_copy, cudaStreamNonBlocking));
        for (auto& g : r->stg) {
            CK(cudaEventCreateWithFlags(&g.ev, cudaEventDisableTiming));
            CK(cudaEventCreateWithFlags(&g.done, cudaEventDisableTiming));
        }
    }
    CK(cudaEventCreateWithFlags(&r->evA, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&r->evB, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&r->evC, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&r->evD, cudaEventDisableTiming));
    CK(cudaHostAlloc(reinterpret_cast<void**>(&r->hc), sizeof(Counters), cudaHostAllocMapped));
    CK(cudaHostGetDevicePointer(reinterpret_cast<void**>(&r->hc_dev), r->hc, 0));
    CK(cudaHostAlloc(reinterpret_cast<void**>(&r->hcf), sizeof(Counters), cudaHostAllocMapped));
    CK(cudaHostGetDevicePointer(reinterpret_cast<void**>(&r->hcf_dev), r->hcf, 0));
    CK(cudaHostAlloc(reinterpret_cast<void**>(&r->hx), 64, cudaHostAllocMapped));
    CK(cudaHostGetDevicePointer(reinterpret_cast<void**>(&r->hx_dev), r->hx, 0));
    r->get<Counters>(r->ctr, 1);
    return r;
}

void free_replica(h2tap_replica* r) {
    if (!r) return;
    if (r->comm) coll::destroy_comm(r);
    Buf* bufs[] = {&r->off[0], &r->off[1], &r->cols[0], &r->cols[1], &r->w[0], &r->w[1], &r->ext[0], &r->ext[1],
                   &r->pk[0], &r->pk[1], &r->ps[0], &r->ps[1], &r->pd[0], &r->pd[1], &r->pw[0], &r->pw[1],
                   &r->pt[0], &r->pt[1], &r->pq[0], &r->pq[1], &r->Wk, &r->Ws, &r->Wd, &r->Ww, &r->Wt, &r->Wq,
                   &r->idx_p, &r->idx_n, &r->idx_e, &r->status, &r->keyA, &r->keyB, &r->valA, &r->valB,
                   &r->hist, &r->dbase, &r->rs_status, &r->rs_ctr, &r->rs_coop, &r->nv, &r->nv_ext, &r->dropped, &r->ins_q,
                   &r->ins_oldpos, &r->hd_rows, &r->hd_bits, &r->op_flags, &r->op_ou, &r->op_ow,
                   &r->ins_pos, &r->ins_row, &r->ins_col, &r->ins_w, &r->del_pos, &r->upd_pos, &r->upd_w,
                   &r->KR, &r->cls_cat, &r->cls_pos, &r->cls_w, &r->misc, &r->nsorted, &r->part, &r->opart, &r->deg, &r->tsum, &r->remap_shift, &r->remap32, &r->casc_wrel, &r->tile_emit, &r->tile_base, &r->del_row, &r->casc_mask, &r->status2, &r->bounds_dev, &r->fence[0], &r->fence[1], &r->bfs_a, &r->bfs_b, &r->pr_a, &r->pr_b, &r->ctr,
                   &r->xrec, &r->xins, &r->xwts, &r->xdel, &r->xcnt, &r->xoff, &r->xbig, &r->xnbig, &r->live[0], &r->live[1], &r->casc_status, &r->idsame, &r->epre, &r->coll, &r->coll_send, &r->coll_recv};
    for (Buf* b : bufs) if (b->p) r->dfree(b->p);
    cudaStreamSynchronize(r->st);
    for (auto& e : r->ev) if (e) cudaEventDestroy(e);
    if (r->evA) cudaEventDestroy(r->evA);
    if (r->evB) cudaEventDestroy(r->evB);
    if (r->evC) cudaEventDestroy(r->evC);
    if (r->evD) cudaEventDestroy(r->evD);
    if (r->evS) cudaEventDestroy(r->evS);
    if (r->evE0) cudaEventDestroy(r->evE0);
    if (r->evE1) cudaEventDestroy(r->evE1);
    if (r->st2) { cudaStreamSynchronize(r->st2); cudaStreamDestroy(r->st2); }
    if (r->st_copy) { cudaStreamSynchronize(r->st_copy); cudaStreamDestroy(r->st_copy); }
    for (auto& g : r->stg) {
        for (Buf* b : {&g.k, &g.s, &g.d, &g.w, &g.t}) if (b->p) r->dfree(b->p);
        if (g.ev) cudaEventDestroy(g.ev);
        if (g.done) cudaEventDestroy(g.done);
    }
    if (r->hc) cudaFreeHost(r->hc);
    if (r->hcf) cudaFreeHost(r->hcf);
    if (r->hx) cudaFreeHost(r->hx);
    for (auto& e : r->evx) if (e) cudaEventDestroy(e);
    delete r;
}

// empty replica over a vertex set (ids strictly increasing or identity)
void init_vertices(h2tap_replica* r, uint64_t nv, const uint64_t* ids, int on_device) {
    r->V = nv;
    r->E = 0;
    uint64_t* ext = r->get<uint64_t>(r->ext[0], nv);
    CK(cudaMemsetAsync(r->get<unsigned long long>(r->idsame, 2), 0, 16, r->st));  // back buffer unknown
    if (ids) copy_in(r, ext, ids, nv, on_device);
    else if (nv) { k_iota_u64<<<g1(nv), 256, 0, r->st>>>(ext, nv); CKL(); }
    int64_t* off = r->get<int64_t>(r->off[0], nv + 1);
    CK(cudaMemsetAsync(off, 0, (nv + 1) * 8, r->st));
    r->get<uint32_t>(r->cols[0], 0);
    r->get<float>(r->w[0], 0);
    r->identity = (ids == nullptr);
    if (ids && nv) {
        // validate strictly increasing ids (and detect identity)
        unsigned long long* bad = r->get<unsigned long long>(r->misc, 1);
        CK(cudaMemsetAsync(bad, 0, 8, r->st));
        k_validate_csr<<<g1(nv), 256, 0, r->st>>>(off, nullptr, nv, ext, bad);
        CKL();
        uint64_t h[2];
        CK(cudaMemcpyAsync(&h[0], bad, 8, cudaMemcpyDeviceToHost, r->st));
        CK(cudaMemcpyAsync(&h[1], ext + nv - 1, 8, cudaMemcpyDeviceToHost, r->st));
        r->sync();
        if (h[0]) { set_err("vertex ids not strictly increasing"); throw Fail{H2TAP_E_INVAL}; }
        r->identity = (h[1] == nv - 1);
    }
    build_fence(r, 0, nv);
    if (r->tomb) {  // every created vertex is live
        uint8_t* lv = r->get<uint8_t>(r->live[0], nv);
        if (nv) CK(cudaMemsetAsync(lv, 1, nv, r->st));
    }
    r->row_lo = 0;
    r->Vr = nv;
    if (r->sharded) {
        k_row_range<<<1, 1, 0, r->st>>>(ext, nv, r->own, r->dctr());
        CKL();
        r->read_counters();
        r->row_lo = r->hc->row_lo_new;
        r->Vr = r->hc->row_hi_new - r->hc->row_lo_new;
        CK(cudaMemsetAsync(off, 0, (r->Vr + 1) * 8, r->st));
    }
}

}  // namespace

// ======================================================================= ABI ==
extern "C" {

const char* h2tap_version(void) { return "h2tap-b200 0.1 (sm_100a)"; }
const char* h2tap_last_error(void) { return g_err.c_str(); }

const char* h2tap_status_str(h2tap_status s) {
    switch (s) {
        case H2TAP_OK: return "OK";
        case H2TAP_E_INVAL: return "E_INVAL";
        case H2TAP_E_NOMEM: return "E_NOMEM";
        case H2TAP_E_CUDA: return "E_CUDA";
        case H2TAP_E_NCCL: return "E_NCCL";
        case H2TAP_E_STALE_TS: return "E_STALE_TS";
        case H2TAP_E_SNAPSHOT_REGRESSION: return "E_SNAPSHOT_REGRESSION";
        case H2TAP_E_CAPACITY: return "E_CAPACITY";
        case H2TAP_E_POISONED: return "E_POISONED";
    }
    return "unknown";
}

constexpr uint64_t kCreateChunk = 1ull << 28;  // edges per create cycle
uint64_t create_chunk() {  // H2TAP_CREATE_CHUNK overrides it (tests of the chunked create)
    const char* e = getenv("H2TAP_CREATE_CHUNK");
    const uint64_t v = e ? strtoull(e, nullptr, 10) : 0;
    return v ? v : kCreateChunk;
}
// free the per-cycle scratch sized by the largest cycle so far (after a create)
void release_scratch(h2tap_replica* r) {
    CK(cudaStreamSynchronize(r->st));
    for (Buf* b : {&r->Wk, &r->Ws, &r->Wd, &r->Ww, &r->Wt, &r->Wq, &r->idx_p, &r->idx_n, &r->idx_e, &r->status,
                   &r->keyA, &r->keyB, &r->valA, &r->valB, &r->rs_status, &r->op_flags, &r->op_ou, &r->op_ow,
                   &r->ins_pos, &r->ins_row, &r->ins_col, &r->ins_w, &r->del_pos, &r->upd_pos, &r->upd_w,
                   &r->del_row, &r->status2, &r->part, &r->KR})
        if (b->p) r->release(*b);
}

h2tap_status h2tap_replica_create_from_edges(const h2tap_config* cfg, size_t n_vertices, const uint64_t* vertex_ids,
                                             size_t n_edges, const uint64_t* src, const uint64_t* dst, const float* w,
                                             int on_device, uint64_t create_ts, h2tap_replica** out) {
    if (!out || (n_edges && (!src || !dst))) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (n_vertices >= 0xFFFFFFFFull) { set_err("n_vertices >= 2^32-1"); return H2TAP_E_CAPACITY; }
    *out = nullptr;
    h2tap_replica* r = nullptr;
    h2tap_status s = run_guarded(nullptr, [&]() -> h2tap_status {
        r = new_replica(cfg);
        init_vertices(r, n_vertices, vertex_ids, on_device);
        r->snap = 0;
        // the edges go in as insert batches of at most kCreateChunk (in order: the last
        // duplicate still wins), which bounds the scratch of one cycle; the scratch is
        // released afterwards (later batches are far smaller than a whole graph)
        const uint64_t chunk = create_chunk();
        for (uint64_t off = 0; off < n_edges || off == 0; off += chunk) {
            const uint64_t len = std::min<uint64_t>(chunk, n_edges - off);
            BatchIn in{len, on_device, nullptr, nullptr, src ? src + off : nullptr, dst ? dst + off : nullptr,
                       w ? w + off : nullptr, nullptr, create_ts};
            h2tap_status st = apply_core(r, in, create_ts, true, nullptr);
            if (st != H2TAP_OK) return st;
            if (n_edges == 0) break;
        }
        release_scratch(r);
        r->snap = create_ts;
        r->next_seq = 0;
        return H2TAP_OK;
    });
    if (s != H2TAP_OK) { free_replica(r); return s; }
    *out = r;
    return H2TAP_OK;
}

h2tap_status h2tap_replica_create_from_csr(const h2tap_config* cfg, size_t n_vertices, const int64_t* offsets,
                                           const uint32_t* cols, const float* w, const uint64_t* ext_ids,
                                           int on_device, uint64_t create_ts, h2tap_replica** out) {
    if (!out || !offsets) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (cfg && cfg->world > 1) { set_err("create_from_csr: sharded replicas are created from edges"); return H2TAP_E_INVAL; }
    if (n_vertices >= 0xFFFFFFFFull) { set_err("n_vertices >= 2^32-1"); return H2TAP_E_CAPACITY; }
    *out = nullptr;
    h2tap_replica* r = nullptr;
    h2tap_status s = run_guarded(nullptr, [&]() -> h2tap_status {
        r = new_replica(cfg);
        init_vertices(r, n_vertices, ext_ids, on_device);
        int64_t* off = static_cast<int64_t*>(r->off[0].p);
        copy_in(r, off, offsets, n_vertices + 1, on_device);
        int64_t E = 0;
        CK(cudaMemcpyAsync(&E, off + n_vertices, 8, cudaMemcpyDeviceToHost, r->st));
        r->sync();
        if (E < 0) { set_err("negative edge count"); return H2TAP_E_INVAL; }
        uint32_t* c = r->get<uint32_t>(r->cols[0], E);
        float* ww = r->get<float>(r->w[0], E);
        if (E && !cols) { set_err("cols is NULL"); return H2TAP_E_INVAL; }
        copy_in(r, c, cols, E, on_device);
        if (w) copy_in(r, ww, w, E, on_device);
        else CK(cudaMemsetAsync(ww, 0, E * 4, r->st));
        unsigned long long* bad = r->get<unsigned long long>(r->misc, 1);
        CK(cudaMemsetAsync(bad, 0, 8, r->st));
        if (n_vertices) {
            k_validate_csr<<<g1(n_vertices), 256, 0, r->st>>>(off, c, n_vertices, nullptr, bad);
            CKL();
        }
        uint64_t hb = 0;
        CK(cudaMemcpyAsync(&hb, bad, 8, cudaMemcpyDeviceToHost, r->st));
        r->sync();
        if (hb || (n_vertices == 0 && E != 0)) { set_err("malformed CSR"); return H2TAP_E_INVAL; }
        r->E = E;
        r->snap = create_ts;
        return H2TAP_OK;
    });
    if (s != H2TAP_OK) { free_replica(r); return s; }
    *out = r;
    return H2TAP_OK;
}

h2tap_status h2tap_delta_apply(h2tap_replica* r, const h2tap_batch* b, uint64_t snapshot_ts, h2tap_apply_stats* stats) {
    if (!r || !b) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (b->n && (!b->kind || !b->src || !b->ts)) { set_err("batch kind/src/ts must be non-NULL"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        if (snapshot_ts < r->snap) {
            set_err("snapshot_ts %llu < current %llu", (unsigned long long)snapshot_ts, (unsigned long long)r->snap);
            return H2TAP_E_SNAPSHOT_REGRESSION;
        }
        CK(cudaSetDevice(r->cfg.device));
        if (r->comm) {  // collective: every rank calls; the swap is agreed inside
            if (r->defer_commit) { set_err("collective replica: apply agrees and commits itself (no prepare)"); return H2TAP_E_INVAL; }
            return coll::apply(r, b, snapshot_ts, stats);
        }
        BatchIn in{b->n, b->on_device, b->seq, b->kind, b->src, b->dst, b->weight, b->ts, 0};
        h2tap_replica::Stage* used = nullptr;
        for (auto& g : r->stg)  // a batch staged by h2tap_batch_stage: its copy is ordered first
            if (b->n && b->on_device && b->kind == g.k.p) {
                CK(cudaStreamWaitEvent(r->st, g.ev, 0));
                in.pre_h2d = g.bytes;
                g.bytes = 0;
                used = &g;
            }
        if (used) in.input_done = used->done;  // recorded by the cycle after its last read of the slot
        const h2tap_status s = apply_core(r, in, snapshot_ts, false, stats);
        if (used && s != H2TAP_OK) CK(cudaEventRecord(used->done, r->st));  // a refused cycle: after all it enqueued
        return s;
    });
}

h2tap_status h2tap_batch_validate(const h2tap_replica* rc, const h2tap_batch* b) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !b) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (b->n && (!b->kind || !b->ts)) { set_err("batch kind/ts must be non-NULL"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        CK(cudaSetDevice(r->cfg.device));
        if (!b->n) return H2TAP_OK;
        const uint8_t* kind = b->kind;
        const uint64_t* ts = b->ts;
        if (!b->on_device) {  // stage host slices
            kind = r->get<uint8_t>(r->Wk, b->n);
            ts = r->get<uint64_t>(r->Wt, b->n);
            copy_in(r, const_cast<uint8_t*>(kind), b->kind, b->n, 0);
            copy_in(r, const_cast<uint64_t*>(ts), b->ts, b->n, 0);
        }
        unsigned long long* st = r->get<unsigned long long>(r->misc, 1);
        CK(cudaMemsetAsync(st, 0, 8, r->st));
        k_validate<<<(unsigned)std::min<uint64_t>(cdiv(b->n, 256), 148 * 8), 256, 0, r->st>>>(kind, ts, b->n, r->snap, st);
        CKL();
        unsigned long long h = 0;
        CK(cudaMemcpyAsync(&h, st, 8, cudaMemcpyDeviceToHost, r->st));
        r->sync();
        if (h & ST_BAD_KIND) { set_err("unknown op kind in batch"); return H2TAP_E_INVAL; }
        if (h & ST_STALE) { set_err("op with ts <= current snapshot_ts (reading A7)"); return H2TAP_E_STALE_TS; }
        return H2TAP_OK;
    });
}

namespace {
// destination counts of a device batch slice (edge ops to the owner of their source,
// node ops to every shard), read back to the host
h2tap_status route_counts(h2tap_replica* r, const h2tap_batch* b, uint64_t* counts) {
    const int P = r->cfg.world;
    const uint64_t* bounds = static_cast<const uint64_t*>(r->bounds_dev.p);
    unsigned long long* cnt = r->get<unsigned long long>(r->misc, P);
    CK(cudaMemsetAsync(cnt, 0, P * 8, r->st));
    if (b->n) {
        k_route_count<<<(unsigned)std::min<uint64_t>(cdiv(b->n, 256), 148 * 8), 256, (P + 1) * 4, r->st>>>(b->kind, b->src, b->n, bounds, P, cnt);
        CKL();
    }
    std::vector<unsigned long long> h(P);
    CK(cudaMemcpyAsync(h.data(), cnt, P * 8, cudaMemcpyDeviceToHost, r->st));
    r->sync();
    for (int d = 0; d < P; ++d) counts[d] = h[d];
    return H2TAP_OK;
}
bool route_batch_ok(h2tap_replica* r, const h2tap_batch* b, const char* who) {
    if (!r->sharded) { set_err("%s: replica is not sharded", who); return false; }
    if (b->n && (!b->on_device || !b->kind || !b->src || !b->ts)) { set_err("%s needs a device batch", who); return false; }
    return true;
}
}  // namespace

h2tap_status h2tap_route_count(const h2tap_replica* rc, const h2tap_batch* b, uint64_t* counts) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !b || !counts) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (!route_batch_ok(r, b, "h2tap_route_count")) return H2TAP_E_INVAL;
    return run_guarded(r, [&]() -> h2tap_status {
        CK(cudaSetDevice(r->cfg.device));
        return route_counts(r, b, counts);
    });
}

h2tap_status h2tap_route_pack_p2p(const h2tap_replica* rc, const h2tap_batch* b, uint64_t seq0,
                                  h2tap_route_rec* const* peer_out, const uint64_t* peer_offset) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !b || !peer_out || !peer_offset) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (!route_batch_ok(r, b, "h2tap_route_pack_p2p")) return H2TAP_E_INVAL;
    const int P = r->cfg.world;
    if (P > kMaxP2P) { set_err("h2tap_route_pack_p2p: world %d > %d", P, kMaxP2P); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        CK(cudaSetDevice(r->cfg.device));
        if (!b->n) return H2TAP_OK;
        PeerOut po{};
        for (int d = 0; d < P; ++d) {
            if (!peer_out[d]) { set_err("h2tap_route_pack_p2p: NULL receive buffer of shard %d", d); return H2TAP_E_INVAL; }
            po.out[d] = reinterpret_cast<RouteRec*>(peer_out[d]);
            po.off[d] = peer_offset[d];
        }
        const uint64_t nt = cdiv(b->n, kTile);
        uint64_t* stt = r->get<uint64_t>(r->status, (uint64_t)P * nt);
        unsigned int* ctr = r->get<unsigned int>(r->rs_ctr, 1);
        CK(cudaMemsetAsync(stt, 0, (uint64_t)P * nt * 8, r->st));
        CK(cudaMemsetAsync(ctr, 0, 4, r->st));
        k_route_pack_p2p<<<(unsigned)nt, kThreads, 0, r->st>>>(b->kind, b->src, b->dst, b->weight, b->ts, b->n, seq0,
                                                             static_cast<const uint64_t*>(r->bounds_dev.p), P, po,
                                                             stt, nt, ctr);
        CKL();
        r->sync();  // the peer stores are complete when this returns
        return H2TAP_OK;
    });
}

// CUDA IPC receive windows for the fused exchange (cudaMalloc'ed: IPC handles need it)
h2tap_status h2tap_ipc_alloc(int device, size_t bytes, void** dptr, void* handle64) {
    if (!dptr || !handle64) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (cudaSetDevice(device) != cudaSuccess) { set_err("cudaSetDevice(%d) failed", device); return H2TAP_E_CUDA; }
    if (cudaMalloc(dptr, bytes ? bytes : 64) != cudaSuccess) { set_err("cudaMalloc(%zu) failed", bytes); return H2TAP_E_NOMEM; }
    cudaIpcMemHandle_t h;
    const cudaError_t e = cudaIpcGetMemHandle(&h, *dptr);
    if (e != cudaSuccess) { cudaFree(*dptr); *dptr = nullptr; set_err("cudaIpcGetMemHandle: %s", cudaGetErrorString(e)); return H2TAP_E_CUDA; }
    static_assert(sizeof(h) == 64, "cudaIpcMemHandle_t is 64 bytes");
    std::memcpy(handle64, &h, 64);
    return H2TAP_OK;
}
h2tap_status h2tap_ipc_open(int device, const void* handle64, void** dptr) {
    if (!dptr || !handle64) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (cudaSetDevice(device) != cudaSuccess) { set_err("cudaSetDevice(%d) failed", device); return H2TAP_E_CUDA; }
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle64, 64);
    const cudaError_t e = cudaIpcOpenMemHandle(dptr, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) { *dptr = nullptr; set_err("cudaIpcOpenMemHandle: %s", cudaGetErrorString(e)); return H2TAP_E_CUDA; }
    return H2TAP_OK;
}
h2tap_status h2tap_ipc_close(void* dptr) {
    if (dptr && cudaIpcCloseMemHandle(dptr) != cudaSuccess) { set_err("cudaIpcCloseMemHandle failed"); return H2TAP_E_CUDA; }
    return H2TAP_OK;
}
h2tap_status h2tap_ipc_free(void* dptr) {
    if (dptr && cudaFree(dptr) != cudaSuccess) { set_err("cudaFree failed"); return H2TAP_E_CUDA; }
    return H2TAP_OK;
}

h2tap_status h2tap_route_pack(const h2tap_replica* rc, const h2tap_batch* b, uint64_t seq0, h2tap_route_rec* out,
                              uint64_t capacity, uint64_t* counts) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !b || !counts) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (!r->sharded) { set_err("h2tap_route_pack: replica is not sharded"); return H2TAP_E_INVAL; }
    if (b->n && (!b->on_device || !b->kind || !b->src || !b->ts)) { set_err("route_pack needs a device batch"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        CK(cudaSetDevice(r->cfg.device));
        const int P = r->cfg.world;
        const uint64_t* bounds = static_cast<const uint64_t*>(r->bounds_dev.p);
        unsigned long long* cnt = r->get<unsigned long long>(r->misc, P);
        CK(cudaMemsetAsync(cnt, 0, P * 8, r->st));
        if (b->n) {
            k_route_count<<<(unsigned)std::min<uint64_t>(cdiv(b->n, 256), 148 * 8), 256, (P + 1) * 4, r->st>>>(b->kind, b->src, b->n, bounds, P, cnt);
            CKL();
        }
        std::vector<unsigned long long> h(P);
        CK(cudaMemcpyAsync(h.data(), cnt, P * 8, cudaMemcpyDeviceToHost, r->st));
        r->sync();
        uint64_t tot = 0;
        for (int d = 0; d < P; ++d) { counts[d] = h[d]; tot += h[d]; }
        if (tot > capacity) { set_err("route_pack: %llu records needed", (unsigned long long)tot); return H2TAP_E_CAPACITY; }
        if (!b->n) return H2TAP_OK;
        const uint64_t nt = cdiv(b->n, kTile);
        uint64_t* stt = r->get<uint64_t>(r->status, nt);
        unsigned int* ctr = r->get<unsigned int>(r->rs_ctr, P);
        CK(cudaMemsetAsync(ctr, 0, P * 4, r->st));
        uint64_t base = 0;
        for (int d = 0; d < P; ++d) {
            CK(cudaMemsetAsync(stt, 0, nt * 8, r->st));
            k_route_pack<<<(unsigned)nt, kThreads, 0, r->st>>>(b->kind, b->src, b->dst, b->weight, b->ts, b->n, seq0, bounds, P, d,
                                                           reinterpret_cast<RouteRec*>(out) + base, stt, ctr + d);
            CKL();
            base += h[d];
        }
        r->sync();
        return H2TAP_OK;
    });
}

h2tap_status h2tap_batch_stage(h2tap_replica* r, const h2tap_batch* host, h2tap_batch* staged) {
    if (!r || !host || !staged) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (host->on_device) { set_err("h2tap_batch_stage takes a host batch"); return H2TAP_E_INVAL; }
    if (host->n && (!host->kind || !host->src || !host->ts)) { set_err("batch kind/src/ts must be non-NULL"); return H2TAP_E_INVAL; }
    if (host->seq) { set_err("h2tap_batch_stage: explicit seq is not staged"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        CK(cudaSetDevice(r->cfg.device));
        auto& g = r->stg[r->stg_next];
        r->stg_next ^= 1;
        const uint64_t n = host->n;
        // the slot's previous copy (a staged batch that was never applied) may still be
        // running: wait for it before get() can free and re-allocate the slot's buffers
        CK(cudaEventSynchronize(g.ev));
        const size_t caps = g.k.cap + g.s.cap + g.d.cap + g.w.cap + g.t.cap;
        uint8_t* k = r->get<uint8_t>(g.k, n);
        uint64_t* s = r->get<uint64_t>(g.s, n);
        uint64_t* d = r->get<uint64_t>(g.d, n);
        float* w = r->get<float>(g.w, n);
        uint64_t* t = r->get<uint64_t>(g.t, n);
        if (caps != g.k.cap + g.s.cap + g.d.cap + g.w.cap + g.t.cap)
            CK(cudaStreamSynchronize(r->st));  // buffers (re)allocated on the replica stream are ready
        cudaStream_t cs = r->st_copy;
        CK(cudaStreamWaitEvent(cs, g.done, 0));  // the cycle that read this slot (asynchronous apply) is done
        uint64_t bytes = 0;
        auto cp = [&](void* dst, const void* src, uint64_t nb) {
            if (!nb) return;
            if (src) { CK(cudaMemcpyAsync(dst, src, nb, cudaMemcpyHostToDevice, cs)); bytes += nb; }
            else CK(cudaMemsetAsync(dst, 0, nb, cs));
        };
        cp(k, host->kind, n);
        cp(s, host->src, n * 8);
        cp(d, host->dst, n * 8);
        cp(w, host->weight, n * 4);
        cp(t, host->ts, n * 8);
        CK(cudaEventRecord(g.ev, cs));
        g.bytes = bytes;
        *staged = h2tap_batch{};
        staged->n = n;
        staged->on_device = 1;
        staged->kind = k; staged->src = s; staged->dst = d; staged->weight = w; staged->ts = t;
        staged->seq = nullptr;
        return H2TAP_OK;
    });
}

}  // extern "C"

namespace {
// One cycle from delta records that are in device memory: the delta-store scan (§5.2) -
// validity / visibility per record, op counts, placement scan, expansion into the
// work-op SoA - then the flat pipeline.  rec / ins / w / del are device pointers; the
// payload arrays hold absolute positions [ins_base, ins_base + n_ins) etc.
h2tap_status apply_records_dev(h2tap_replica* r, const DeltaRec* rec, uint64_t nr, const uint64_t* ins,
                               const float* wts, const double* wts64, uint64_t n_ins, const uint64_t* del,
                               uint64_t n_del, uint64_t vis_ts, uint64_t ins_base, uint64_t del_base,
                               uint64_t snapshot_ts, h2tap_apply_stats* stats,
                               const std::function<void()>& overlap = {},
                               const std::function<void()>* before_readback = nullptr) {
    cudaStream_t st = r->st;
    if (nr >= 0xFFFFFFFFull) { set_err("%llu delta records in one cycle (limit 2^32 - 2)", (unsigned long long)nr); return H2TAP_E_CAPACITY; }
    uint64_t* cnt = r->get<uint64_t>(r->xcnt, nr + 1);
    uint64_t* off = r->get<uint64_t>(r->xoff, nr + 1);
    unsigned long long* tb = r->get<unsigned long long>(r->misc, 2);
    CK(cudaMemsetAsync(tb, 0, 16, st));
    if (nr) {
        k_rec_count<<<g1(nr), 256, 0, st>>>(rec, nr, n_ins, n_del, cnt, tb, vis_ts, ins_base, del_base);
        CKL();
        const uint64_t nt = cdiv(nr, kTile);
        uint64_t* stt = r->get<uint64_t>(r->status2, nt);
        unsigned int* ctr = reinterpret_cast<unsigned int*>(r->get<uint64_t>(r->tsum, 1));
        CK(cudaMemsetAsync(stt, 0, nt * 8, st));
        CK(cudaMemsetAsync(ctr, 0, 4, st));
        k_scan_exclusive_u64<<<(unsigned)nt, kThreads, 0, st>>>(cnt, off, nr, stt, ctr);
        CKL();
    }
    // the op count and flags come back through mapped host words (a one-warp kernel store: no
    // pageable copy, no copy-engine queue behind an H2D transfer)
    k_store_words<<<1, 32, 0, st>>>(tb, 2, r->hx_dev);
    CKL();
    g_d2h += 16;
    g_ht.mark("count_issued");
    // host work that overlaps the cycle (the delta store's read-ahead copies): issued behind
    // the merge launch by default.  While a host-to-device DMA runs, the short kernels of the
    // cycle start late (measured: the sort / classify / partition segments of a C3 cycle grow
    // by ~0.25 ms), so the copy is issued where one long kernel follows.  H2TAP_RA=0: behind
    // the scan kernels instead; 2: after the cycle (profiles/r2/store/README.md)
    static const int ra_mode = [] { const char* e = getenv("H2TAP_RA"); return e ? atoi(e) : 1; }();
    bool ran = false;
    const std::function<void()> late = [&] { if (!ran && overlap) { ran = true; overlap(); } };
    if (ra_mode == 0) late();
    g_ht.mark("overlap");
    r->sync();  // the expanded op count sizes the work buffers
    const unsigned long long h[2] = {r->hx[0], r->hx[1]};
    g_ht.mark("count_sync");
    if (h[1] & REC_BAD_FLAG) { set_err("delta record flag other than 0/1"); return H2TAP_E_INVAL; }
    if (h[1] & REC_BAD_SLICE) { set_err("delta record slice outside the inserts/weights/deletes arrays"); return H2TAP_E_INVAL; }
    BatchIn in{h[0], 1, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, 0};
    in.drec = rec; in.n_drec = nr; in.drec_off = off; in.dins = ins; in.dwts = wts; in.ddel = del;
    in.dwts64 = wts64; in.vis_ts = vis_ts; in.ins_base = ins_base; in.del_base = del_base;
    in.pre_h2d = g_h2d; in.pre_d2h = g_d2h; in.pre_launches = g_launches;
    if (ra_mode == 1) in.after_merge_launch = &late;
    in.before_readback = before_readback;
    const h2tap_status s = apply_core(r, in, snapshot_ts, false, stats);
    if (s == H2TAP_OK) late();  // no merge this cycle (or H2TAP_RA=2): after it
    if (s == H2TAP_OK && stats) {  // the scan pre-pass is part of ingest
        const float pre = ev_ms(r->ev[7], r->ev[0]);
        stats->ms_ingest += pre;
        stats->ms_total += pre;
    }
    return s;
}
}  // namespace

extern "C" {

h2tap_status h2tap_delta_apply_records(h2tap_replica* r, const h2tap_record_batch* b, uint64_t snapshot_ts,
                                       h2tap_apply_stats* stats) {
    if (!r || !b) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (b->n_records && !b->records) { set_err("records must be non-NULL"); return H2TAP_E_INVAL; }
    if ((b->n_inserts && (!b->inserts || (!b->weights && !b->weights64))) || (b->n_deletes && !b->deletes)) {
        set_err("inserts/weights/deletes must be non-NULL when their size is non-zero");
        return H2TAP_E_INVAL;
    }
    return run_guarded(r, [&]() -> h2tap_status {
        if (snapshot_ts < r->snap) {
            set_err("snapshot_ts %llu < current %llu", (unsigned long long)snapshot_ts, (unsigned long long)r->snap);
            return H2TAP_E_SNAPSHOT_REGRESSION;
        }
        g_ht.init();
        g_ht.mark("entry");
        CK(cudaSetDevice(r->cfg.device));
        g_launches = g_h2d = g_d2h = 0;
        if (!r->ev[7]) CK(cudaEventCreate(&r->ev[7]));
        CK(cudaEventRecord(r->ev[7], r->st));
        const uint64_t nr = b->n_records;
        const DeltaRec* rec = reinterpret_cast<const DeltaRec*>(b->records);
        const uint64_t *ins = b->inserts, *del = b->deletes;
        const float* wts = b->weights64 ? nullptr : b->weights;
        const double* w64 = b->weights64;
        if (!b->on_device) {  // the scan reads the records where they live: copy them in once
            DeltaRec* xr = r->get<DeltaRec>(r->xrec, nr);
            copy_in(r, xr, rec, nr, 0);
            rec = xr;
            uint64_t* xi = r->get<uint64_t>(r->xins, b->n_inserts);
            uint64_t* xd = r->get<uint64_t>(r->xdel, b->n_deletes);
            copy_in(r, xi, ins, b->n_inserts, 0);
            if (w64) {
                double* xw = r->get<double>(r->xwts, b->n_inserts);
                copy_in(r, xw, w64, b->n_inserts, 0);
                w64 = xw;
            } else {
                float* xw = r->get<float>(r->xwts, b->n_inserts);
                copy_in(r, xw, wts, b->n_inserts, 0);
                wts = xw;
            }
            copy_in(r, xd, del, b->n_deletes, 0);
            ins = xi; del = xd;
        }
        const h2tap_status rc = apply_records_dev(r, rec, nr, ins, wts, w64, b->n_inserts, del, b->n_deletes,
                                                  ~0ull, 0, 0, snapshot_ts, stats);
        g_ht.mark("return");
        g_ht.dump("records cycle");
        return rc;
    });
}

h2tap_status h2tap_delta_apply_routed(h2tap_replica* r, const h2tap_route_rec* recs, size_t n, uint64_t snapshot_ts,
                                      h2tap_apply_stats* stats) {
    if (!r || (n && !recs)) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        if (snapshot_ts < r->snap) {
            set_err("snapshot_ts %llu < current %llu", (unsigned long long)snapshot_ts, (unsigned long long)r->snap);
            return H2TAP_E_SNAPSHOT_REGRESSION;
        }
        CK(cudaSetDevice(r->cfg.device));
        BatchIn in{n, 1, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, 0, reinterpret_cast<const RouteRec*>(recs)};
        return apply_core(r, in, snapshot_ts, false, stats);
    });
}

h2tap_status h2tap_delta_apply_async(h2tap_replica* r, const h2tap_batch* b, uint64_t snapshot_ts,
                                     h2tap_apply_stats* completed, int* has_completed) {
    if (!r) { set_err("null replica"); return H2TAP_E_INVAL; }
    r->async_req = true;
    const h2tap_status s = h2tap_delta_apply(r, b, snapshot_ts, nullptr);
    r->async_req = false;
    if (has_completed) *has_completed = r->fin_ready ? 1 : 0;
    if (r->fin_ready && completed) *completed = r->fin_stats;
    r->fin_ready = false;
    return s;
}

h2tap_status h2tap_replica_sync(h2tap_replica* r, h2tap_apply_stats* completed, int* has_completed) {
    if (!r) { set_err("null replica"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        ensure_final(r);
        if (has_completed) *has_completed = r->fin_ready ? 1 : 0;
        if (r->fin_ready && completed) *completed = r->fin_stats;
        r->fin_ready = false;
        return H2TAP_OK;
    });
}

h2tap_status h2tap_delta_apply_prepare(h2tap_replica* r, const h2tap_batch* b, uint64_t snapshot_ts,
                                       h2tap_apply_stats* stats) {
    if (!r) { set_err("null replica"); return H2TAP_E_INVAL; }
    r->defer_commit = true;  // run the cycle with the swap deferred
    const h2tap_status s = h2tap_delta_apply(r, b, snapshot_ts, stats);
    r->defer_commit = false;
    return s;
}

h2tap_status h2tap_delta_apply_routed_prepare(h2tap_replica* r, const h2tap_route_rec* recs, size_t n,
                                              uint64_t snapshot_ts, h2tap_apply_stats* stats) {
    if (!r) { set_err("null replica"); return H2TAP_E_INVAL; }
    r->defer_commit = true;
    const h2tap_status s = h2tap_delta_apply_routed(r, recs, n, snapshot_ts, stats);
    r->defer_commit = false;
    return s;
}

h2tap_status h2tap_delta_commit(h2tap_replica* r) {
    if (!r) { set_err("null replica"); return H2TAP_E_INVAL; }
    if (r->poisoned) { set_err("replica poisoned by an earlier CUDA error"); return H2TAP_E_POISONED; }
    if (!r->prep.on) { set_err("no prepared cycle to commit"); return H2TAP_E_INVAL; }
    r->commit();
    return H2TAP_OK;
}

h2tap_status h2tap_delta_abort(h2tap_replica* r) {
    if (!r) { set_err("null replica"); return H2TAP_E_INVAL; }
    r->prep.on = false;  // the back buffers are simply overwritten by the next cycle
    return H2TAP_OK;
}

h2tap_status h2tap_pending_export(const h2tap_replica* rc, uint8_t* kind, uint64_t* src, uint64_t* dst, float* w,
                                  uint64_t* ts, uint64_t* seq, int on_device) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r) { set_err("null replica"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        ensure_final(r);
        CK(cudaSetDevice(r->cfg.device));
        const uint64_t n = r->n_pend;
        const int pc = r->pcur;
        const cudaMemcpyKind kd = on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost;
        auto cp = [&](void* dst_, const Buf& b, size_t el) {
            if (dst_ && n) CK(cudaMemcpyAsync(dst_, b.p, n * el, kd, r->st));
        };
        cp(kind, r->pk[pc], 1);
        cp(src, r->ps[pc], 8);
        cp(dst, r->pd[pc], 8);
        cp(w, r->pw[pc], 4);
        cp(ts, r->pt[pc], 8);
        cp(seq, r->pq[pc], 8);
        r->sync();
        return H2TAP_OK;
    });
}

h2tap_status h2tap_replica_info(const h2tap_replica* r, uint64_t* nv, uint64_t* ne, uint64_t* snap, uint64_t* npend,
                                uint64_t* vbase, uint64_t* ebase) {
    if (!r) { set_err("null replica"); return H2TAP_E_INVAL; }
    if (r->infl.on) {
        const h2tap_status st = run_guarded(const_cast<h2tap_replica*>(r), [&]() -> h2tap_status {
            ensure_final(r);
            return H2TAP_OK;
        });
        if (st != H2TAP_OK) return st;
    }
    if (nv) *nv = r->Vr;  // rows of this shard (= all vertices when not sharded)
    if (ne) *ne = r->E;
    if (snap) *snap = r->snap;
    if (npend) *npend = r->n_pend;
    if (vbase) *vbase = r->row_lo;
    if (ebase) *ebase = r->edge_base;  // collective mode; 0 when the caller routes (it sums the shards)
    return H2TAP_OK;
}

h2tap_status h2tap_replica_export(const h2tap_replica* rc, int64_t* offsets, uint32_t* cols, float* w,
                                  uint64_t* ext_ids, int on_device, uint64_t checksums[4]) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r) { set_err("null replica"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        ensure_final(r);
        CK(cudaSetDevice(r->cfg.device));
        cudaMemcpyKind k = on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost;
        const int c = r->cur;
        const uint64_t* ext_own = static_cast<const uint64_t*>(r->ext[r->ext_cur].p) + r->row_lo;
        if (offsets) CK(cudaMemcpyAsync(offsets, r->off[c].p, (r->Vr + 1) * 8, k, r->st));
        if (cols && r->E) CK(cudaMemcpyAsync(cols, r->cols[c].p, r->E * 4, k, r->st));
        if (w && r->E) CK(cudaMemcpyAsync(w, r->w[c].p, r->E * 4, k, r->st));
        if (ext_ids && r->Vr) CK(cudaMemcpyAsync(ext_ids, ext_own, r->Vr * 8, k, r->st));
        if (checksums) {
            unsigned long long* cs = r->get<unsigned long long>(r->misc, 4);
            CK(cudaMemsetAsync(cs, 0, 32, r->st));
            auto grid = [](uint64_t n) { return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(cdiv(n, 256), 148 * 16)); };
            k_checksum<int64_t><<<grid(r->Vr + 1), 256, 0, r->st>>>(static_cast<int64_t*>(r->off[c].p), r->Vr + 1, 1, cs);
            k_checksum<uint32_t><<<grid(r->E), 256, 0, r->st>>>(static_cast<uint32_t*>(r->cols[c].p), r->E, 2, cs + 1);
            k_checksum<float><<<grid(r->E), 256, 0, r->st>>>(static_cast<float*>(r->w[c].p), r->E, 3, cs + 2);
            k_checksum<uint64_t><<<grid(r->Vr), 256, 0, r->st>>>(ext_own, r->Vr, 4, cs + 3);
            CKL();
            CK(cudaMemcpyAsync(checksums, cs, 32, cudaMemcpyDeviceToHost, r->st));
        }
        r->sync();
        return H2TAP_OK;
    });
}

// dense id of a live vertex (V if absent): identity map, else a binary search of the
// device ID map through single-element reads (the analytics' source lookup only)
static uint64_t live_or_none(h2tap_replica* r, uint64_t k) {  // tombstone mode: a dead slot is no source
    if (!r->tomb) return k;
    uint8_t l = 0;
    CK(cudaMemcpy(&l, static_cast<const uint8_t*>(r->live[r->ext_cur].p) + k, 1, cudaMemcpyDeviceToHost));
    return l ? k : r->V;
}
static uint64_t dense_of(h2tap_replica* r, uint64_t x_ext) {
    const uint64_t V = r->V;
    if (r->identity) return x_ext < V ? live_or_none(r, x_ext) : V;
    const uint64_t* ext = static_cast<const uint64_t*>(r->ext[r->ext_cur].p);
    uint64_t lo = 0, hi = V;
    while (lo < hi) {
        uint64_t mid = (lo + hi) / 2, x;
        CK(cudaMemcpy(&x, ext + mid, 8, cudaMemcpyDeviceToHost));
        if (x < x_ext) lo = mid + 1; else hi = mid;
    }
    uint64_t x = ~0ull;
    if (lo < V) CK(cudaMemcpy(&x, ext + lo, 8, cudaMemcpyDeviceToHost));
    const uint64_t k = (lo < V && x == x_ext) ? lo : V;
    return k < V ? live_or_none(r, k) : V;
}

h2tap_status h2tap_bfs(const h2tap_replica* rc, uint64_t source_ext, int32_t* level_out, int on_device) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !level_out) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (r->sharded && !r->comm) { set_err("h2tap_bfs: caller-routed sharded replica (use the shard steps)"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        ensure_final(r);
        CK(cudaSetDevice(r->cfg.device));
        if (r->comm) return coll::bfs(r, source_ext, level_out, on_device);
        const uint64_t V = r->V;
        const uint64_t src = dense_of(r, source_ext);
        if (src >= V) { set_err("BFS source %llu is not a live vertex", (unsigned long long)source_ext); return H2TAP_E_INVAL; }
        int32_t* level = on_device ? level_out : r->get<int32_t>(r->pr_a, V);
        uint32_t* fa = r->get<uint32_t>(r->bfs_a, V);
        uint32_t* fb = r->get<uint32_t>(r->bfs_b, V);
        unsigned long long* cnt = r->get<unsigned long long>(r->misc, 1);
        k_fill_i32<<<g1(V), 256, 0, r->st>>>(level, V, -1);
        CKL();
        int32_t zero = 0;
        uint32_t s32 = (uint32_t)src;
        CK(cudaMemcpyAsync(level + src, &zero, 4, cudaMemcpyHostToDevice, r->st));
        CK(cudaMemcpyAsync(fa, &s32, 4, cudaMemcpyHostToDevice, r->st));
        uint64_t nf = 1;
        const int64_t* off = static_cast<const int64_t*>(r->off[r->cur].p);
        const uint32_t* cols = static_cast<const uint32_t*>(r->cols[r->cur].p);
        for (int32_t depth = 0; nf; ++depth) {
            CK(cudaMemsetAsync(cnt, 0, 8, r->st));
            unsigned grid = (unsigned)std::min<uint64_t>(cdiv(nf * 32, 256), 148 * 32);
            k_bfs_expand<<<grid, 256, 0, r->st>>>(off, cols, fa, nf, level, depth, fb, cnt);
            CKL();
            unsigned long long h = 0;
            CK(cudaMemcpyAsync(&h, cnt, 8, cudaMemcpyDeviceToHost, r->st));
            r->sync();
            nf = h;
            std::swap(fa, fb);
        }
        if (!on_device) CK(cudaMemcpyAsync(level_out, level, V * 4, cudaMemcpyDeviceToHost, r->st));
        r->sync();
        return H2TAP_OK;
    });
}

h2tap_status h2tap_sssp(const h2tap_replica* rc, uint64_t source_ext, double* dist_out, int on_device) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !dist_out) { set_err("null argument"); return H2TAP_E_INVAL; }
    if (r->sharded && !r->comm) { set_err("h2tap_sssp: caller-routed sharded replica (use the shard steps)"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        ensure_final(r);
        CK(cudaSetDevice(r->cfg.device));
        if (r->comm) return coll::sssp(r, source_ext, dist_out, on_device);
        const uint64_t V = r->V, E = r->E;
        const uint64_t src = dense_of(r, source_ext);
        if (src >= V) { set_err("SSSP source %llu is not a live vertex", (unsigned long long)source_ext); return H2TAP_E_INVAL; }
        const int64_t* off = static_cast<const int64_t*>(r->off[r->cur].p);
        const uint32_t* cols = static_cast<const uint32_t*>(r->cols[r->cur].p);
        const float* w = static_cast<const float*>(r->w[r->cur].p);
        unsigned long long* cnt = r->get<unsigned long long>(r->misc, 2);
        CK(cudaMemsetAsync(cnt, 0, 16, r->st));
        if (E) {
            k_sssp_check_w<<<(unsigned)std::min<uint64_t>(cdiv(E, 256 * 8), (uint64_t)r->n_sm * 8), 256, 0, r->st>>>(
                w, E, reinterpret_cast<unsigned int*>(cnt + 1));
            CKL();
        }
        double* dist = on_device ? dist_out : r->get<double>(r->pr_a, V);
        uint32_t* stamp = r->get<uint32_t>(r->pr_b, V);
        uint32_t* fa = r->get<uint32_t>(r->bfs_a, V);
        uint32_t* fb = r->get<uint32_t>(r->bfs_b, V);
        k_fill_u64<<<g1(V), 256, 0, r->st>>>(reinterpret_cast<uint64_t*>(dist), V, 0x7FF0000000000000ull);  // +inf
        CKL();
        CK(cudaMemsetAsync(stamp, 0, V * 4, r->st));
        const double zero = 0.0;
        const uint32_t s32 = (uint32_t)src;
        CK(cudaMemcpyAsync(dist + src, &zero, 8, cudaMemcpyHostToDevice, r->st));
        CK(cudaMemcpyAsync(fa, &s32, 4, cudaMemcpyHostToDevice, r->st));
        unsigned long long h[2] = {0, 0};
        CK(cudaMemcpyAsync(h, cnt, 16, cudaMemcpyDeviceToHost, r->st));
        r->sync();
        if (h[1]) { set_err("h2tap_sssp: negative or NaN edge weight"); return H2TAP_E_INVAL; }
        uint64_t nf = 1;
        for (uint32_t round = 1; nf; ++round) {
            CK(cudaMemsetAsync(cnt, 0, 8, r->st));
            const unsigned grid = (unsigned)std::min<uint64_t>(cdiv(nf * 32, 256), (uint64_t)r->n_sm * 32);
            k_sssp_relax<<<grid, 256, 0, r->st>>>(off, cols, w, fa, nf, reinterpret_cast<unsigned long long*>(dist),
                                                  stamp, round, fb, cnt);
            CKL();
            CK(cudaMemcpyAsync(h, cnt, 8, cudaMemcpyDeviceToHost, r->st));
            r->sync();
            nf = h[0];
            std::swap(fa, fb);
        }
        if (!on_device) CK(cudaMemcpyAsync(dist_out, dist, V * 8, cudaMemcpyDeviceToHost, r->st));
        r->sync();
        return H2TAP_OK;
    });
}

// ---- checks on a sharded replica: per-shard steps, combined by the
// caller's collectives (paper_conf_edbt_jibrilabs23_b200/sharded.py)
namespace {
struct ShardView {
    const int64_t* off;
    const uint32_t* cols;
    const float* w;
    uint64_t Vr, row_lo, V;
};
ShardView shard_view(h2tap_replica* r) {
    return ShardView{static_cast<const int64_t*>(r->off[r->cur].p), static_cast<const uint32_t*>(r->cols[r->cur].p),
                     static_cast<const float*>(r->w[r->cur].p), r->Vr, r->row_lo, r->V};
}
unsigned warp_grid(h2tap_replica* r, uint64_t rows) {
    return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(cdiv(rows * 32, 256), (uint64_t)r->n_sm * 32));
}
}  // namespace
}  // extern "C"

#include "collective.cuh"

extern "C" {

h2tap_status h2tap_nccl_unique_id(void* id_out, size_t cap) {
    if (!id_out || cap < sizeof(ncclUniqueId)) { set_err("h2tap_nccl_unique_id: need %zu bytes", sizeof(ncclUniqueId)); return H2TAP_E_INVAL; }
    const coll::Api* A = coll::api();
    if (!A) return H2TAP_E_INVAL;
    ncclUniqueId id;
    const ncclResult_t e = A->GetUniqueId(&id);
    if (e != ncclSuccess) { set_err("ncclGetUniqueId: %s", A->GetErrorString(e)); return H2TAP_E_CUDA; }
    std::memcpy(id_out, &id, sizeof id);
    return H2TAP_OK;
}

h2tap_status h2tap_collective_stats(const h2tap_replica* r, uint64_t* global_seq, uint64_t* route_bytes) {
    if (!r) { set_err("null replica"); return H2TAP_E_INVAL; }
    if (!r->comm) { set_err("replica has no communicator (collective mode off)"); return H2TAP_E_INVAL; }
    if (global_seq) *global_seq = r->coll_seq;
    if (route_bytes) *route_bytes = r->last_route_bytes;
    return H2TAP_OK;
}

h2tap_status h2tap_replica_lookup(const h2tap_replica* rc, uint64_t ext_id, uint64_t* dense_out) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !dense_out) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        ensure_final(r);
        CK(cudaSetDevice(r->cfg.device));
        const uint64_t k = dense_of(r, ext_id);
        if (k >= r->V) { set_err("%llu is not a live vertex", (unsigned long long)ext_id); return H2TAP_E_INVAL; }
        *dense_out = k;
        return H2TAP_OK;
    });
}

h2tap_status h2tap_shard_bfs_expand(const h2tap_replica* rc, const int32_t* level, int32_t depth, uint8_t* mark) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !level || !mark) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        CK(cudaSetDevice(r->cfg.device));
        const ShardView s = shard_view(r);
        if (s.Vr) { k_shard_bfs_expand<<<warp_grid(r, s.Vr), 256, 0, r->st>>>(s.off, s.cols, s.Vr, s.row_lo, level, depth, mark); CKL(); }
        r->sync();
        return H2TAP_OK;
    });
}

h2tap_status h2tap_shard_bfs_settle(const h2tap_replica* rc, int32_t* level, const uint8_t* mark, int32_t depth,
                                    uint64_t* n_new) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !level || !mark || !n_new) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        CK(cudaSetDevice(r->cfg.device));
        unsigned long long* c = r->get<unsigned long long>(r->misc, 1);
        CK(cudaMemsetAsync(c, 0, 8, r->st));
        if (r->V) { k_shard_bfs_settle<<<g1(r->V), 256, 0, r->st>>>(level, mark, r->V, depth, c); CKL(); }
        unsigned long long h = 0;
        CK(cudaMemcpyAsync(&h, c, 8, cudaMemcpyDeviceToHost, r->st));
        r->sync();
        *n_new = h;
        return H2TAP_OK;
    });
}

h2tap_status h2tap_shard_pr_push(const h2tap_replica* rc, const double* pr, double* acc, double* dangling) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !pr || !acc || !dangling) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        CK(cudaSetDevice(r->cfg.device));
        const ShardView s = shard_view(r);
        if (s.Vr) { k_shard_pr_push<<<warp_grid(r, s.Vr), 256, 0, r->st>>>(s.off, s.cols, s.Vr, s.row_lo, pr, acc, dangling); CKL(); }
        r->sync();
        return H2TAP_OK;
    });
}

h2tap_status h2tap_shard_pr_finish(const h2tap_replica* rc, double* acc_to_rank, const double* dangling, double damping) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !acc_to_rank || !dangling) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        CK(cudaSetDevice(r->cfg.device));
        if (r->V) { k_shard_pr_finish<<<g1(r->V), 256, 0, r->st>>>(acc_to_rank, r->V, damping, dangling); CKL(); }
        r->sync();
        return H2TAP_OK;
    });
}

h2tap_status h2tap_shard_check_weights(const h2tap_replica* rc, int* bad) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !bad) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        CK(cudaSetDevice(r->cfg.device));
        unsigned long long* c = r->get<unsigned long long>(r->misc, 1);
        CK(cudaMemsetAsync(c, 0, 8, r->st));
        const ShardView s = shard_view(r);
        const uint64_t E = r->E;
        if (E) {
            k_sssp_check_w<<<(unsigned)std::min<uint64_t>(cdiv(E, 256 * 8), (uint64_t)r->n_sm * 8), 256, 0, r->st>>>(
                s.w, E, reinterpret_cast<unsigned int*>(c));
            CKL();
        }
        unsigned int h = 0;
        CK(cudaMemcpyAsync(&h, c, 4, cudaMemcpyDeviceToHost, r->st));
        r->sync();
        *bad = h ? 1 : 0;
        return H2TAP_OK;
    });
}

h2tap_status h2tap_shard_sssp_relax(const h2tap_replica* rc, const uint8_t* frontier, const double* dist, double* nd) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !frontier || !dist || !nd) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        CK(cudaSetDevice(r->cfg.device));
        const ShardView s = shard_view(r);
        if (s.Vr) {
            k_shard_sssp_relax<<<warp_grid(r, s.Vr), 256, 0, r->st>>>(s.off, s.cols, s.w, s.Vr, s.row_lo, frontier, dist,
                                                                    reinterpret_cast<unsigned long long*>(nd));
            CKL();
        }
        r->sync();
        return H2TAP_OK;
    });
}

h2tap_status h2tap_shard_sssp_settle(const h2tap_replica* rc, double* dist, const double* nd, uint8_t* frontier,
                                     uint64_t* n_changed) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !dist || !nd || !frontier || !n_changed) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        CK(cudaSetDevice(r->cfg.device));
        unsigned long long* c = r->get<unsigned long long>(r->misc, 1);
        CK(cudaMemsetAsync(c, 0, 8, r->st));
        if (r->V) { k_shard_sssp_settle<<<g1(r->V), 256, 0, r->st>>>(dist, nd, frontier, r->V, c); CKL(); }
        unsigned long long h = 0;
        CK(cudaMemcpyAsync(&h, c, 8, cudaMemcpyDeviceToHost, r->st));
        r->sync();
        *n_changed = h;
        return H2TAP_OK;
    });
}

h2tap_status h2tap_replica_liveness(const h2tap_replica* rc, uint8_t* live_out, int on_device) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !live_out) { set_err("null argument"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        ensure_final(r);
        CK(cudaSetDevice(r->cfg.device));
        const uint64_t V = r->V;
        if (!r->tomb) {  // compacting replica: every vertex in the ID map is live
            if (V) {
                if (on_device) CK(cudaMemsetAsync(live_out, 1, V, r->st));
                else std::memset(live_out, 1, V);
            }
        } else if (V) {
            CK(cudaMemcpyAsync(live_out, r->live[r->ext_cur].p, V,
                               on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, r->st));
        }
        r->sync();
        return H2TAP_OK;
    });
}

h2tap_status h2tap_pagerank(const h2tap_replica* rc, double damping, int iterations, double* rank_out, int on_device) {
    h2tap_replica* r = const_cast<h2tap_replica*>(rc);
    if (!r || !rank_out || iterations < 0) { set_err("bad argument"); return H2TAP_E_INVAL; }
    if (r->sharded && !r->comm) { set_err("h2tap_pagerank: caller-routed sharded replica (use the shard steps)"); return H2TAP_E_INVAL; }
    return run_guarded(r, [&]() -> h2tap_status {
        ensure_final(r);
        CK(cudaSetDevice(r->cfg.device));
        if (r->comm) return coll::pagerank(r, damping, iterations, rank_out, on_device);
        const uint64_t V = r->V;
        if (V == 0) return H2TAP_OK;
        double* a = r->get<double>(r->pr_a, V);
        double* b = r->get<double>(r->pr_b, V);
        double* ds = r->get<double>(r->misc, 1);
        const int64_t* off = static_cast<const int64_t*>(r->off[r->cur].p);
        const uint32_t* cols = static_cast<const uint32_t*>(r->cols[r->cur].p);
        const uint8_t* live = r->tomb ? static_cast<const uint8_t*>(r->live[r->ext_cur].p) : nullptr;
        uint64_t nl = V;
        if (live) {  // the graph is the live vertices (reading A23)
            unsigned long long* c = reinterpret_cast<unsigned long long*>(r->get<double>(r->misc, 2)) + 1;
            CK(cudaMemsetAsync(c, 0, 8, r->st));
            k_count_u8<<<(unsigned)std::min<uint64_t>(g1(V), 148 * 8), 256, 0, r->st>>>(live, V, c);
            CKL();
            unsigned long long h = 0;
            CK(cudaMemcpyAsync(&h, c, 8, cudaMemcpyDeviceToHost, r->st));
            r->sync();
            nl = h;
            if (nl == 0) {
                CK(cudaMemsetAsync(on_device ? rank_out : a, 0, V * 8, r->st));
                if (!on_device) { CK(cudaMemcpyAsync(rank_out, a, V * 8, cudaMemcpyDeviceToHost, r->st)); }
                r->sync();
                return H2TAP_OK;
            }
        }
        k_pr_init<<<g1(V), 256, 0, r->st>>>(a, V, live, nl);
        CKL();
        unsigned gs = (unsigned)std::min<uint64_t>(g1(V), 148 * 8);
        unsigned gw = (unsigned)std::min<uint64_t>(cdiv(V * 32, 256), 148 * 32);
        for (int it = 0; it < iterations; ++it) {
            CK(cudaMemsetAsync(ds, 0, 8, r->st));
            CK(cudaMemsetAsync(b, 0, V * 8, r->st));
            k_pr_dangling<<<gs, 256, 0, r->st>>>(off, a, V, ds);
            k_pr_push<<<gw, 256, 0, r->st>>>(off, cols, a, V, b);
            k_pr_finish<<<g1(V), 256, 0, r->st>>>(b, V, damping, ds, live, nl);
            CKL();
            std::swap(a, b);
        }
        CK(cudaMemcpyAsync(rank_out, a, V * 8, on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, r->st));
        r->sync();
        return H2TAP_OK;
    });
}

void h2tap_replica_destroy(h2tap_replica* r) {
    try {
        free_replica(r);
    } catch (...) {
    }
}

}  // extern "C"

#include "dyn.cuh"  // the dynamic replica (Algorithm 1), SURVEY §8(f) NEXT-3
#include "delta_store.cuh"  // the append-only delta store (§5.1) and the cycle from it, NEXT-1
