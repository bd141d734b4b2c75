/*
 * o3_alg2.cpp - ORACLE O3 (test infrastructure only).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference
 * arm may load this library.  The product path (paper_conf_edbt_jibrilabs23_b200)
 * never imports, links or calls it, and shares no code with it; it shares no
 * code with O1 either (o1_replay.cpp), against which it is pinned bit for bit.
 *
 * What it is: the paper's own propagation method on the host (SURVEY.md §2.6
 * "O3", §8(d) baseline 2) - a flat CSR updated by the delta merge of
 * Algorithm 2 and merge(), single-threaded or with
 * OpenMP over rows.  It reaches the same result as O1's sequential replay
 * (readings A1-A13, A17 of DESIGN.md §2), so it serves as the checksum
 * reference at sizes O1 cannot hold (configs[1]-[3] whole exports after every
 * batch) and as the "paper's method on today's host" CPU baseline.
 *
 * One cycle (o3_apply), in the paper's order:
 *   1. the scan (§5.2-§5.3): validate, number the ops (seq),
 *      split visible (ts <= snapshot_ts) from pending, order the visible ops
 *      by commit (ts, seq) and combine them per node into its delta
 *      ("combines such deltas into a single delta"): the node's
 *      final liveness, whether a delete removed its old edges, and per
 *      destination the net outcome (present with weight / absent).  Each op
 *      is folded at its commit point, so an edge op sees the liveness and the
 *      edge state that its predecessors left (A2-A4, A8, A12, A13).
 *   2. Algorithm 2 lines 1-5: A = the node IDs in the deltas, xid = the
 *      largest ID of the old CSR; L = updated nodes already in the old CSR,
 *      U = new nodes.  Reading A10: a new ID need not exceed xid, so U is
 *      placed by rank among the surviving IDs (= the paper's append when every
 *      new ID exceeds xid); reading A9: deleted nodes leave the ID map.
 *   3. Algorithm 2 lines 6-17 over the new rows: an untouched row is the old
 *      row copied (lines 8-10, 13-15; its column IDs renumbered and the
 *      columns of deleted nodes dropped - the cascade of A8); an updated old
 *      row is merge(old row, delta) (line 11: empty if the node
 *      was deleted, else old entries plus inserts minus deletes, columns kept
 *      sorted); a new node's row is its delta alone (line 17,
 *      reading A11: i advances).  Row degrees first, then offsets by prefix
 *      sum ("entirely dependent on the number of updates in the preceding
 *      nodes"), then the rows - the two row passes run over rows
 *      with OpenMP.
 *   4. the new CSR replaces the old one.
 * Create (o3_create_edges): reading A17 - the vertex set, then the edges with
 * the last duplicate winning; a textbook counting-sort CSR build (rows by
 * source, each row sorted by destination, keeping the last occurrence).
 * Checksums (o3_checksums): sum_i sm64(bits(a_i) ^ sm64(i ^ salt)) mod 2^64,
 * the definition in oracle/__init__.py (pinned against it in the tests).
 * Pins: tests/test_oracle_o3.py (bit-exact vs O1 on fuzz streams with every op
 * kind, equal timestamps, deferral and sparse IDs; the Fig. 2 example; the
 * LDBC-shaped and RMAT generators; 1 vs N threads; create = textbook build).
 */
#include <omp.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cstring>
#include <map>
#include <unordered_map>
#include <vector>

namespace {

enum { OK = 0, E_INVAL = -1, E_STALE_TS = -5, E_SNAPSHOT_REGRESSION = -6 };
enum { NODE_INSERT = 0, NODE_DELETE = 1, EDGE_INSERT = 2, EDGE_DELETE = 3, EDGE_WEIGHT = 4 };
constexpr uint32_t kNone = 0xFFFFFFFFu;

// O3_TRACE=1: wall time of each step on stderr (diagnostics only)
struct Tr {
    bool on = getenv("O3_TRACE") != nullptr;
    double t = omp_get_wtime();
    void operator()(const char* what) {
        if (!on) return;
        const double n = omp_get_wtime();
        fprintf(stderr, "[o3] %s %.3f s\n", what, n - t);
        t = n;
    }
};


struct Op {
    uint8_t kind;
    uint64_t src, dst;
    float w;
    uint64_t ts, seq;
};

// one node's combined delta (§5.2): liveness now, whether a delete removed its
// old edges, and per destination (external ID, ascending) the net edge state
struct Delta {
    int64_t old = -1;          // dense ID in the old CSR, -1 for a new node
    bool live = false;         // liveness at the current point of the scan
    bool had_delete = false;   // a NODE_DELETE took effect: every old edge of it is gone
    std::map<uint64_t, std::pair<bool, float>> e;  // dst -> (present, weight)
};

struct Csr {
    std::vector<uint64_t> ext;   // external ID of each dense row, strictly increasing
    std::vector<int64_t> off;    // V + 1
    std::vector<uint32_t> cols;  // dense destination IDs, ascending within a row
    std::vector<float> w;
};

constexpr int kFenceShift = 6;  // every 64th external ID in a small (cache-resident) table

struct Graph {
    uint64_t snap_ts = 0, next_seq = 0;
    std::vector<Op> pending;
    Csr g;
    bool identity = true;         // ext[i] == i for all i (dense lookup without a search)
    std::vector<uint64_t> fence;  // fence[j] = ext[64 j]
    void index() {
        const std::vector<uint64_t>& ext = g.ext;
        identity = true;
        for (uint64_t i = 0; i < ext.size() && identity; ++i) identity = ext[i] == i;
        fence.clear();
        for (uint64_t i = 0; i < ext.size(); i += 1u << kFenceShift) fence.push_back(ext[i]);
    }
};

// dense ID of external ID x in the current CSR, -1 if absent: binary search of the
// fence, then of the 64-ID block it selects
int64_t dense_of(const Graph& G, uint64_t x) {
    const std::vector<uint64_t>& ext = G.g.ext;
    if (G.identity) return x < ext.size() ? (int64_t)x : -1;
    auto f = std::upper_bound(G.fence.begin(), G.fence.end(), x);
    if (f == G.fence.begin()) return -1;
    const uint64_t b = (uint64_t)(f - G.fence.begin() - 1) << kFenceShift;
    auto lo = ext.begin() + b, hi = ext.begin() + std::min<uint64_t>(ext.size(), b + (1u << kFenceShift));
    auto it = std::lower_bound(lo, hi, x);
    return (it != hi && *it == x) ? (int64_t)(it - ext.begin()) : -1;
}

bool old_edge(const Graph& G, int64_t u, int64_t v) {
    const uint32_t* b = G.g.cols.data() + G.g.off[u];
    const uint32_t* e = G.g.cols.data() + G.g.off[u + 1];
    const uint32_t* p = std::lower_bound(b, e, (uint32_t)v);
    return p != e && *p == (uint32_t)v;
}

struct Scan {
    const Graph& G;
    std::unordered_map<uint64_t, Delta> nd;
    std::unordered_map<uint64_t, std::vector<uint64_t>> rin;  // dst -> nodes with a delta entry for it
    explicit Scan(const Graph& g) : G(g) {}

    Delta& get(uint64_t v) {
        auto it = nd.find(v);
        if (it != nd.end()) return it->second;
        Delta& d = nd[v];
        d.old = dense_of(G, v);
        d.live = d.old >= 0;
        return d;
    }
    const Delta* find(uint64_t v) const {
        auto it = nd.find(v);
        return it == nd.end() ? nullptr : &it->second;
    }
    bool live(uint64_t v) const {
        const Delta* d = find(v);
        return d ? d->live : dense_of(G, v) >= 0;
    }
    // is (u, w) an edge at the current point of the scan
    bool present(uint64_t u, uint64_t w) const {
        const Delta* du = find(u);
        if (du) {
            auto it = du->e.find(w);
            if (it != du->e.end()) return it->second.first;
            if (du->had_delete) return false;
        }
        const Delta* dw = find(w);
        if (dw && dw->had_delete) return false;
        const int64_t ou = dense_of(G, u), ow = dense_of(G, w);
        return ou >= 0 && ow >= 0 && old_edge(G, ou, ow);
    }
    void fold(const Op& o) {
        switch (o.kind) {
        case NODE_INSERT: {  // A12: insert of a live node is a no-op
            Delta& d = get(o.src);
            d.live = true;
            break;
        }
        case NODE_DELETE: {  // A8: the node and every in- and out-edge go
            Delta& d = get(o.src);
            if (!d.live) break;  // A12
            d.live = false;
            d.had_delete = true;
            d.e.clear();
            auto it = rin.find(o.src);
            if (it != rin.end()) {
                for (uint64_t u : it->second) {
                    auto du = nd.find(u);
                    if (du != nd.end()) du->second.e.erase(o.src);
                }
                rin.erase(it);
            }
            break;
        }
        case EDGE_INSERT:  // A2 upsert; A13 both endpoints live at this point
            if (live(o.src) && live(o.dst)) {
                get(o.src).e[o.dst] = {true, o.w};
                rin[o.dst].push_back(o.src);
            }
            break;
        case EDGE_DELETE:  // A4: absent -> no-op (recording "absent" is the same)
            if (live(o.src)) get(o.src).e[o.dst] = {false, 0.f};
            break;
        case EDGE_WEIGHT:  // A3: update-if-present
            if (live(o.src) && present(o.src, o.dst)) {
                get(o.src).e[o.dst] = {true, o.w};
                rin[o.dst].push_back(o.src);
            }
            break;
        }
    }
};

// Algorithm 2 over the combined deltas: old CSR + deltas -> new CSR
void alg2_merge(Graph& G, Scan& S) {
    Tr tr;
    const Csr& o = G.g;
    const uint64_t V = o.ext.size();
    // lines 1-5: A, L (old IDs with a delta), U (new IDs, ascending)
    std::vector<uint8_t> killed(V, 0);   // old node whose old edges a delete removed (cascade, A8)
    std::vector<uint8_t> dead(V, 0);     // old node not live after the cycle (A9: leaves the ID map)
    std::vector<const Delta*> dl(V, nullptr);
    std::vector<std::pair<uint64_t, const Delta*>> U;
    bool ids_change = false;
    for (auto& kv : S.nd) {
        const Delta& d = kv.second;
        if (d.old >= 0) {
            dl[d.old] = &d;
            if (d.had_delete) killed[d.old] = 1;
            if (!d.live) { dead[d.old] = 1; ids_change = true; }
        } else if (d.live) {
            U.push_back({kv.first, &d});
            ids_change = true;
        }
    }
    std::sort(U.begin(), U.end(), [](const auto& a, const auto& b) { return a.first < b.first; });
    // new ID map: surviving old IDs and U merged by rank (A9, A10); remap old dense -> new dense
    Csr n;
    std::vector<uint32_t> remap;
    std::vector<int64_t> src_old;          // per new row: old dense row or -1
    std::vector<const Delta*> src_delta;   // per new row: its delta or null
    if (ids_change) {
        remap.assign(V, kNone);
        n.ext.reserve(V + U.size());
        src_old.reserve(V + U.size());
        src_delta.reserve(V + U.size());
        uint64_t i = 0, j = 0;
        while (i < V || j < U.size()) {
            if (i < V && dead[i]) { ++i; continue; }
            if (j == U.size() || (i < V && o.ext[i] < U[j].first)) {
                remap[i] = (uint32_t)n.ext.size();
                n.ext.push_back(o.ext[i]);
                src_old.push_back((int64_t)i);
                src_delta.push_back(dl[i]);
                ++i;
            } else {
                n.ext.push_back(U[j].first);
                src_old.push_back(-1);
                src_delta.push_back(U[j].second);
                ++j;
            }
        }
    } else {
        n.ext = o.ext;
    }
    const uint64_t Vn = n.ext.size();
    tr("merge: lines 1-5 (A, L, U; new ID map)");
    auto new_dense = [&](uint64_t x) -> uint32_t {  // external ID -> dense ID in the new map
        auto it = std::lower_bound(n.ext.begin(), n.ext.end(), x);
        return (uint32_t)(it - n.ext.begin());
    };
    auto row_old = [&](uint64_t r) -> int64_t { return ids_change ? src_old[r] : (int64_t)r; };
    auto row_delta = [&](uint64_t r) -> const Delta* { return ids_change ? src_delta[r] : dl[r]; };
    // one gather per old column: kNone if a delete removed the target's old edges (cascade),
    // else the target's new dense ID
    std::vector<uint64_t> kbits((V + 63) / 64, 0);
    for (uint64_t c = 0; c < V; ++c) if (killed[c]) kbits[c >> 6] |= 1ull << (c & 63);
    std::vector<uint32_t> colmap(V);
#pragma omp parallel for schedule(static)
    for (int64_t c = 0; c < (int64_t)V; ++c) colmap[c] = killed[c] ? kNone : (ids_change ? remap[c] : (uint32_t)c);
    // lines 6-17 for one new row r: returns its length, writes it when cols != nullptr
    auto row = [&](uint64_t r, uint32_t* cols, float* w) -> int64_t {
        const int64_t u = row_old(r);
        const Delta* d = row_delta(r);
        int64_t k = 0;
        auto put = [&](uint32_t c, float x) {
            if (cols) { cols[k] = c; w[k] = x; }
            ++k;
        };
        const bool keep_old = u >= 0 && !killed[u];  // merge(): deleted node -> no old entries
        if (!d) {  // lines 8-10 / 13-15: new_csr[i] = old_csr[i]
            if (!cols) {  // length only: the killed bitmap is small enough to stay in cache
                for (int64_t e = o.off[u]; e < o.off[u + 1]; ++e)
                    k += !((kbits[o.cols[e] >> 6] >> (o.cols[e] & 63)) & 1);
                return k;
            }
            for (int64_t e = o.off[u]; e < o.off[u + 1]; ++e) {
                const uint32_t c = colmap[o.cols[e]];
                if (c != kNone) put(c, o.w[e]);
            }
            return k;
        }
        // line 11 merge(old_csr[i], delta_i) / line 17 delta_i: both ascending by ID
        int64_t e = keep_old ? o.off[u] : 0, ee = keep_old ? o.off[u + 1] : 0;
        auto it = d->e.begin();
        while (e < ee || it != d->e.end()) {
            if (e < ee && colmap[o.cols[e]] == kNone) { ++e; continue; }
            const bool take_old = it == d->e.end() || (e < ee && o.ext[o.cols[e]] < it->first);
            if (take_old) { put(colmap[o.cols[e]], o.w[e]); ++e; continue; }
            if (e < ee && o.ext[o.cols[e]] == it->first) ++e;  // the delta's outcome replaces it
            if (it->second.first) put(new_dense(it->first), it->second.second);
            ++it;
        }
        return k;
    };
    n.off.assign(Vn + 1, 0);
    tr("merge: column map");
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t r = 0; r < (int64_t)Vn; ++r) n.off[r + 1] = row(r, nullptr, nullptr);
    for (uint64_t r = 0; r < Vn; ++r) n.off[r + 1] += n.off[r];
    tr("merge: row lengths + offsets");
    n.cols.resize(n.off[Vn]);
    n.w.resize(n.off[Vn]);
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t r = 0; r < (int64_t)Vn; ++r) row(r, n.cols.data() + n.off[r], n.w.data() + n.off[r]);
    tr("merge: rows");
    G.g = std::move(n);  // the new CSR replaces the old one
    G.index();
}

inline uint64_t sm64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

template <typename F>
uint64_t checksum(uint64_t n, uint64_t salt, F bits) {
    uint64_t s = 0;
#pragma omp parallel for reduction(+ : s) schedule(static)
    for (int64_t i = 0; i < (int64_t)n; ++i) s += sm64(bits(i) ^ sm64((uint64_t)i ^ salt));
    return s;
}

}  // namespace

extern "C" {

typedef struct {
    uint64_t n_visible, n_deferred;
} o3_stats;

void* o3_new(uint64_t create_ts) {
    Graph* g = new Graph();
    g->snap_ts = create_ts;
    g->g.off.assign(1, 0);
    return g;
}

void o3_destroy(void* h) { delete static_cast<Graph*>(h); }

/* OpenMP threads for the row passes, create and checksums (0 = all host threads). */
void o3_set_threads(int n) { omp_set_num_threads(n > 0 ? n : omp_get_num_procs()); }
int o3_max_threads(void) { return omp_get_max_threads(); }

/* Create (A17): vertex set (strictly increasing, or 0..nv-1 if ids == NULL), then the
 * edges, the last duplicate (u, v) winning.  Endpoints must be in the vertex set and
 * ne < 2^32.  Returns OK or E_INVAL (graph left empty). */
int o3_create_edges(void* h, uint64_t nv, const uint64_t* ids, uint64_t ne, const uint64_t* src,
                    const uint64_t* dst, const float* w) {
    Graph& G = *static_cast<Graph*>(h);
    G.g = Csr();
    G.g.off.assign(1, 0);
    if (ne >= 0xFFFFFFFFull || nv >= 0xFFFFFFFFull) return E_INVAL;
    std::vector<uint64_t> ext(nv);
    for (uint64_t i = 0; i < nv; ++i) {
        ext[i] = ids ? ids[i] : i;
        if (i && ext[i] <= ext[i - 1]) return E_INVAL;
    }
    G.g.ext = std::move(ext);
    G.index();
    Tr tr;
    std::vector<uint32_t> s(ne), d(ne);
    int bad = 0;
#pragma omp parallel for reduction(| : bad) schedule(static)
    for (int64_t e = 0; e < (int64_t)ne; ++e) {
        const int64_t a = dense_of(G, src[e]), b = dense_of(G, dst[e]);
        if (a < 0 || b < 0) { bad |= 1; continue; }
        s[e] = (uint32_t)a;
        d[e] = (uint32_t)b;
    }
    if (bad) { G.g = Csr(); G.g.off.assign(1, 0); G.g.ext.clear(); return E_INVAL; }
    tr("create: endpoint lookup");
    // counting sort by source row: (dst << 32 | input index) per row
    // (the order inside a row does not matter yet: every row is sorted below)
    std::vector<int64_t> cnt(nv + 1, 0);
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < (int64_t)ne; ++e) __atomic_fetch_add(&cnt[s[e] + 1], 1, __ATOMIC_RELAXED);
    for (uint64_t v = 0; v < nv; ++v) cnt[v + 1] += cnt[v];
    std::vector<uint64_t> key(ne);
    {
        std::vector<int64_t> cur(cnt.begin(), cnt.end() - 1);
#pragma omp parallel for schedule(static)
        for (int64_t e = 0; e < (int64_t)ne; ++e)
            key[__atomic_fetch_add(&cur[s[e]], 1, __ATOMIC_RELAXED)] = (uint64_t)d[e] << 32 | (uint64_t)e;
    }
    std::vector<uint32_t>().swap(s);
    std::vector<uint32_t>().swap(d);
    tr("create: counting sort by row");
    // each row by (dst, index); the last index of a dst wins
    std::vector<int64_t>& off = G.g.off;
    off.assign(nv + 1, 0);
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t v = 0; v < (int64_t)nv; ++v) {
        std::sort(key.begin() + cnt[v], key.begin() + cnt[v + 1]);
        int64_t k = 0;
        for (int64_t e = cnt[v]; e < cnt[v + 1]; ++e)
            if (e + 1 == cnt[v + 1] || (key[e + 1] >> 32) != (key[e] >> 32)) ++k;
        off[v + 1] = k;
    }
    tr("create: row sorts");
    for (uint64_t v = 0; v < nv; ++v) off[v + 1] += off[v];
    G.g.cols.resize(off[nv]);
    G.g.w.resize(off[nv]);
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t v = 0; v < (int64_t)nv; ++v) {
        int64_t k = off[v];
        for (int64_t e = cnt[v]; e < cnt[v + 1]; ++e)
            if (e + 1 == cnt[v + 1] || (key[e + 1] >> 32) != (key[e] >> 32)) {
                G.g.cols[k] = (uint32_t)(key[e] >> 32);
                G.g.w[k] = w ? w[key[e] & 0xFFFFFFFFu] : 0.f;
                ++k;
            }
    }
    tr("create: rows written");
    return OK;
}

/* One propagation cycle: the scan (validate, number, split by visibility, order by
 * (ts, seq), combine per node), then Algorithm 2 into a new CSR. */
int o3_apply(void* h, uint64_t n, const uint8_t* kind, const uint64_t* src, const uint64_t* dst,
             const float* w, const uint64_t* ts, uint64_t snapshot_ts, o3_stats* st) {
    Graph& G = *static_cast<Graph*>(h);
    if (snapshot_ts < G.snap_ts) return E_SNAPSHOT_REGRESSION;
    for (uint64_t i = 0; i < n; ++i) if (kind[i] > EDGE_WEIGHT) return E_INVAL;
    for (uint64_t i = 0; i < n; ++i) if (ts[i] <= G.snap_ts) return E_STALE_TS;
    std::vector<Op> vis, pend;
    for (const Op& o : G.pending) (o.ts <= snapshot_ts ? vis : pend).push_back(o);
    for (uint64_t i = 0; i < n; ++i) {
        const Op o{kind[i], src[i], dst ? dst[i] : 0, w ? w[i] : 0.f, ts[i], G.next_seq + i};
        (o.ts <= snapshot_ts ? vis : pend).push_back(o);
    }
    G.next_seq += n;
    std::stable_sort(vis.begin(), vis.end(), [](const Op& a, const Op& b) {
        return a.ts != b.ts ? a.ts < b.ts : a.seq < b.seq;
    });
    Tr tr;
    tr("apply: split + order");
    if (!vis.empty()) {
        Scan S(G);
        S.nd.reserve(vis.size());
        for (const Op& o : vis) S.fold(o);
        tr("apply: scan (per-node deltas)");
        alg2_merge(G, S);
        tr("apply: Algorithm 2 merge");
    }
    G.pending.swap(pend);
    G.snap_ts = snapshot_ts;
    if (st) { st->n_visible = vis.size(); st->n_deferred = G.pending.size(); }
    return OK;
}

void o3_info(void* h, uint64_t* nv, uint64_t* ne, uint64_t* snap, uint64_t* npend) {
    Graph& G = *static_cast<Graph*>(h);
    if (nv) *nv = G.g.ext.size();
    if (ne) *ne = G.g.cols.size();
    if (snap) *snap = G.snap_ts;
    if (npend) *npend = G.pending.size();
}

/* Export the CSR (any pointer may be NULL). */
void o3_export(void* h, int64_t* off, uint32_t* cols, float* w, uint64_t* ids) {
    Graph& G = *static_cast<Graph*>(h);
    const Csr& c = G.g;
    if (off) std::memcpy(off, c.off.data(), c.off.size() * 8);
    if (cols && !c.cols.empty()) std::memcpy(cols, c.cols.data(), c.cols.size() * 4);
    if (w && !c.w.empty()) std::memcpy(w, c.w.data(), c.w.size() * 4);
    if (ids && !c.ext.empty()) std::memcpy(ids, c.ext.data(), c.ext.size() * 8);
}

/* Position-keyed checksums of offsets, cols, weights (bit patterns), ext IDs. */
void o3_checksums(void* h, uint64_t out[4]) {
    const Csr& c = static_cast<Graph*>(h)->g;
    out[0] = checksum(c.off.size(), 1, [&](int64_t i) { return (uint64_t)c.off[i]; });
    out[1] = checksum(c.cols.size(), 2, [&](int64_t i) { return (uint64_t)c.cols[i]; });
    out[2] = checksum(c.w.size(), 3, [&](int64_t i) {
        uint32_t b;
        std::memcpy(&b, &c.w[i], 4);
        return (uint64_t)b;
    });
    out[3] = checksum(c.ext.size(), 4, [&](int64_t i) { return c.ext[i]; });
}

}  // extern "C"
