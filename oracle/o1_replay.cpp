/*
 * o1_replay.cpp - ORACLE (test infrastructure only).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference
 * arm may load this library.  The product path (paper_conf_edbt_jibrilabs23_b200)
 * never imports, links or calls it, and shares no code with it.
 *
 * What it computes: the plain definition of update propagation into a CSR
 * replica — the sequential replay of every visible op, in commit order, onto
 * per-vertex ordered adjacency maps, followed by emitting a compact CSR with
 * sorted column indices.  Single-threaded, no blocking, no fusion.
 *
 * Passages (PAPER.md line numbers, "P:L<n>"):
 *   CSR = row offsets + column indices + edge values ........ §2.1
 *   the four topology-changing update types .................. §5.1
 *   deltas of one node combined per propagation cycle ........ §5.2
 *   visibility: only deltas of txns older than Tp; invisible
 *   ones wait for the next cycle; each delta used once ....... §5.3 P:L755-769,
 *                                                              P:L615-619
 *   merge(): deleted node -> no entries; else old row U inserts
 *   minus deletes, column indices kept sorted ................ §5.4 P:L825-826,
 *                                                              P:L879-887
 *   new CSR replaces the old one ............................. P:L888-890
 * Readings where the paper is silent:
 *   A1 simple directed graph; A2 insert of an existing edge = upsert; A3
 *   EDGE_WEIGHT = update-if-present; A4 delete of an absent edge = no-op; A5
 *   equal ts ordered by arrival seq; A6 visible iff ts <= snapshot_ts, later ops
 *   stay pending; A7 an op with ts <= current snapshot -> E_STALE_TS; A8 node
 *   delete cascades all in- and out-edges; A9 compaction: dense ID = rank of the
 *   external ID among live vertices; A12 redundant node ops are no-ops; A13 edge
 *   ops on a non-live endpoint are no-ops; A17 create from edges: last duplicate
 *   wins.
 * Pins: tests/test_oracle_*.py (brute force O2, the Fig. 2 worked example,
 * invariants, algebraic properties, textbook CSR build).
 */
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <deque>
#include <limits>
#include <queue>
#include <map>
#include <set>
#include <vector>

namespace {

enum { OK = 0, E_INVAL = -1, E_STALE_TS = -5, E_SNAPSHOT_REGRESSION = -6 };
enum { NODE_INSERT = 0, NODE_DELETE = 1, EDGE_INSERT = 2, EDGE_DELETE = 3, EDGE_WEIGHT = 4 };

struct Op {
    uint8_t kind;
    uint64_t src, dst;
    float w;
    uint64_t ts, seq;
};

struct Graph {
    uint64_t snap_ts = 0, next_seq = 0;
    std::vector<Op> pending;
    std::map<uint64_t, std::map<uint64_t, float>> adj;  // live vertex -> (dst -> weight)
    std::map<uint64_t, std::set<uint64_t>> rin;          // reverse index (makes R2 plain)
    bool tombstone = false;   // reading A23: deleted nodes keep their id and an empty row
    std::set<uint64_t> dead;  // tombstoned ids (tombstone mode only)
};

// The fold: one op applied to the current state (SURVEY.md §8(c) rules R1-R5).
void fold(Graph& g, const Op& o) {
    switch (o.kind) {
    case NODE_INSERT:  // R1: insert of a live node is a no-op (A12); revives a tombstone (A23)
        if (!g.adj.count(o.src)) { g.adj[o.src]; g.rin[o.src]; g.dead.erase(o.src); }
        break;
    case NODE_DELETE: {  // R2: remove the node and every in- and out-edge (A8)
        auto it = g.adj.find(o.src);
        if (it == g.adj.end()) break;
        for (uint64_t u : g.rin[o.src]) if (u != o.src) g.adj[u].erase(o.src);
        for (auto& kv : it->second) if (kv.first != o.src) g.rin[kv.first].erase(o.src);
        g.adj.erase(it);
        g.rin.erase(o.src);
        if (g.tombstone) g.dead.insert(o.src);  // A23: id kept, row empty
        break;
    }
    case EDGE_INSERT:  // R3: upsert when both endpoints are live (A2, A13)
        if (g.adj.count(o.src) && g.adj.count(o.dst)) {
            g.adj[o.src][o.dst] = o.w;
            g.rin[o.dst].insert(o.src);
        }
        break;
    case EDGE_DELETE: {  // R4: absent edge -> no-op (A4)
        auto it = g.adj.find(o.src);
        if (it != g.adj.end() && it->second.erase(o.dst)) g.rin[o.dst].erase(o.src);
        break;
    }
    case EDGE_WEIGHT: {  // R5: update-if-present (A3)
        auto it = g.adj.find(o.src);
        if (it != g.adj.end()) {
            auto e = it->second.find(o.dst);
            if (e != it->second.end()) e->second = o.w;
        }
        break;
    }
    }
}

}  // namespace

extern "C" {

typedef struct {
    uint64_t n_visible, n_deferred;
} o1_stats;

void* o1_new(uint64_t create_ts) {
    Graph* g = new Graph();
    g->snap_ts = create_ts;
    return g;
}

void o1_destroy(void* h) { delete static_cast<Graph*>(h); }

/* Tombstone-row mode (the paper's merge(): a deleted node keeps "an empty entry",
 * P:L879-881; reading A23).  Set before any load/apply. */
void o1_set_tombstone(void* h) { static_cast<Graph*>(h)->tombstone = true; }

/* all ids of the export (live and tombstoned) ascending, in the export's order */
static std::vector<std::pair<uint64_t, bool>> export_ids(const Graph& g) {
    std::vector<std::pair<uint64_t, bool>> v;
    auto a = g.adj.begin();
    auto d = g.dead.begin();
    while (a != g.adj.end() || d != g.dead.end()) {
        if (d == g.dead.end() || (a != g.adj.end() && a->first < *d)) { v.push_back({a->first, true}); ++a; }
        else { v.push_back({*d, false}); ++d; }
    }
    return v;
}

/* liveness of every exported vertex (1 live, 0 tombstoned) */
void o1_live(void* h, uint8_t* live) {
    size_t i = 0;
    for (auto& x : export_ids(*static_cast<Graph*>(h))) live[i++] = x.second ? 1 : 0;
}

/* Create: vertex set (strictly increasing ids, or 0..nv-1 if ids == NULL), then
 * the edges inserted in order, last duplicate wins (A17).  Edges must join
 * listed vertices.  Returns OK or E_INVAL (graph left empty). */
int o1_load_edges(void* h, size_t nv, const uint64_t* ids, size_t ne, const uint64_t* src,
                  const uint64_t* dst, const float* w) {
    Graph& g = *static_cast<Graph*>(h);
    for (size_t i = 0; i < nv; ++i) {
        uint64_t v = ids ? ids[i] : (uint64_t)i;
        if (ids && i > 0 && ids[i] <= ids[i - 1]) { g.adj.clear(); g.rin.clear(); return E_INVAL; }
        g.adj[v]; g.rin[v];
    }
    for (size_t e = 0; e < ne; ++e) {
        if (!g.adj.count(src[e]) || !g.adj.count(dst[e])) { g.adj.clear(); g.rin.clear(); return E_INVAL; }
        g.adj[src[e]][dst[e]] = w ? w[e] : 0.f;
        g.rin[dst[e]].insert(src[e]);
    }
    return OK;
}

/* Create from a CSR whose row i belongs to external id ids[i] (or i). */
int o1_load_csr(void* h, size_t nv, const int64_t* off, const uint32_t* cols, const float* w,
                const uint64_t* ids) {
    Graph& g = *static_cast<Graph*>(h);
    for (size_t i = 0; i < nv; ++i) { uint64_t v = ids ? ids[i] : i; g.adj[v]; g.rin[v]; }
    for (size_t i = 0; i < nv; ++i) {
        uint64_t u = ids ? ids[i] : i;
        for (int64_t e = off[i]; e < off[i + 1]; ++e) {
            uint64_t v = ids ? ids[cols[e]] : cols[e];
            g.adj[u][v] = w ? w[e] : 0.f;
            g.rin[v].insert(u);
        }
    }
    return OK;
}

/* One propagation cycle (SURVEY.md §8(c) apply): validate, number, split by
 * visibility, replay the visible ops in (ts, seq) order, advance the snapshot. */
int o1_apply(void* h, size_t n, const uint8_t* kind, const uint64_t* src, const uint64_t* dst,
             const float* w, const uint64_t* ts, uint64_t snapshot_ts, o1_stats* st) {
    Graph& g = *static_cast<Graph*>(h);
    if (snapshot_ts < g.snap_ts) return E_SNAPSHOT_REGRESSION;
    for (size_t i = 0; i < n; ++i) if (kind[i] > EDGE_WEIGHT) return E_INVAL;
    for (size_t i = 0; i < n; ++i) if (ts[i] <= g.snap_ts) return E_STALE_TS;
    std::vector<Op> all = g.pending;  // earlier pending ops carry earlier seq numbers
    for (size_t i = 0; i < n; ++i)
        all.push_back(Op{kind[i], src[i], dst[i], w ? w[i] : 0.f, ts[i], g.next_seq + i});
    g.next_seq += n;
    std::vector<Op> vis;
    g.pending.clear();
    for (const Op& o : all) (o.ts <= snapshot_ts ? vis : g.pending).push_back(o);
    std::stable_sort(vis.begin(), vis.end(), [](const Op& a, const Op& b) {
        return a.ts != b.ts ? a.ts < b.ts : a.seq < b.seq;
    });
    std::set<uint64_t> known;  // tombstone mode: ids with a slot before this cycle
    if (g.tombstone) {
        for (auto& kv : g.adj) known.insert(kv.first);
        known.insert(g.dead.begin(), g.dead.end());
    }
    for (const Op& o : vis) fold(g, o);
    if (g.tombstone)  // A23: a node created and deleted within one cycle never gets a slot
        for (auto it = g.dead.begin(); it != g.dead.end();) it = known.count(*it) ? std::next(it) : g.dead.erase(it);
    g.snap_ts = snapshot_ts;
    if (st) { st->n_visible = vis.size(); st->n_deferred = g.pending.size(); }
    return OK;
}

void o1_info(void* h, uint64_t* nv, uint64_t* ne, uint64_t* snap, uint64_t* npend) {
    Graph& g = *static_cast<Graph*>(h);
    uint64_t m = 0;
    for (auto& kv : g.adj) m += kv.second.size();
    if (nv) *nv = g.adj.size() + g.dead.size();
    if (ne) *ne = m;
    if (snap) *snap = g.snap_ts;
    if (npend) *npend = g.pending.size();
}

/* Export: ext_ids = live ids ascending (tombstone mode: live and tombstoned ids);
 * dense id = rank; offsets = prefix sums of row lengths; cols/weights row by row
 * in ascending dst order (A9, A23). */
void o1_export(void* h, int64_t* off, uint32_t* cols, float* w, uint64_t* ids) {
    Graph& g = *static_cast<Graph*>(h);
    const std::vector<std::pair<uint64_t, bool>> all = export_ids(g);  // = keys(adj) unless tombstones
    std::map<uint64_t, uint32_t> dense;
    uint32_t r = 0;
    for (auto& x : all) dense[x.first] = r++;
    int64_t e = 0;
    size_t i = 0;
    for (auto& x : all) {
        if (ids) ids[i] = x.first;
        if (off) off[i] = e;
        if (x.second) {  // a tombstoned vertex has an empty row
            for (auto& y : g.adj.at(x.first)) {
                if (cols) cols[e] = dense[y.first];
                if (w) w[e] = y.second;
                ++e;
            }
        }
        ++i;
    }
    if (off) off[i] = e;
}

/* Pending ops (for deferral checks): kinds/src/dst/w/ts/seq in stored order. */
uint64_t o1_pending(void* h, uint8_t* kind, uint64_t* src, uint64_t* dst, float* w, uint64_t* ts,
                    uint64_t* seq) {
    Graph& g = *static_cast<Graph*>(h);
    for (size_t i = 0; i < g.pending.size() && kind; ++i) {
        const Op& o = g.pending[i];
        kind[i] = o.kind; src[i] = o.src; dst[i] = o.dst; w[i] = o.w; ts[i] = o.ts; seq[i] = o.seq;
    }
    return g.pending.size();
}

/* ---------------------------------------------------------------------------
 * Analytics used as freshness checks (LDBC Graphalytics; reading
 * A18), on an exported CSR.
 * BFS: textbook FIFO queue over out-edges; level[source] = 0, -1 unreachable.
 */
void o1_bfs(uint64_t nv, const int64_t* off, const uint32_t* cols, uint64_t source, int32_t* level) {
    for (uint64_t v = 0; v < nv; ++v) level[v] = -1;
    if (source >= nv) return;
    std::deque<uint64_t> q;
    level[source] = 0;
    q.push_back(source);
    while (!q.empty()) {
        uint64_t u = q.front();
        q.pop_front();
        for (int64_t e = off[u]; e < off[u + 1]; ++e) {
            uint32_t v = cols[e];
            if (level[v] < 0) { level[v] = level[u] + 1; q.push_back(v); }
        }
    }
}

/* PageRank (Graphalytics definition): PR_0 = 1/|V|;
 * PR_t(v) = (1-d)/|V| + d * ( sum_{u->v} PR_{t-1}(u)/outdeg(u)
 *                             + (1/|V|) * sum_{w dangling} PR_{t-1}(w) ). fp64. */
void o1_pagerank(uint64_t nv, const int64_t* off, const uint32_t* cols, double d, int iters,
                 double* pr) {
    if (nv == 0) return;
    std::vector<double> cur(nv, 1.0 / (double)nv), nxt(nv);
    for (int it = 0; it < iters; ++it) {
        double dangling = 0.0;
        for (uint64_t u = 0; u < nv; ++u) if (off[u + 1] == off[u]) dangling += cur[u];
        std::fill(nxt.begin(), nxt.end(), 0.0);
        for (uint64_t u = 0; u < nv; ++u) {
            int64_t deg = off[u + 1] - off[u];
            if (deg == 0) continue;
            double c = cur[u] / (double)deg;
            for (int64_t e = off[u]; e < off[u + 1]; ++e) nxt[cols[e]] += c;
        }
        for (uint64_t v = 0; v < nv; ++v)
            nxt[v] = (1.0 - d) / (double)nv + d * (nxt[v] + dangling / (double)nv);
        cur.swap(nxt);
    }
    std::memcpy(pr, cur.data(), nv * sizeof(double));
}

/* SSSP (Table 1's third analytic; reading A21):
 * textbook Dijkstra with a binary heap over out-edges, edge length = the f32
 * weight widened to fp64, path length = left-to-right fp64 sum along the path;
 * dist[source] = 0, unreachable = +inf.  Requires weights >= 0 and not NaN
 * (returns -1 otherwise, dist untouched). */
int o1_sssp(uint64_t nv, const int64_t* off, const uint32_t* cols, const float* w, uint64_t source,
            double* dist) {
    for (uint64_t e = 0; nv && e < (uint64_t)off[nv]; ++e)
        if (w[e] != w[e] || w[e] < 0.0f) return -1;  // NaN or negative (-0.0 is allowed)
    const double inf = std::numeric_limits<double>::infinity();
    for (uint64_t v = 0; v < nv; ++v) dist[v] = inf;
    if (source >= nv) return 0;
    std::vector<char> done(nv, 0);
    typedef std::pair<double, uint64_t> item;
    std::priority_queue<item, std::vector<item>, std::greater<item>> pq;
    dist[source] = 0.0;
    pq.push(item(0.0, source));
    while (!pq.empty()) {
        item t = pq.top();
        pq.pop();
        uint64_t u = t.second;
        if (done[u]) continue;
        done[u] = 1;
        for (int64_t e = off[u]; e < off[u + 1]; ++e) {
            uint32_t v = cols[e];
            double nd = dist[u] + (double)w[e];
            if (nd < dist[v]) { dist[v] = nd; pq.push(item(nd, v)); }
        }
    }
    return 0;
}

}  // extern "C"
