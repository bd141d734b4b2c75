"""Pins for the oracle (CPU only): O1 is checked against things other than itself.

* O2 brute force (independent implementation) on exhaustive and random tiny cases
* the paper's Fig. 2 worked example (tests/golden/fig2.json)
* a textbook CSR build (numpy lexsort + keep-last unique) for insert-only batches
* invariants I1-I5 of a compact sorted CSR
* algebraic properties: composition, deferral, permutation of distinct-ts ops
* error codes and the strong guarantee
"""
import itertools
import json
import os

import numpy as np
import pytest

import oracle
import synth
from oracle import O1, BruteForce
from synth import Batch, NODE_INSERT, NODE_DELETE, EDGE_INSERT, EDGE_DELETE, EDGE_WEIGHT

HERE = os.path.dirname(os.path.abspath(__file__))


def same_export(a, b):
    return all(np.array_equal(np.asarray(x), np.asarray(y)) for x, y in zip(a, b))


def check_invariants(off, cols, w, ids):
    V = len(ids)
    assert len(off) == V + 1 and off[0] == 0 and off[-1] == len(cols) == len(w)  # I1
    assert np.all(np.diff(off) >= 0)                                              # I1
    assert np.all(cols < max(V, 1)) if len(cols) else True                         # I3
    if V > 1:
        assert np.all(np.diff(ids.astype(np.uint64)) > 0)                         # I4
    for r in range(V):                                                             # I2
        row = cols[off[r]:off[r + 1]].astype(np.int64)
        assert np.all(np.diff(row) > 0)


# ------------------------------------------------------------ Fig. 2 ----
def test_fig2_worked_example():
    g = json.load(open(os.path.join(HERE, "golden", "fig2.json")))
    e = np.array(g["edges"], dtype=object)
    o = O1.from_edges(len(g["vertices"]), np.array(g["vertices"], np.uint64),
                      np.array(e[:, 0], np.uint64), np.array(e[:, 1], np.uint64),
                      np.array(e[:, 2], np.float32), g["create_ts"])
    rc, st = o.apply(Batch.of(g["ops"]), g["snapshot_ts"])
    assert rc == 0 and st["n_visible"] == len(g["ops"])
    off, cols, w, ids = o.export()
    ex = g["expected"]
    assert ids.tolist() == ex["ext_ids"]
    assert off.tolist() == ex["offsets"]
    assert cols.tolist() == ex["cols"]
    assert w.tolist() == ex["weights"]


# ------------------------------------------- exhaustive vs brute force ----
def _all_ops(nv):
    ops = []
    for v in range(nv):
        ops.append((NODE_INSERT, v, 0, 0.0))
        ops.append((NODE_DELETE, v, 0, 0.0))
    for u in range(nv):
        for v in range(nv):
            ops.append((EDGE_INSERT, u, v, 7.0))
            ops.append((EDGE_DELETE, u, v, 0.0))
            ops.append((EDGE_WEIGHT, u, v, 9.0))
    return ops


INIT_LIVE = [0, 1]           # vertex 2 never existed
INIT_EDGES = [(0, 1, 1.0), (1, 1, 0.5), (1, 0, 2.0)]


def _run_both(seq, ts, snapshot):
    o = O1.from_edges(len(INIT_LIVE), np.array(INIT_LIVE, np.uint64),
                      np.array([e[0] for e in INIT_EDGES], np.uint64),
                      np.array([e[1] for e in INIT_EDGES], np.uint64),
                      np.array([e[2] for e in INIT_EDGES], np.float32))
    bf = BruteForce(INIT_LIVE, INIT_EDGES)
    b = Batch.of([(k, s, d, w, t) for (k, s, d, w), t in zip(seq, ts)])
    rc1, _ = o.apply(b, snapshot)
    rc2 = bf.apply(b.kind, b.src, b.dst, b.w, b.ts, snapshot)
    assert rc1 == rc2 == 0
    return o.export(), bf.export()


def test_exhaustive_length2_all_orders():
    ops = _all_ops(3)
    n = 0
    for a, b in itertools.product(ops, ops):
        for ts in ((1, 2), (2, 1), (1, 1)):
            x, y = _run_both([a, b], ts, 2)
            assert same_export(x, y), (a, b, ts)
            n += 1
    assert n == 3 * len(ops) ** 2


def test_exhaustive_length3():
    ops = _all_ops(3)
    for seq in itertools.product(ops, repeat=3):
        x, y = _run_both(list(seq), (1, 2, 3), 3)
        assert same_export(x, y), seq


def test_random_vs_bruteforce_multibatch():
    """Random multi-batch streams with equal ts, out-of-order arrival, deferral."""
    for case in range(400):
        nid = 3 + case % 5
        live = list(range(0, nid, 2))
        rng = np.random.default_rng(case)
        edges = [(int(u), int(v), float(rng.integers(0, 8)) / 4)
                 for u in live for v in live if rng.random() < 0.4]
        o = O1.from_edges(len(live), np.array(live, np.uint64),
                          np.array([e[0] for e in edges], np.uint64),
                          np.array([e[1] for e in edges], np.uint64),
                          np.array([e[2] for e in edges], np.float32))
        bf = BruteForce(live, edges)
        snap = 0
        for k in range(3):
            b = synth.fuzz_batch(seed=case, k=k, n=4 + case % 9, n_ids=nid, ts_lo=snap + 1,
                                 ts_span=6)
            s_new = snap + 3 + k
            rc1, st = o.apply(b, s_new)
            rc2 = bf.apply(b.kind, b.src, b.dst, b.w, b.ts, s_new)
            assert rc1 == rc2 == 0
            assert st["n_deferred"] == len(bf.pending)
            x, y = o.export(), bf.export()
            assert same_export(x, y), (case, k)
            check_invariants(*x)
            snap = s_new


# ------------------------------------------------- textbook CSR build ----
def textbook_csr(n, src, dst, w):
    """Insert-only into identity vertices 0..n-1: lexsort + keep the last duplicate."""
    idx = np.arange(len(src))
    order = np.lexsort((idx, dst, src))            # by (src, dst, arrival)
    s, d, ww = src[order], dst[order], w[order]
    last = np.ones(len(s), bool)
    last[:-1] = (s[1:] != s[:-1]) | (d[1:] != d[:-1])
    s, d, ww = s[last], d[last], ww[last]
    off = np.zeros(n + 1, np.int64)
    np.add.at(off, s.astype(np.int64) + 1, 1)
    return np.cumsum(off), d.astype(np.uint32), ww.astype(np.float32)


@pytest.mark.parametrize("scale", [6, 9])
def test_insert_only_equals_textbook_csr(scale):
    n = 1 << scale
    src, dst, w = synth.rmat_edges(scale, seed=scale, n=8 * n)
    o = O1.from_edges(n, None, np.array([], np.uint64), np.array([], np.uint64),
                      np.array([], np.float32))
    b = Batch(np.full(len(src), EDGE_INSERT, np.uint8), src, dst, w,
              np.arange(1, len(src) + 1, dtype=np.uint64))
    rc, _ = o.apply(b, len(src))
    assert rc == 0
    off, cols, ww, ids = o.export()
    toff, tcols, tw = textbook_csr(n, src, dst, w)
    assert np.array_equal(ids, np.arange(n, dtype=np.uint64))
    assert np.array_equal(off, toff) and np.array_equal(cols, tcols) and np.array_equal(ww, tw)
    # create-from-edges (A17) is the same thing
    o2 = O1.from_edges(n, None, src, dst, w)
    assert same_export(o2.export(), (off, cols, ww, ids))


def test_delete_all_and_empty_batch():
    n = 64
    src, dst, w = synth.rmat_edges(6, seed=3, n=400)
    o = O1.from_edges(n, None, src, dst, w)
    before = o.export()
    rc, _ = o.apply(Batch.empty(0), 5)                  # empty batch: identity
    assert rc == 0 and same_export(o.export(), before)
    off, cols, _, ids = before
    u = np.repeat(ids, np.diff(off))
    v = ids[cols]
    b = Batch(np.full(len(u), EDGE_DELETE, np.uint8), u, v, np.zeros(len(u), np.float32),
              np.full(len(u), 6, np.uint64))
    rc, _ = o.apply(b, 6)
    off2, cols2, _, ids2 = o.export()
    assert rc == 0 and len(cols2) == 0 and np.all(off2 == 0) and np.array_equal(ids2, ids)


# ----------------------------------------------------------- properties ----
def _rmat_oracle(scale=7, seed=1):
    n = 1 << scale
    src, dst, w = synth.rmat_edges(scale, seed=seed, n=6 * n)
    return n, (src, dst, w)


def _fresh(n, edges):
    return O1.from_edges(n, None, *edges)


def _mixed_batch(seed, k, n_ids, n, ts_lo, ts_span):
    return synth.fuzz_batch(seed, k, n, n_ids, probs=(0.05, 0.03, 0.5, 0.25, 0.17), ts_lo=ts_lo,
                            ts_span=ts_span)


def test_composition():
    n, edges = _rmat_oracle()
    for s in range(20):
        b1 = _mixed_batch(s, 0, n + 4, 300, 1, 50)
        b2 = _mixed_batch(s, 1, n + 4, 300, 51, 50)
        a = _fresh(n, edges); a.apply(b1, 50); a.apply(b2, 100)
        c = _fresh(n, edges); c.apply(b1.concat(b2), 100)
        assert same_export(a.export(), c.export())


def test_deferral():
    n, edges = _rmat_oracle()
    for s in range(20):
        b = _mixed_batch(s, 0, n + 4, 300, 1, 100)
        a = _fresh(n, edges)
        rc, st = a.apply(b, 40)
        assert rc == 0 and st["n_deferred"] == int(np.sum(b.ts > 40))
        a.apply(Batch.empty(0), 100)
        c = _fresh(n, edges); c.apply(b, 100)
        assert same_export(a.export(), c.export())
        assert a.info()["n_pending"] == 0


def test_permutation_of_distinct_ts():
    n, edges = _rmat_oracle()
    for s in range(20):
        b = _mixed_batch(s, 0, n + 4, 300, 1, 1)
        b.ts = np.arange(1, len(b) + 1, dtype=np.uint64)      # distinct timestamps
        perm = np.random.default_rng(s).permutation(len(b))
        a = _fresh(n, edges); a.apply(b, len(b))
        c = _fresh(n, edges); c.apply(b.slice(perm), len(b))
        assert same_export(a.export(), c.export())


def test_equal_ts_ties_follow_arrival():
    # same txn: insert then delete of one key -> absent; delete then insert -> present
    o = O1.from_edges(2, None, np.array([], np.uint64), np.array([], np.uint64),
                      np.array([], np.float32))
    o.apply(Batch.of([(EDGE_INSERT, 0, 1, 1.0, 5), (EDGE_DELETE, 0, 1, 0, 5)]), 5)
    assert o.info()["n_edges"] == 0
    o.apply(Batch.of([(EDGE_DELETE, 0, 1, 0, 6), (EDGE_INSERT, 0, 1, 3.0, 6)]), 6)
    assert o.export()[2].tolist() == [3.0]


# --------------------------------------------------------- error codes ----
def test_errors_leave_state_unchanged():
    n, edges = _rmat_oracle(6, 2)
    o = _fresh(n, edges)
    o.apply(_mixed_batch(1, 0, n, 50, 1, 10), 20)
    before = o.export()
    rc, _ = o.apply(_mixed_batch(1, 1, n, 5, 30, 5), 10)
    assert rc == oracle.E_SNAPSHOT_REGRESSION
    rc, _ = o.apply(Batch.of([(EDGE_INSERT, 0, 1, 1.0, 20)]), 30)     # ts <= snapshot
    assert rc == oracle.E_STALE_TS
    rc, _ = o.apply(Batch.of([(7, 0, 1, 1.0, 25)]), 30)               # unknown kind
    assert rc == oracle.E_INVAL
    assert same_export(o.export(), before) and o.info()["snapshot_ts"] == 20


# ----------------------------------------------------------- analytics ----
def test_bfs_matches_scipy():
    from scipy.sparse import csr_matrix
    from scipy.sparse.csgraph import shortest_path
    for scale in (5, 8):
        n = 1 << scale
        src, dst, w = synth.rmat_edges(scale, seed=scale + 10, n=4 * n)
        off, cols, _, _ = O1.from_edges(n, None, src, dst, w).export()
        A = csr_matrix((np.ones(len(cols)), cols.astype(np.int64), off), shape=(n, n))
        for s in (0, 1, n // 2):
            lvl = oracle.bfs(off, cols, s)
            d = shortest_path(A, unweighted=True, indices=s)
            ref = np.where(np.isinf(d), -1, d).astype(np.int32)
            assert np.array_equal(lvl, ref)


def test_pagerank_closed_forms_and_dense_power_iteration():
    # directed n-cycle: the uniform vector is the fixed point -> 1/n exactly
    n = 7
    off = np.arange(n + 1, dtype=np.int64)
    cols = ((np.arange(n) + 1) % n).astype(np.uint32)
    pr = oracle.pagerank(off, cols, 0.85, 30)
    assert np.allclose(pr, 1.0 / n, rtol=0, atol=1e-15)
    # random graph with dangling vertices: dense matrix power iteration, sum = 1
    scale = 7
    N = 1 << scale
    src, dst, w = synth.rmat_edges(scale, seed=5, n=3 * N)
    off, cols, _, _ = O1.from_edges(N, None, src, dst, w).export()
    deg = np.diff(off)
    M = np.zeros((N, N))
    for u in range(N):
        for e in range(off[u], off[u + 1]):
            M[cols[e], u] += 1.0 / deg[u]
    dang = (deg == 0).astype(float)
    x = np.full(N, 1.0 / N)
    for _ in range(20):
        x = (1 - 0.85) / N + 0.85 * (M @ x + dang @ x / N)
    pr = oracle.pagerank(off, cols, 0.85, 20)
    assert abs(pr.sum() - 1.0) < 1e-12
    assert np.max(np.abs(pr - x) / x) < 1e-12


def test_checksum_is_position_keyed():
    a = np.array([1, 2, 3], np.uint32)
    b = np.array([2, 1, 3], np.uint32)
    assert oracle.checksum(a, 2) != oracle.checksum(b, 2)
    assert oracle.checksum(a, 2) == oracle.checksum(a.copy(), 2)
    assert oracle.checksum(np.array([], np.uint32), 2) == 0


# ------------------------------------------------------------------ SSSP ----
def _bellman_ford(n, off, cols, w, s):
    """brute force: |V| rounds of relaxing every edge (pure Python, tiny graphs only)"""
    d = [float("inf")] * n
    d[s] = 0.0
    for _ in range(n):
        for u in range(n):
            for e in range(off[u], off[u + 1]):
                nd = d[u] + float(w[e])
                if nd < d[cols[e]]:
                    d[cols[e]] = nd
    return np.array(d)


def test_sssp_matches_scipy_dijkstra():
    from scipy.sparse import csr_matrix
    from scipy.sparse.csgraph import dijkstra
    for scale in (5, 9):
        n = 1 << scale
        src, dst, w = synth.rmat_edges(scale, seed=scale + 20, n=6 * n)
        off, cols, wt, _ = O1.from_edges(n, None, src, dst, w).export()
        wt = (wt + np.float32(2.0 ** -24)).astype(np.float32)  # strictly positive (scipy drops explicit zeros)
        A = csr_matrix((wt.astype(np.float64), cols.astype(np.int64), off), shape=(n, n))
        for s in (0, 3, n - 1):
            d = oracle.sssp(off, cols, wt, s)
            ref = dijkstra(A, directed=True, indices=s)
            # weights are multiples of 2^-24 below 1: every path sum is exact in fp64
            assert np.array_equal(d, ref)


def test_sssp_brute_force_closed_forms_and_errors():
    rng = np.random.default_rng(7)
    for trial in range(30):
        n = int(rng.integers(1, 9))
        m = int(rng.integers(0, 3 * n))
        es = {}
        for _ in range(m):
            es[(int(rng.integers(n)), int(rng.integers(n)))] = rng.choice([0.0, -0.0, 0.25, 0.5, 1.0, 3.0])
        keys = sorted(es)
        off = np.zeros(n + 1, np.int64)
        for (u, _) in keys:
            off[u + 1] += 1
        off = np.cumsum(off)
        cols = np.array([v for (_, v) in keys], np.uint32)
        w = np.array([es[k] for k in keys], np.float32)
        s = int(rng.integers(n))
        d = oracle.sssp(off, cols, w, s)
        assert np.array_equal(d, _bellman_ford(n, off, cols, w, s))
        assert d[s] == 0.0 and not np.signbit(d[s])
    # path 0 -> 1 -> ... -> n-1 with unit weights plus a shortcut 0 -> n-1 of weight 2.5
    n = 6
    off = np.array([0, 2, 3, 4, 5, 6, 6], np.int64)
    cols = np.array([1, 5, 2, 3, 4, 5], np.uint32)
    w = np.array([1, 2.5, 1, 1, 1, 1], np.float32)
    assert np.array_equal(oracle.sssp(off, cols, w, 0), [0, 1, 2, 3, 4, 2.5])
    assert np.array_equal(oracle.sssp(off, cols, w, 3), [np.inf, np.inf, np.inf, 0, 1, 2])
    with pytest.raises(ValueError):
        oracle.sssp(off, cols, np.array([1, -1, 1, 1, 1, 1], np.float32), 0)
    with pytest.raises(ValueError):
        oracle.sssp(off, cols, np.array([1, np.nan, 1, 1, 1, 1], np.float32), 0)


# ------------------------------------------------- delta-record batches ----
def load_fig2_records():
    g = json.load(open(os.path.join(HERE, "golden", "fig2_records.json")))
    rec = np.zeros(len(g["records"]), synth.RECORD_DTYPE)
    for i, r in enumerate(g["records"]):
        for k, v in r.items():
            rec[k][i] = v

    def arr(spec, dt):
        a = np.full(spec["size"], spec["fill"], dt)
        for k, v in spec["set"].items():
            a[int(k)] = v
        return a
    rb = synth.RecordBatch(rec, arr(g["inserts"], np.uint64), arr(g["weights"], np.float32),
                           arr(g["deletes"], np.uint64))
    return g, rb


def test_fig2_records_worked_example():
    g, rb = load_fig2_records()
    e = np.array(g["edges"], dtype=object)
    o = O1.from_edges(len(g["vertices"]), np.array(g["vertices"], np.uint64),
                      np.array(e[:, 0], np.uint64), np.array(e[:, 1], np.uint64),
                      np.array(e[:, 2], np.float32), g["create_ts"])
    ops = list(zip(*oracle.expand_records(rb.records, rb.inserts, rb.weights, rb.deletes)))
    assert len(ops) == 7                                      # the invalid record is skipped
    rc, st = o.apply(Batch.of(ops), g["snapshot_ts"])
    assert rc == 0
    off, cols, w, ids = o.export()
    ex = g["expected"]
    assert ids.tolist() == ex["ext_ids"] and off.tolist() == ex["offsets"]
    assert cols.tolist() == ex["cols"] and w.tolist() == ex["weights"]


def test_records_round_trip_and_bounds():
    for k in range(6):
        b = synth.fuzz_batch(seed=3, k=k, n=3000, n_ids=40, probs=(0.05, 0.03, 0.6, 0.32, 0.0),
                             ts_lo=1, ts_span=300)
        b = b.slice(np.lexsort((b.src, b.ts)))                # transactions grouped by node
        rb = synth.records_from_ops(b)
        assert len(rb) < len(b)                               # some ops share a record
        kind, src, dst, w, ts = oracle.expand_records(rb.records, rb.inserts, rb.weights, rb.deletes)
        assert np.array_equal(np.array(kind, np.uint8), b.kind) and np.array_equal(np.array(ts, np.uint64), b.ts)
        assert np.array_equal(np.array(src, np.uint64), b.src)
        e = (b.kind == EDGE_INSERT) | (b.kind == EDGE_DELETE)
        assert np.array_equal(np.array(dst, np.uint64)[e], b.dst[e])
        ins = b.kind == EDGE_INSERT
        assert np.array_equal(np.array(w, np.float32)[ins], b.w[ins])
    g, rb = load_fig2_records()
    rb.records["del_cnt"][3] = 4                              # slice past the end of deletes
    with pytest.raises(ValueError):
        oracle.expand_records(rb.records, rb.inserts, rb.weights, rb.deletes)


# ------------------------------------------------------- tombstone rows ----
def compact_view(off, cols, w, ids, live):
    """drop tombstoned vertices and renumber: what compaction would keep"""
    keep = np.flatnonzero(live)
    newid = np.full(len(ids), -1, np.int64)
    newid[keep] = np.arange(len(keep))
    deg = np.diff(off)[keep]
    rows = [np.arange(off[k], off[k + 1]) for k in keep]
    e = np.concatenate(rows) if rows else np.zeros(0, np.int64)
    assert np.all(newid[cols[e]] >= 0)                      # no edge touches a tombstone
    return (np.concatenate([[0], np.cumsum(deg)]).astype(np.int64), newid[cols[e]].astype(np.uint32),
            w[e], ids[keep])


def test_tombstone_fig2_hand_derived():
    g = json.load(open(os.path.join(HERE, "golden", "fig2.json")))
    e = np.array(g["edges"], dtype=object)
    o = O1.from_edges(len(g["vertices"]), np.array(g["vertices"], np.uint64),
                      np.array(e[:, 0], np.uint64), np.array(e[:, 1], np.uint64),
                      np.array(e[:, 2], np.float32), g["create_ts"], tombstone=True)
    assert o.apply(Batch.of(g["ops"]), g["snapshot_ts"])[0] == 0
    off, cols, w, ids = o.export()
    # node 4 keeps dense id 3 with an empty entry; 5 is appended after it
    assert ids.tolist() == [1, 2, 3, 4, 5] and o.live().tolist() == [1, 1, 1, 0, 1]
    assert off.tolist() == [0, 0, 1, 2, 2, 3]
    assert cols.tolist() == [2, 4, 0] and w.tolist() == [0.25, 5.0, 2.0]


def test_tombstone_equals_compaction_of_the_live_part():
    for k in range(40):
        n = 12
        ids = np.arange(n, dtype=np.uint64) * 3
        rng = np.random.default_rng(k)
        src, dst = ids[rng.integers(0, n, 30)], ids[rng.integers(0, n, 30)]
        w = rng.random(30).astype(np.float32)
        a = O1.from_edges(n, ids, src, dst, w)
        t = O1.from_edges(n, ids, src, dst, w, tombstone=True)
        ts = 0
        seen = set(ids.tolist())
        for j in range(4):
            b = synth.fuzz_batch(seed=k, k=j, n=60, n_ids=3 * n + 3, probs=(0.12, 0.1, 0.4, 0.25, 0.13),
                                 ts_lo=ts + 1, ts_span=50)
            snap = ts + 40
            assert a.apply(b, snap)[0] == 0 and t.apply(b, snap)[0] == 0
            ts = snap + 10
            live = t.live()
            assert same_export(compact_view(*t.export(), live), a.export())
            seen |= set(a.export()[3].tolist())
            assert set(t.export()[3].tolist()) == seen      # an id, once known, keeps its slot
            if not live.all():   # tombstones keep their rows' slot, empty
                off = t.export()[0]
                assert np.all(np.diff(off)[live == 0] == 0)


def test_from_csr_round_trip_and_continuation():
    """O1.from_csr (the checkpoint/restore direction of create): loading an
    exported CSR reproduces it exactly, and the restored replica continues exactly like the
    original under further batches; a CSR over sparse external IDs keeps them."""
    for seed in range(6):
        rng = np.random.default_rng(seed)
        ids = np.unique(rng.integers(0, 500, 60).astype(np.uint64))
        src, dst = ids[rng.integers(0, len(ids), 300)], ids[rng.integers(0, len(ids), 300)]
        w = rng.random(300).astype(np.float32)
        a = O1.from_edges(len(ids), ids, src, dst, w, 4)
        off, cols, ww, got = a.export()
        b = O1.from_csr(off, cols, ww, got, 4)
        assert same_export(b.export(), (off, cols, ww, got))
        for k in range(3):
            bt = synth.fuzz_batch(seed=seed, k=k, n=80, n_ids=600, ts_lo=5 + 10 * k, ts_span=10)
            assert a.apply(bt, 14 + 10 * k)[0] == b.apply(bt, 14 + 10 * k)[0] == 0
            assert same_export(a.export(), b.export())
    # identity ids: ext_ids = None means row i is vertex i
    c = O1.from_csr(np.array([0, 2, 2, 3], np.int64), np.array([1, 2, 0], np.uint32), np.ones(3, np.float32))
    assert c.export()[3].tolist() == [0, 1, 2] and c.export()[1].tolist() == [1, 2, 0]


def test_pending_is_the_invisible_ops_in_arrival_order():
    """O1.pending: the ops not yet visible (ts > snapshot_ts, reading A6), in
    arrival order, each with its arrival number seq (reading A5); an op leaves the pending
    set in the cycle whose snapshot reaches its ts (each delta is used once)."""
    o = O1.from_edges(4, None, np.array([0], np.uint64), np.array([1], np.uint64), np.ones(1, np.float32))
    b1 = Batch.of([(EDGE_INSERT, 1, 2, 1.0, 5), (EDGE_INSERT, 2, 3, 2.0, 9), (EDGE_DELETE, 0, 1, 0.0, 3),
                   (EDGE_WEIGHT, 1, 2, 4.0, 12)])
    assert o.apply(b1, 6)[0] == 0
    k, s, d, w, t, q = o.pending()
    assert t.tolist() == [9, 12] and q.tolist() == [1, 3] and k.tolist() == [EDGE_INSERT, EDGE_WEIGHT]
    assert s.tolist() == [2, 1] and d.tolist() == [3, 2] and w.tolist() == [2.0, 4.0]
    b2 = Batch.of([(NODE_INSERT, 7, 0, 0.0, 11), (EDGE_INSERT, 7, 0, 1.0, 20)])
    assert o.apply(b2, 11)[0] == 0
    k, s, d, w, t, q = o.pending()
    assert t.tolist() == [12, 20] and q.tolist() == [3, 5]   # 9 and 11 became visible
    assert o.apply(Batch.of([]), 30)[0] == 0 and len(o.pending()[0]) == 0
    off, cols, ww, ids = o.export()
    assert ids.tolist() == [0, 1, 2, 3, 7] and cols.tolist() == [2, 3, 0] and ww.tolist() == [4.0, 2.0, 1.0]


# ------------------------------------------------------- delta store model ----
def test_delta_store_model_fig2_two_cycles():
    """Fig. 2's transactions appended to the store model (§5.1): a cycle at ts 10 sees only
    transaction x (y is invisible), the next cycle at 20 sees only y (x's deltas
    were marked invalid), a third cycle sees nothing; the replica ends at the
    Fig. 2 result (tests/golden/fig2_records.json)."""
    g, rb = load_fig2_records()
    m = oracle.DeltaStoreModel()
    valid = rb.records[rb.records["valid"] == 1]
    m.append_records(valid, rb.inserts, rb.weights.astype(np.float64), rb.deletes)
    e = np.array(g["edges"], dtype=object)
    o = O1.from_edges(len(g["vertices"]), np.array(g["vertices"], np.uint64), np.array(e[:, 0], np.uint64),
                      np.array(e[:, 1], np.uint64), np.array(e[:, 2], np.float32), g["create_ts"])
    x = m.cycle(10)
    assert sorted(set(x[4])) == [10] and len(x[0]) == 3          # NODE_INSERT 5, 5->1, 3->5
    assert o.apply(Batch.of(list(zip(*x))), 10)[0] == 0
    y = m.cycle(20)
    assert sorted(set(y[4])) == [20] and len(y[0]) == 4          # 1-/->2, 1-/->4, delete 4, 3-/->4
    assert o.apply(Batch.of(list(zip(*y))), 20)[0] == 0
    assert len(m.cycle(30)[0]) == 0 and all(r["valid"] == 0 for r in m.records)
    off, cols, w, ids = o.export()
    ex = g["expected"]
    assert ids.tolist() == ex["ext_ids"] and off.tolist() == ex["offsets"]
    assert cols.tolist() == ex["cols"] and w.tolist() == ex["weights"]


def test_delta_store_model_eight_byte_weights_round_to_nearest_even():
    """8-byte weights reach the f32 replica rounded to nearest, ties to even
    (reading A15): 1 + 2^-24 is a tie between 1 and 1 + 2^-23 -> 1 (even); 1 + 3 * 2^-24 a tie
    between 1 + 2^-23 and 1 + 2^-22 -> 1 + 2^-22; 1 + 2^-24 + 2^-40 is above the tie."""
    m = oracle.DeltaStoreModel()
    ws = [1 + 2.0 ** -24, 1 + 3 * 2.0 ** -24, 1 + 2.0 ** -24 + 2.0 ** -40, 0.1]
    m.append(1, 7, inserts=[1, 2, 3, 4], weights=ws)
    k, s, d, w, t = m.cycle(1)
    assert [float(np.float32(x)) for x in w] == [1.0, 1 + 2.0 ** -22, 1 + 2.0 ** -23, float(np.float32(0.1))]
