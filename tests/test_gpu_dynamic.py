"""Parity of the dynamic replica (h2tap_dyn_*: Algorithm 1, §5.4) with
OD (oracle/od_dynamic.py, pinned in tests/test_oracle_pins_dyn.py).  Bar: bit-exact
offsets / cols / weights / ext ids / liveness and equal counters after every cycle
(integer work; the weights are copied, never computed)."""
import numpy as np
import pytest

import synth
from oracle.od_dynamic import DynamicOracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def h2():
    import paper_conf_edbt_jibrilabs23_b200 as h2
    return h2


KEYS = ("n_new", "n_upd", "n_del", "n_casc", "n_gated", "n_vertex_inserted", "n_vertex_deleted")


def same(g, o, ctx=""):
    a, b = g.export(), o.export()
    for name, x, y in zip(("offsets", "cols", "w", "ext_ids", "live"), a, b):
        assert np.array_equal(np.asarray(x), np.asarray(y)), f"{ctx}: {name} differs"


def cycle(g, o, rb, ctx=""):
    st = g.apply_records(rb)
    ost = o.apply_records(rb.records, rb.inserts, rb.weights, rb.deletes)
    for k in KEYS:
        assert st[k] == ost[k], f"{ctx}: {k} {st[k]} != {ost[k]}"
    same(g, o, ctx)
    return st


def pair(h2, ids, src, dst, w):
    ids = np.asarray(ids, np.uint64)
    src, dst, w = np.asarray(src, np.uint64), np.asarray(dst, np.uint64), np.asarray(w, np.float32)
    return h2.DynReplica.from_edges(len(ids), ids, src, dst, w), DynamicOracle(ids, src, dst, w)


def test_fig2_records(h2):
    from test_oracle_pins import load_fig2_records
    g0, rb = load_fig2_records()
    e = np.array(g0["edges"], dtype=object)
    g, o = pair(h2, g0["vertices"], e[:, 0], e[:, 1], e[:, 2])
    same(g, o, "create")
    cycle(g, o, rb, "fig2")
    off, cols, w, ids, live = g.export()
    assert ids.tolist() == [1, 2, 3, 4, 5] and live.tolist() == [1, 1, 1, 0, 1]
    assert off.tolist() == [0, 0, 1, 2, 2, 3] and cols.tolist() == [2, 4, 0]
    assert w.tolist() == [0.25, 5.0, 2.0]


@pytest.mark.parametrize("seed", range(6))
def test_small_random_cycles(h2, seed):
    rng = np.random.default_rng(100 + seed)
    n = 24
    ids = np.arange(n, dtype=np.uint64) * 3 + 1
    m = 80
    g, o = pair(h2, ids, ids[rng.integers(0, n, m)], ids[rng.integers(0, n, m)], rng.random(m))
    for cyc in range(8):
        rb = synth.dyn_record_batch(seed, cyc, int(o.ids[-1]), 40, n_new=6, max_slice=5, p_deleted=0.06)
        cycle(g, o, rb, f"seed {seed} cycle {cyc}")


def test_bfs_after_cycles(h2):
    """h2tap_dyn_bfs vs the oracle's BFS (oracle.bfs) on OD's export, after cycles with node
    deletes (dead vertices: level -1)."""
    import oracle
    rng = np.random.default_rng(3)
    n = 3000
    ids = np.arange(n, dtype=np.uint64) * 5
    m = 12000
    g, o = pair(h2, ids, ids[rng.integers(0, n, m)], ids[rng.integers(0, n, m)], rng.random(m))
    for cyc in range(3):
        xid = int(o.ids[-1])
        rb = synth.dyn_record_batch(21, cyc, xid, 800, n_new=40, max_slice=6, p_deleted=0.02)
        rb.records["node"] = np.where(rb.records["node"] <= xid, ids[(rb.records["node"] % n).astype(np.int64)],
                                      rb.records["node"])
        rb = synth.RecordBatch(rb.records, np.where(rb.inserts <= xid, ids[(rb.inserts % n).astype(np.int64)],
                                                    rb.inserts), rb.weights,
                               ids[(rb.deletes % n).astype(np.int64)])
        cycle(g, o, rb, f"bfs cycle {cyc}")
    off, cols, ww, ext, live = o.export()
    for s_dense in np.flatnonzero(live)[:5]:
        assert np.array_equal(g.bfs(int(ext[s_dense])), oracle.bfs(off, cols, int(s_dense)))
        # SSSP over the tables in place vs Dijkstra on OD's export (dead: unreachable)
        assert np.array_equal(g.sssp(int(ext[s_dense])), oracle.sssp(off, cols, ww, int(s_dense)))
    dead = np.flatnonzero(live == 0)
    assert len(dead)
    with pytest.raises(Exception):
        g.bfs(int(ext[dead[0]]))
    # PageRank over the live vertices (reading A18 on the live subgraph, D3: a dead vertex keeps
    # an empty table and rank 0) vs the oracle on the compacted live part of OD's export
    from test_oracle_pins import compact_view
    coff, ccols, _, _ = compact_view(off, cols, ww, ext, live)
    ref = np.zeros(len(live))
    ref[np.flatnonzero(live)] = oracle.pagerank(coff, ccols, 0.85, 20)
    pr = g.pagerank(0.85, 20)
    assert np.all(pr[live == 0] == 0)
    assert np.max(np.abs(pr - ref)[live == 1] / ref[live == 1]) <= 1e-6


def test_staged_host_records_pipeline(h2):
    """h2tap_dyn_stage: batch k+1 is copied on the copy stream while batch k is applied; the
    result equals OD after every cycle (pinned host records)."""
    import torch
    rng = np.random.default_rng(11)
    n = 2000
    ids = np.arange(n, dtype=np.uint64)
    m = 9000
    g, o = pair(h2, ids, ids[rng.integers(0, n, m)], ids[rng.integers(0, n, m)], rng.random(m))
    pin = lambda a: torch.from_numpy(a.view(np.uint8) if a.dtype.fields else a.view(np.int64) if a.dtype == np.uint64 else a).pin_memory()  # noqa: E731
    rbs = []
    xid = n - 1
    for cyc in range(5):
        rb = synth.dyn_record_batch(31, cyc, xid, 3000, n_new=30, max_slice=4, p_deleted=0.01)
        rbs.append(rb)
        xid += 30
    host = [synth.RecordBatch(pin(r.records), pin(r.inserts), pin(r.weights), pin(r.deletes)) for r in rbs]
    staged = g.stage(host[0])
    for k in range(5):
        nxt = g.stage(host[k + 1]) if k + 1 < 5 else None
        st = g.apply_records(staged)
        ost = o.apply_records(rbs[k].records, rbs[k].inserts, rbs[k].weights, rbs[k].deletes)
        for key in KEYS:
            assert st[key] == ost[key], f"staged cycle {k}: {key}"
        assert st["h2d_bytes"] > 0
        same(g, o, f"staged cycle {k}")
        staged = nxt


def test_multi_tile_cycles_with_rehash_and_device_inputs(h2):
    import torch
    rng = np.random.default_rng(7)
    n = 20000
    ids = np.sort(rng.choice(1 << 40, n, replace=False)).astype(np.uint64)
    m = 60000
    g, o = pair(h2, ids, ids[rng.integers(0, n, m)], ids[rng.integers(0, n, m)], rng.random(m))
    slots0 = g.info()["table_slots"]
    for cyc in range(6):
        xid = int(o.ids[-1])
        rb = synth.dyn_record_batch(11, cyc, xid, 9000, n_new=300, max_slice=12, p_deleted=0.01)
        # map the generator's dense-ish ids onto the replica's sparse id space
        idmap = lambda a: np.where(a <= xid, ids[(a % np.uint64(n)).astype(np.int64)], a)
        rb = synth.RecordBatch(rb.records.copy(), idmap(rb.inserts), rb.weights, idmap(rb.deletes))
        rb.records["node"] = idmap(rb.records["node"])
        if cyc % 2:
            dev = synth.RecordBatch(torch.from_numpy(rb.records.view(np.uint8)).cuda(),
                                    torch.from_numpy(rb.inserts.view(np.int64)).cuda(),
                                    torch.from_numpy(rb.weights).cuda(),
                                    torch.from_numpy(rb.deletes.view(np.int64)).cuda())
            st = g.apply_records(dev)
            ost = o.apply_records(rb.records, rb.inserts, rb.weights, rb.deletes)
            for k in KEYS:
                assert st[k] == ost[k], f"cycle {cyc}: {k}"
            same(g, o, f"cycle {cyc} (device inputs)")
        else:
            cycle(g, o, rb, f"cycle {cyc}")
    assert g.info()["table_slots"] > slots0          # the table grew (re-hash) and stayed exact


def test_hub_record_spans_many_warps(h2):
    n = 5000
    ids = np.arange(n, dtype=np.uint64)
    g, o = pair(h2, ids, [0, 1], [1, 2], [1.0, 2.0])
    rec = np.zeros(2, synth.RECORD_DTYPE)
    rec["node"] = [3, 3]
    rec["valid"] = 1
    rec["ins_cnt"] = [n, 40]
    rec["ins_off"] = [0, n]
    rec["del_cnt"] = [0, 100]
    ins = np.concatenate([np.arange(n), np.arange(40) * 7]).astype(np.uint64)
    w = np.arange(n + 40, dtype=np.float32)
    rb = synth.RecordBatch(rec, ins, w, np.arange(100, dtype=np.uint64) * 3)
    st = cycle(g, o, rb, "hub")
    assert st["n_new"] == n and st["n_del"] > 0


def test_errors_leave_the_replica_unchanged(h2):
    g, o = pair(h2, [1, 2, 3], [1], [2], [1.0])
    from test_oracle_pins import load_fig2_records
    _, rb = load_fig2_records()
    bad = synth.RecordBatch(rb.records.copy(), rb.inserts, rb.weights, rb.deletes)
    bad.records["deleted"][2] = 2
    rc, _ = g.apply_records(bad, raise_on_error=False)
    assert rc == -1                                   # E_INVAL
    bad = synth.RecordBatch(rb.records.copy(), rb.inserts, rb.weights, rb.deletes)
    bad.records["del_cnt"][3] = 9
    rc, _ = g.apply_records(bad, raise_on_error=False)
    assert rc != 0
    same(g, o, "after rejected cycles")
    with pytest.raises(Exception):
        h2.DynReplica.from_edges(2, np.array([2, 1], np.uint64), None, None, None)
    with pytest.raises(Exception):
        h2.DynReplica.from_edges(2, np.array([1, 2], np.uint64), np.array([1], np.uint64),
                                 np.array([7], np.uint64), np.array([1.0], np.float32))


def test_empty_graph_and_empty_cycle(h2):
    g, o = pair(h2, [], [], [], [])
    rb = synth.RecordBatch(np.zeros(0, synth.RECORD_DTYPE), np.zeros(0, np.uint64), np.zeros(0, np.float32),
                           np.zeros(0, np.uint64))
    cycle(g, o, rb, "empty")
    rec = np.zeros(3, synth.RECORD_DTYPE)
    rec["node"] = [5, 9, 5]
    rec["valid"] = 1
    rec["ins_cnt"] = [1, 1, 0]
    rec["ins_off"] = [0, 1, 0]
    rb = synth.RecordBatch(rec, np.array([9, 5], np.uint64), np.array([1.5, 2.5], np.float32),
                           np.zeros(0, np.uint64))
    cycle(g, o, rb, "first nodes into an empty replica")


def test_full_size_sampled_rows(h2):
    """bench_dyn.py's workload (configs[2]'s RMAT-24 graph, 500 K records with node deletes and
    new nodes, device-resident): ext ids and liveness compared in full, the rows of 256 sampled
    sources (+ every node-delete victim's row) against OD run on the sub-problem that decides
    them (all vertices, the sampled sources' edges, the records of those sources, every
    deletion and every new node: no other record can touch those rows)."""
    import torch
    scale = 24
    n = 1 << scale
    seed = synth.seed_of("c3")
    src, dst, w = synth.rmat_edges(scale, seed, n=16 * n)
    dev = [torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a).cuda() for a in (src, dst, w)]
    g = h2.DynReplica.from_edges(n, None, *dev)
    del dev
    rb = synth.dyn_record_batch(seed, 1000, n - 1, 500_000, n_new=64, max_slice=2, p_deleted=0.0002,
                                p_new=0.0005, p_invalid=0.0)
    st = g.apply_records(synth.RecordBatch(torch.from_numpy(rb.records.view(np.uint8)).cuda(),
                                           torch.from_numpy(rb.inserts.view(np.int64)).cuda(),
                                           torch.from_numpy(rb.weights).cuda(),
                                           torch.from_numpy(rb.deletes.view(np.int64)).cuda()))
    rng = np.random.default_rng(5)
    sample = np.unique(np.concatenate([rng.integers(0, n, 256),
                                       rb.records["node"][rb.records["deleted"] == 1][:16].astype(np.int64)]))
    sample = sample[sample < n].astype(np.uint64)
    keep_e = np.isin(src, sample)
    o = DynamicOracle(np.arange(n, dtype=np.uint64), src[keep_e], dst[keep_e], w[keep_e])
    r = rb.records
    keep_r = np.isin(r["node"], sample) | (r["deleted"] == 1) | (r["node"] > n - 1)
    o.apply_records(r[keep_r], rb.inserts, rb.weights, rb.deletes)
    off, cols, ww, ids, live = g.export()
    ooff, ocols, ow, oids, olive = o.export()
    assert np.array_equal(ids, oids) and np.array_equal(live, olive)
    assert st["n_vertex_inserted"] == len(ids) - n and int((live == 0).sum()) == st["n_vertex_deleted"]
    for s in sample.astype(np.int64):
        a, b = slice(off[s], off[s + 1]), slice(ooff[s], ooff[s + 1])
        assert np.array_equal(cols[a], ocols[b]) and np.array_equal(ww[a], ow[b]), f"row {s}"
    assert off[-1] == g.info()["n_edges"]
