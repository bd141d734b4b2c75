"""Tombstone-row mode (reading A23; the paper's merge() keeps an empty entry for a deleted
node) on the GPU vs the oracle in the same mode.  Bar: offsets / cols / weights
/ ID map / liveness bit-exact after every batch; BFS and SSSP bit-exact; PageRank of the
live subgraph within 1e-6 max relative error."""
import json
import os

import numpy as np
import pytest

import oracle
import synth
from oracle import O1
from synth import Batch, NODE_INSERT, NODE_DELETE, EDGE_INSERT, EDGE_DELETE

from test_gpu_parity import assert_same
from test_oracle_pins import compact_view

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module")
def h2():
    import paper_conf_edbt_jibrilabs23_b200 as h2
    return h2


def pair(h2, n, ids, src, dst, w):
    return (h2.Replica.from_edges(n, ids, src, dst, w, 0, tombstone=True),
            O1.from_edges(n, ids, src, dst, w, 0, tombstone=True))


def tstep(g, o, b, snap, ctx):
    st = g.apply(b, snap)
    rc, ost = o.apply(b, snap)
    assert rc == 0 and st["n_visible"] == ost["n_visible"], ctx
    ex = g.export()
    assert_same(ex, o.export(), ctx)
    assert np.array_equal(g.live(), o.live()), ctx
    return ex


def check_analytics(g, o, ex):
    off, cols, w, ids = ex
    live = o.live()
    for d in np.flatnonzero(live)[:: max(1, int(live.sum()) // 3)][:3]:
        assert np.array_equal(g.bfs(int(ids[d])), oracle.bfs(off, cols, int(d)))
        assert np.array_equal(g.sssp(int(ids[d])), oracle.sssp(off, cols, w, int(d)))
    coff, ccols, _, _ = compact_view(off, cols, w, ids, live)
    ref = np.zeros(len(ids))
    ref[live == 1] = oracle.pagerank(coff, ccols, 0.85, 20)   # the graph is the live vertices
    got = g.pagerank(0.85, 20)
    assert np.all(got[live == 0] == 0.0)
    m = live == 1
    assert np.max(np.abs(got[m] - ref[m]) / ref[m]) < 1e-6


def test_tombstone_fig2(h2):
    gj = json.load(open(os.path.join(HERE, "golden", "fig2.json")))
    e = np.array(gj["edges"], dtype=object)
    g = h2.Replica.from_edges(len(gj["vertices"]), np.array(gj["vertices"], np.uint64),
                              np.array(e[:, 0], np.uint64), np.array(e[:, 1], np.uint64),
                              np.array(e[:, 2], np.float32), gj["create_ts"], tombstone=True)
    g.apply(Batch.of(gj["ops"]), gj["snapshot_ts"])
    off, cols, w, ids = g.export()
    assert ids.tolist() == [1, 2, 3, 4, 5] and g.live().tolist() == [1, 1, 1, 0, 1]
    assert off.tolist() == [0, 0, 1, 2, 2, 3] and cols.tolist() == [2, 4, 0]
    with pytest.raises(h2.H2tapError):
        g.bfs(4)                                              # a tombstone is no source


def test_tombstone_fuzz_multibatch(h2):
    n = 1 << 11
    src, dst, w = synth.rmat_edges(11, 9, n=8 * n)
    ids = np.arange(n, dtype=np.uint64) * 3 + 5
    g, o = pair(h2, n, ids, ids[src], ids[dst], w)
    ts = 0
    for k in range(6):
        b = synth.fuzz_batch(seed=31, k=k, n=20000, n_ids=3 * n + 40, probs=(0.04, 0.03, 0.55, 0.25, 0.13),
                             ts_lo=ts + 1, ts_span=3000)
        hit = np.arange(len(b)) % 3 != 0                       # most ops touch existing ids
        b.src[hit] = ids[b.src[hit] % n]
        b.dst[hit] = ids[b.dst[hit] % n]
        snap = ts + 2500
        ex = tstep(g, o, b, snap, f"tombstone fuzz {k}")
        ts = snap + 500
    assert (g.live() == 0).any() and len(ex[3]) >= n
    check_analytics(g, o, ex)


def test_tombstone_identity_map_edge_only_batches_gate_dead_vertices(h2):
    n = 1 << 12
    src, dst, w = synth.rmat_edges(12, 4, n=16 * n)
    g, o = pair(h2, n, None, src, dst, w)
    dead = [3, 77, 1000, 4095]
    tstep(g, o, Batch.of([(NODE_DELETE, v, 0, 0.0, 10) for v in dead]), 10, "deletes")
    # edge-only batch (no node ops: the identity fast path) with ops touching tombstones
    b = synth.rmat_batch(12, 4, 0, 20000, len(src), p_insert=0.7, p_weight=0.1, ts_base=10)
    extra = Batch.of([(EDGE_INSERT, 3, 5, 1.0, 20), (EDGE_INSERT, 5, 77, 1.0, 20), (EDGE_DELETE, 1000, 1, 0.0, 20)])
    b = b.concat(extra)
    ex = tstep(g, o, b, int(b.ts.max()), "edge-only after tombstones")
    # revive one: empty row, then new edges
    ts = int(b.ts.max())
    r = Batch.of([(NODE_INSERT, 77, 0, 0.0, ts + 1), (EDGE_INSERT, 77, 9, 2.0, ts + 2), (EDGE_INSERT, 9, 77, 3.0, ts + 2)])
    ex = tstep(g, o, r, ts + 2, "revive")
    assert g.live()[77] == 1 and g.live()[3] == 0
    check_analytics(g, o, ex)


def test_tombstone_ldbc_shaped(h2):
    shape = synth.LdbcShape(n_person=512, n_msg=20000, e_person=40000)
    seed = synth.seed_of("c2")
    ids = synth.ldbc_vertices(shape)
    src, dst, w = synth.ldbc_edges(shape, seed)
    g, o = pair(h2, shape.n_vertices, ids, src, dst, w)
    ts = 0
    for k in range(3):
        b = synth.ldbc_batch(shape, seed, k, 5000, ts_base=ts)
        ts = int(b.ts.max())
        ex = tstep(g, o, b, ts, f"ldbc tombstone {k}")
    check_analytics(g, o, ex)
