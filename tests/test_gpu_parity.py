"""Parity of the CUDA path (libh2tap.so through its C ABI) with the oracle O1.

Bar: offsets, cols, weights and the ID map bit-exact after every
batch; BFS levels bit-exact; PageRank within 1e-6 max relative error.
"""
import json
import os

import numpy as np
import pytest

import oracle
import synth
from oracle import O1
from synth import Batch, NODE_INSERT, NODE_DELETE, EDGE_INSERT, EDGE_DELETE, EDGE_WEIGHT

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module")
def h2():
    import paper_conf_edbt_jibrilabs23_b200 as h2
    return h2


def assert_same(gpu, ora, ctx=""):
    names = ("offsets", "cols", "weights", "ext_ids")
    for n, a, b in zip(names, gpu, ora):
        a, b = np.asarray(a), np.asarray(b)
        assert a.shape == b.shape, f"{ctx} {n}: shape {a.shape} vs {b.shape}"
        if n == "weights":
            a, b = a.view(np.uint32), b.view(np.uint32)
        if not np.array_equal(a, b):
            bad = np.nonzero(a != b)[0]
            raise AssertionError(f"{ctx} {n}: {len(bad)} mismatches, first at {bad[:5]}: "
                                 f"{a[bad[:5]]} vs {b[bad[:5]]}")


def pair_from_edges(h2, n, ids, src, dst, w, create_ts=0):
    g = h2.Replica.from_edges(n, ids, src, dst, w, create_ts)
    o = O1.from_edges(n, ids, src, dst, w, create_ts)
    step.last_E[id(g)] = g.info()["n_edges"]
    return g, o


def step(g, o, batch, snap, ctx=""):
    st = g.apply(batch, snap)
    rc, ost = o.apply(batch, snap)
    assert rc == 0
    assert st["n_visible"] == ost["n_visible"] and st["n_deferred"] == ost["n_deferred"], ctx
    E_old = step.last_E.get(id(g))
    ex = g.export()
    assert_same(ex, o.export(), ctx)
    if E_old is not None:  # I6: E' = E + NEW - DEL - CASC
        assert len(ex[1]) == E_old + st["n_new"] - st["n_del"] - st["n_casc"], ctx
    step.last_E[id(g)] = len(ex[1])
    return st


step.last_E = {}


# ------------------------------------------------------------------ cases ----
def test_fig2_worked_example(h2):
    gj = json.load(open(os.path.join(HERE, "golden", "fig2.json")))
    e = np.array(gj["edges"], dtype=object)
    ids = np.array(gj["vertices"], np.uint64)
    g = h2.Replica.from_edges(len(ids), ids, np.array(e[:, 0], np.uint64), np.array(e[:, 1], np.uint64),
                              np.array(e[:, 2], np.float32), gj["create_ts"])
    st = g.apply(Batch.of(gj["ops"]), gj["snapshot_ts"])
    off, cols, w, ext = g.export()
    ex = gj["expected"]
    assert ext.tolist() == ex["ext_ids"] and off.tolist() == ex["offsets"]
    assert cols.tolist() == ex["cols"] and w.tolist() == ex["weights"]
    assert st["n_vertex_inserted"] == 1 and st["n_vertex_deleted"] == 1


def test_tiny_fuzz_multibatch(h2):
    """Adversarial tiny streams: equal ts, out-of-order arrival, deferral, all op kinds."""
    for case in range(150):
        nid = 3 + case % 6
        rng = np.random.default_rng(1000 + case)
        live = np.array(sorted(rng.choice(nid, size=max(1, nid // 2), replace=False)), np.uint64)
        pairs = [(u, v) for u in live for v in live if rng.random() < 0.5]
        src = np.array([p[0] for p in pairs], np.uint64)
        dst = np.array([p[1] for p in pairs], np.uint64)
        w = (rng.integers(0, 16, len(pairs)) / 4).astype(np.float32)
        g, o = pair_from_edges(h2, len(live), live, src, dst, w)
        snap = 0
        for k in range(4):
            b = synth.fuzz_batch(seed=case, k=k, n=1 + (case * 7 + k) % 23, n_ids=nid, ts_lo=snap + 1,
                                 ts_span=8)
            snap += 4
            step(g, o, b, snap, f"case {case} batch {k}")


def test_rmat_c1_config(h2):
    """BASELINE configs[0]: RMAT scale 16, 1M generated edges, one 10K 80/20 batch."""
    cfg = synth.CONFIGS["c1"]
    seed = synth.seed_of("c1")
    n = 1 << cfg["scale"]
    src, dst, w = synth.rmat_edges(cfg["scale"], seed)
    g, o = pair_from_edges(h2, n, None, src, dst, w)
    assert_same(g.export(), o.export(), "create")
    b = synth.rmat_batch(cfg["scale"], seed, 0, cfg["batch"], len(src), p_insert=0.8, ts_base=0)
    st = step(g, o, b, int(b.ts.max()), "c1 batch")
    assert st["n_new"] > 0 and st["n_del"] > 0
    # freshness checks on the new snapshot
    off, cols, _, _ = g.export()
    for s in (0, 17, 4242):
        assert np.array_equal(g.bfs(s), oracle.bfs(off, cols, s))
    pr_g, pr_o = g.pagerank(0.85, 20), oracle.pagerank(off, cols, 0.85, 20)
    assert np.max(np.abs(pr_g - pr_o) / pr_o) < 1e-6
    w_new = g.export()[2]
    for s in (0, 17, 4242):                               # SSSP: bit-exact (unique fixpoint)
        assert np.array_equal(g.sssp(s), oracle.sssp(off, cols, w_new, s))


def test_rmat_parity_variant_weights_repeats_txns(h2):
    """C1 parity variant: 10% EDGE_WEIGHT, repeated keys, 4-op transactions (equal ts)."""
    seed = synth.seed_of("c1") + 77
    scale = 14
    src, dst, w = synth.rmat_edges(scale, seed)
    g, o = pair_from_edges(h2, 1 << scale, None, src, dst, w)
    ts = 0
    for k in range(3):
        b = synth.rmat_batch(scale, seed, k, 20000, len(src), p_insert=0.6, p_weight=0.1, p_repeat=0.3,
                             ops_per_txn=4, ts_base=ts)
        snap = int(np.quantile(b.ts, 0.9))          # defer ~10%
        step(g, o, b, snap, f"variant batch {k}")
        ts = int(b.ts.max())
    step(g, o, Batch.empty(0), ts, "flush pending")
    assert g.info()["n_pending"] == 0


def test_mixed_node_ops_multi_tile(h2):
    """Node inserts/deletes (incl. re-insert, ids outside the graph), many merge tiles."""
    scale = 13
    n = 1 << scale
    src, dst, w = synth.rmat_edges(scale, 5, n=12 * n)
    ids = (np.arange(n, dtype=np.uint64) * 3 + 7)       # sparse external ids
    g, o = pair_from_edges(h2, n, ids, ids[src], ids[dst], w)
    ts = 0
    for k in range(4):
        b = synth.fuzz_batch(seed=99, k=k, n=30000, n_ids=3 * n + 20, probs=(0.03, 0.01, 0.6, 0.25, 0.11),
                             ts_lo=ts + 1, ts_span=5000)
        # map half the random ids onto existing vertices so edge ops hit the graph
        hit = np.arange(len(b)) % 2 == 0
        b.src[hit] = ids[b.src[hit] % n]
        b.dst[hit] = ids[b.dst[hit] % n]
        snap = ts + 4000
        step(g, o, b, snap, f"mixed batch {k}")
        ts = snap + 1000


def test_ldbc_shaped_small(h2):
    shape = synth.LdbcShape(n_person=512, n_msg=20000, e_person=40000)
    seed = synth.seed_of("c2")
    ids = synth.ldbc_vertices(shape)
    src, dst, w = synth.ldbc_edges(shape, seed)
    g, o = pair_from_edges(h2, shape.n_vertices, ids, src, dst, w)
    ts = 0
    for k in range(3):
        b = synth.ldbc_batch(shape, seed, k, 5000, lodeg=(k == 1), ts_base=ts)
        ts = int(b.ts.max())
        st = step(g, o, b, ts, f"ldbc batch {k}")
        assert st["n_vertex_inserted"] > 0
        # analytics on the compacted replica, sources named by external id
        off, cols, ww, ext = g.export()
        for d in (0, len(ext) // 3, len(ext) - 1):
            assert np.array_equal(g.sssp(int(ext[d])), oracle.sssp(off, cols, ww, d))
            assert np.array_equal(g.bfs(int(ext[d])), oracle.bfs(off, cols, d))


def test_sssp_edge_cases(h2):
    """zero / -0.0 weights, unreachable vertices, unknown source, negative and NaN weights"""
    ids = np.array([10, 20, 30, 40, 50], np.uint64)
    src = np.array([10, 10, 20, 30, 40], np.uint64)
    dst = np.array([20, 30, 30, 40, 10], np.uint64)
    w = np.array([0.0, 2.0, -0.0, 0.5, 1.0], np.float32)
    g = h2.Replica.from_edges(5, ids, src, dst, w)
    off, cols, ww, _ = g.export()
    d = g.sssp(10)
    assert np.array_equal(d, oracle.sssp(off, cols, ww, 0))
    assert np.array_equal(d, [0.0, 0.0, 0.0, 0.5, np.inf]) and not np.signbit(d[2])
    with pytest.raises(h2.H2tapError):
        g.sssp(11)                                            # not a live vertex
    for bad in (-1.0, np.nan):
        wb = w.copy()
        wb[3] = bad
        with pytest.raises(h2.H2tapError):
            h2.Replica.from_edges(5, ids, src, dst, wb).sssp(10)


def test_empty_batch_is_identity_and_errors_leave_state(h2):
    scale = 10
    src, dst, w = synth.rmat_edges(scale, 3)
    g, o = pair_from_edges(h2, 1 << scale, None, src, dst, w)
    before = g.export(checksums=True)
    g.apply(Batch.empty(0), 5)
    after = g.export(checksums=True)
    assert_same(after[:4], before[:4]) and after[4] == before[4]
    assert g.info()["snapshot_ts"] == 5
    rc, _ = g.apply(Batch.of([(EDGE_INSERT, 0, 1, 1.0, 9)]), 4, raise_on_error=False)
    assert rc == -6                                              # snapshot regression
    rc, _ = g.apply(Batch.of([(EDGE_INSERT, 0, 1, 1.0, 5)]), 9, raise_on_error=False)
    assert rc == -5                                              # stale ts
    rc, _ = g.apply(Batch.of([(9, 0, 1, 1.0, 7)]), 9, raise_on_error=False)
    assert rc == -1                                              # unknown kind
    assert_same(g.export(), before[:4])
    assert g.info()["snapshot_ts"] == 5


def test_delete_all_edges(h2):
    src, dst, w = synth.rmat_edges(9, 4)
    g, o = pair_from_edges(h2, 512, None, src, dst, w)
    off, cols, _, ids = g.export()
    u = np.repeat(ids, np.diff(off))
    b = Batch(np.full(len(u), EDGE_DELETE, np.uint8), u, ids[cols], np.zeros(len(u), np.float32),
              np.full(len(u), 3, np.uint64))
    st = step(g, o, b, 3, "delete all")
    assert g.info()["n_edges"] == 0 and st["n_del"] == len(u)


def test_create_from_csr_roundtrip_and_validation(h2):
    src, dst, w = synth.rmat_edges(11, 8)
    ids = np.arange(1 << 11, dtype=np.uint64) * 5 + 1
    g = h2.Replica.from_edges(1 << 11, ids, ids[src], ids[dst], w, 3)
    off, cols, ww, ext = g.export()
    g2 = h2.Replica.from_csr(off, cols, ww, ext, 3)
    assert_same(g2.export(), (off, cols, ww, ext))
    bad = cols.copy()
    bad[0] = 1 << 11                                          # column out of range
    with pytest.raises(h2.H2tapError):
        h2.Replica.from_csr(off, bad, ww, ext)
    r = int(np.argmax(np.diff(off) >= 2))                     # a row with >= 2 entries
    dup = cols.copy()
    dup[off[r] + 1] = dup[off[r]]                             # duplicate column in a row
    with pytest.raises(h2.H2tapError):
        h2.Replica.from_csr(off, dup, ww, ext)
    with pytest.raises(h2.H2tapError):                        # edge endpoint outside the vertex set
        h2.Replica.from_edges(4, None, np.array([0], np.uint64), np.array([9], np.uint64),
                              np.array([1.0], np.float32))


def test_checksums_match_oracle_definition(h2):
    src, dst, w = synth.rmat_edges(12, 6)
    g, o = pair_from_edges(h2, 1 << 12, None, src, dst, w)
    b = synth.rmat_batch(12, 6, 0, 5000, len(src))
    step(g, o, b, int(b.ts.max()))
    assert g.checksums() == oracle.checksums(*o.export())


def test_device_resident_batch(h2):
    import torch
    src, dst, w = synth.rmat_edges(12, 12)
    g, o = pair_from_edges(h2, 1 << 12, None, src, dst, w)
    b = synth.rmat_batch(12, 12, 0, 8000, len(src), p_weight=0.1)
    dev = Batch(*(torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a).cuda()
                  for a in (b.kind, b.src, b.dst, b.w, b.ts)))
    st = g.apply(dev, int(b.ts.max()))
    o.apply(b, int(b.ts.max()))
    assert_same(g.export(), o.export(), "device batch")
    assert st["n_visible"] == len(b)


def test_device_resident_batches_with_node_ops(h2):
    """device batches are read in place when nothing is pending: node ops, deferral, then
    a batch that lands on top of pending ops (the staged path)"""
    import torch
    shape = synth.LdbcShape(n_person=256, n_msg=8000, e_person=12000)
    seed = synth.seed_of("c2") + 5
    ids = synth.ldbc_vertices(shape)
    src, dst, w = synth.ldbc_edges(shape, seed)
    g, o = pair_from_edges(h2, shape.n_vertices, ids, src, dst, w)
    ts = 0
    for k in range(4):
        b = synth.ldbc_batch(shape, seed, k, 4000, ts_base=ts)
        dev = Batch(*(torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a).cuda()
                      for a in (b.kind, b.src, b.dst, b.w, b.ts)))
        snap = int(b.ts.max()) - (200 if k % 2 == 0 else 0)    # even batches leave ops pending
        st = g.apply(dev, snap)
        rc, ost = o.apply(b, snap)
        assert rc == 0 and st["n_visible"] == ost["n_visible"] and st["n_deferred"] == ost["n_deferred"]
        assert_same(g.export(), o.export(), f"device ldbc batch {k}")
        ts = int(b.ts.max())


def test_staged_batches_pipeline(h2):
    """h2tap_batch_stage: batch k+1's copy overlaps batch k's apply; results as the oracle"""
    import torch
    src, dst, w = synth.rmat_edges(12, 33)
    g, o = pair_from_edges(h2, 1 << 12, None, src, dst, w)
    bs, ts = [], 0
    for k in range(5):
        b = synth.rmat_batch(12, 33, k, 6000, len(src), p_weight=0.1, ts_base=ts)
        ts = int(b.ts.max())
        bs.append(b)
    pin = [Batch(*(torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a).pin_memory()
                   for a in (b.kind, b.src, b.dst, b.w, b.ts))) for b in bs]
    staged = g.stage(pin[0])
    for k, b in enumerate(bs):
        nxt = g.stage(pin[k + 1]) if k + 1 < len(bs) else None
        snap = int(b.ts.max()) - (50 if k == 2 else 0)          # batch 3 lands on pending ops
        st = g.apply(staged, snap)
        rc, ost = o.apply(b, snap)
        assert rc == 0 and st["n_visible"] == ost["n_visible"]
        assert st["h2d_bytes"] >= b.nbytes()                    # the staged copy is accounted
        assert_same(g.export(), o.export(), f"staged batch {k}")
        staged = nxt


def test_staged_slots_interleaved(h2):
    """A staged slot is refilled once the cycle that used it passed its last read of it:
    staged batches interleaved with device-resident and host batches, a cycle with no merge,
    a staged batch applied right away, and two staged at once - all as the oracle"""
    import torch
    src, dst, w = synth.rmat_edges(11, 35)
    g, o = pair_from_edges(h2, 1 << 11, None, src, dst, w)
    ts = 0
    bs = []
    for k in range(8):
        b = synth.rmat_batch(11, 35, k, 3000, len(src), p_weight=0.1, ts_base=ts)
        ts = int(b.ts.max())
        bs.append(b)

    def pin(b):
        return Batch(*(torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a).pin_memory()
                       for a in (b.kind, b.src, b.dst, b.w, b.ts)))

    def dev(b):
        return Batch(*(torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a).cuda()
                       for a in (b.kind, b.src, b.dst, b.w, b.ts)))

    def both(x, b):
        st = g.apply(x, int(b.ts.max()))
        rc, _ = o.apply(b, int(b.ts.max()))
        assert rc == 0
        return st

    p = [pin(b) for b in bs]
    s1 = g.stage(p[1])
    both(dev(bs[0]), bs[0])
    both(s1, bs[1])
    both(g.stage(p[2]), bs[2])              # staged and applied at once
    s3, s4 = g.stage(p[3]), g.stage(p[4])   # two outstanding
    empty = Batch.empty(0)
    g.apply(empty, int(bs[2].ts.max()))     # a cycle with no merge
    o.apply(empty, int(bs[2].ts.max()))
    both(s3, bs[3])
    both(s4, bs[4])
    both(bs[5], bs[5])                      # host batch (copied inside the call)
    s6 = g.stage(p[6])
    both(s6, bs[6])
    assert_same(g.export(), o.export(), "deferred staging")


def test_chunked_create_last_duplicate_wins(h2, monkeypatch):
    """create_from_edges goes in as insert batches of H2TAP_CREATE_CHUNK edges (2^28 by
    default); duplicates across chunks: the last one wins, as in one batch"""
    monkeypatch.setenv("H2TAP_CREATE_CHUNK", "997")
    src, dst, w = synth.rmat_edges(10, 44, n=20000)             # many duplicate (src, dst) pairs
    ids = np.arange(1 << 10, dtype=np.uint64) * 2 + 1
    g, o = pair_from_edges(h2, 1 << 10, ids, ids[src], ids[dst], w)
    assert_same(g.export(), o.export(), "chunked create")
    b = synth.rmat_batch(10, 44, 0, 3000, len(src), p_weight=0.1)
    b.src, b.dst = ids[b.src % (1 << 10)], ids[b.dst % (1 << 10)]
    step(g, o, b, int(b.ts.max()), "after chunked create")


def test_two_phase_prepare_commit_abort(h2):
    """h2tap_delta_apply_prepare leaves every read at the old snapshot until commit;
    abort drops the prepared cycle (replica unchanged, the same batch applies later);
    a prepared cycle blocks other applies (E_INVAL) - the all-or-nothing step of a
    sharded apply."""
    shape = synth.LdbcShape(n_person=256, n_msg=6000, e_person=9000)
    seed = synth.seed_of("c2")
    ids = synth.ldbc_vertices(shape)
    src, dst, w = synth.ldbc_edges(shape, seed)
    g, o = pair_from_edges(h2, len(ids), ids, src, dst, w)
    before = g.export(checksums=True)
    b = synth.ldbc_batch(shape, seed, 0, 3000, ts_base=1)
    snap = int(b.ts.max())
    rc, st = g.prepare(b, snap)
    assert rc == 0 and st["n_visible"] == len(b)
    assert g.export(checksums=True)[4] == before[4] and g.info()["snapshot_ts"] == 0
    rc2, _ = g.apply(b, snap, raise_on_error=False)
    assert rc2 == -1                                   # prepared: commit or abort first
    g.abort()
    assert g.export(checksums=True)[4] == before[4]
    rc, _ = g.prepare(b, snap)
    assert rc == 0
    g.commit()
    o.apply(b, snap)
    assert_same(g.export(), o.export(), "two-phase commit")
    assert g.info()["snapshot_ts"] == snap
    assert g.info()["n_edges"] == step.last_E[id(g)] + st["n_new"] - st["n_del"] - st["n_casc"]   # I6
    step.last_E[id(g)] = g.info()["n_edges"]
    with pytest.raises(h2.H2tapError):
        g.commit()                                     # nothing prepared
    b2 = synth.ldbc_batch(shape, seed, 1, 3000, ts_base=snap)
    step(g, o, b2, int(b2.ts.max()), "after two-phase")


def test_async_apply_stream(h2):
    """h2tap_delta_apply_async: cycles enqueued back to back (the next one reads the previous
    cycle's sizes at its first read-back) give the same replica as the synchronous path, with
    node ops, deferral and sparse ids; stats come out one call late and at h2tap_replica_sync;
    a read call (export) completes the in-flight cycle; a refused batch leaves the committed
    cycles in place."""
    shape = synth.LdbcShape(n_person=256, n_msg=6000, e_person=9000)
    seed = synth.seed_of("c2")
    ids = synth.ldbc_vertices(shape)
    src, dst, w = synth.ldbc_edges(shape, seed)
    g, o = pair_from_edges(h2, len(ids), ids, src, dst, w)
    ts, seen = 1, []
    for k in range(6):
        b = synth.ldbc_batch(shape, seed, k, 2500, ts_base=ts)
        snap = int(np.quantile(b.ts, 0.9)) if k % 2 else int(b.ts.max())   # some ops deferred
        st = g.apply_async(b, snap)
        if st is not None:
            seen.append(st)
        rc, _ = o.apply(b, snap)
        assert rc == 0
        ts = int(b.ts.max()) + 1
        if k == 2:                                       # a read completes the in-flight cycle
            assert_same(g.export(), o.export(), "async, read in the middle")
    last = g.sync()
    assert last is not None and g.sync() is None
    seen.append(last)
    assert len(seen) == 6
    assert_same(g.export(), o.export(), "async stream")
    assert g.info()["n_pending"] == o.info()["n_pending"]
    # a stale op refused by an asynchronous call: the earlier cycles stay committed
    before = g.export(checksums=True)
    with pytest.raises(h2.H2tapError):
        g.apply_async(Batch.of([(EDGE_INSERT, int(ids[0]), int(ids[1]), 1.0, 1)]), ts + 5)
    assert g.export(checksums=True)[4] == before[4]
    g.apply(Batch.empty(0), ts + 100)
    o.apply(Batch.empty(0), ts + 100)
    assert_same(g.export(), o.export(), "sync after async")


def test_pending_export_and_checkpoint_restore(h2):
    """h2tap_pending_export equals O1's pending set (pinned in test_oracle_pins.py) after cycles
    with deferral; a checkpoint (CSR export + pending ops) restored through create_from_csr and
    one apply of the pending ops at the same snapshot continues exactly like the original."""
    scale, seed = 10, 21
    n = 1 << scale
    src, dst, w = synth.rmat_edges(scale, seed)
    g, o = pair_from_edges(h2, n, None, src, dst, w)
    ts = 0
    for k in range(3):
        b = synth.rmat_batch(scale, seed, k, 3000, len(src), p_insert=0.7, p_weight=0.1, ts_base=ts)
        snap = int(np.quantile(b.ts, 0.7))
        step(g, o, b, snap, f"pending {k}")
        ts = int(b.ts.max())
        got, ref = g.pending(), o.pending()
        for name, x, y in zip(("kind", "src", "dst", "w", "ts"), got[:5], ref[:5]):
            assert np.array_equal(x.view(np.uint32) if x.dtype == np.float32 else x,
                                  y.view(np.uint32) if y.dtype == np.float32 else y), f"pending {name}"
        # arrival numbers: the same order and spacing (the replica also numbered its create edges)
        assert len(got[5]) == len(ref[5])
        if len(got[5]):
            assert np.array_equal(got[5] - got[5][0], ref[5] - ref[5][0])
    # checkpoint -> restore
    off, cols, ww, ext = g.export()
    kind, s_, d_, w_, t_, q_ = g.pending()
    S = g.info()["snapshot_ts"]
    h = h2.Replica.from_csr(off, cols, ww, ext, create_ts=S)
    h.apply(Batch(kind, s_, d_, w_, t_), S)
    assert h.info()["n_pending"] == len(kind)
    b = synth.rmat_batch(scale, seed, 9, 3000, len(src), p_insert=0.7, p_weight=0.1, ts_base=ts)
    last = int(b.ts.max())
    g.apply(b, last)
    h.apply(b, last)
    assert_same(h.export(), g.export(), "restored checkpoint")


def test_idmap_prefix_reuse_across_cycles(h2):
    """Node-mode cycles leave the ID-map prefix the two buffers already share:
    node ops alternate between the top, the bottom and the middle of the id space, prepared
    cycles are aborted in between (the back buffer then holds a partial rewrite), and the
    asynchronous path swaps buffers without a host read-back - the ID map and the CSR stay
    bit-exact with O1 after every cycle."""
    n = 1 << 12
    src, dst, w = synth.rmat_edges(12, 11, n=8 * n)
    ids = np.arange(n, dtype=np.uint64) * 4 + 100          # gaps: new ids fit anywhere
    g, o = pair_from_edges(h2, n, ids, ids[src], ids[dst], w)
    rng = np.random.default_rng(5)
    live = set(int(x) for x in ids)
    ts = 0

    def batch(lo_frac, hi_frac, k):
        nonlocal ts
        ops = []
        cand = sorted(x for x in live if lo_frac * 4 * n <= x - 100 < hi_frac * 4 * n)
        for v in rng.choice(cand, size=min(6, len(cand)), replace=False):
            ts += 1
            ops.append((NODE_DELETE, int(v), 0, 0.0, ts))
            live.discard(int(v))
        for j in range(5):   # new ids inside the region (odd offsets: never an old id)
            v = 100 + int(rng.integers(int(lo_frac * 4 * n), int(hi_frac * 4 * n))) | 1
            if v in live:
                continue
            ts += 1
            ops.append((NODE_INSERT, v, 0, 0.0, ts))
            live.add(v)
            u = int(rng.choice(sorted(live)))
            ops.append((EDGE_INSERT, v, u, float(j), ts))
            ops.append((EDGE_INSERT, u, v, float(k), ts))
        for _ in range(40):  # edge ops over the whole graph
            ts += 1
            a, b = (int(x) for x in rng.choice(sorted(live), 2))
            ops.append((EDGE_INSERT if rng.random() < 0.7 else EDGE_DELETE, a, b, float(rng.random()), ts))
        return Batch.of(ops)

    regions = [(0.9, 1.0), (0.0, 0.1), (0.45, 0.55), (0.95, 1.0), (0.95, 1.0), (0.0, 0.05)]
    for k, (lo, hi) in enumerate(regions):
        if k % 2 == 1:  # a prepared cycle that is thrown away (its ops never happened)
            saved_live, saved_ts = set(live), ts
            bad = batch(0.0, 1.0, 100 + k)
            rc, _ = g.prepare(bad, ts)
            assert rc == 0
            g.abort()
            live, ts = saved_live, saved_ts
        b = batch(lo, hi, k)
        step(g, o, b, ts, f"region {lo}-{hi} cycle {k}")
    # asynchronous cycles: the swap is enqueued, the next cycle reads the ID map it left
    for k, (lo, hi) in enumerate(regions[:4]):
        b = batch(lo, hi, 50 + k)
        g.apply_async(b, ts)
        o.apply(b, ts)
    g.sync()
    assert_same(g.export(), o.export(), "async node-mode cycles")


def test_sort_heavy_duplicate_keys(h2):
    """The edge-key sort's sample-sort path puts equal keys in one bucket: a batch where one
    (src, dst) pair carries 20K ops (a bucket far above the 8K a CTA sorts in shared memory,
    so its chunked global-memory path runs) and another 9K, around 30K other ops, all with
    interleaved timestamps - latest commit wins must still come out of a stable sort."""
    n = 1 << 12
    src, dst, w = synth.rmat_edges(12, 21, n=8 * n)
    g, o = pair_from_edges(h2, n, None, src, dst, w)
    rng = np.random.default_rng(9)
    m = 60000
    kind = rng.choice([EDGE_INSERT, EDGE_DELETE, EDGE_WEIGHT], size=m, p=[0.6, 0.2, 0.2]).astype(np.uint8)
    s = rng.integers(0, n, m).astype(np.uint64)
    d = rng.integers(0, n, m).astype(np.uint64)
    s[:20000], d[:20000] = 7, 9            # one heavy key
    s[20000:29000], d[20000:29000] = 4095, 0
    perm = rng.permutation(m)
    b = Batch(kind[perm], s[perm], d[perm], rng.random(m).astype(np.float32),
              rng.integers(1, 5000, m).astype(np.uint64))
    step(g, o, b, 5000, "heavy duplicate keys")
    b2 = synth.rmat_batch(12, 21, 1, 30000, len(src))
    b2.ts += 5000
    step(g, o, b2, int(b2.ts.max()), "after heavy keys")


def test_cascade_deleted_ids_spread_wide(h2):
    """Node deletes whose ids span more than the cascade pass's shared-memory bitmap window
    (8192 words = 262,144 ids): the pass reads the global deleted-vertex bitmap instead; and a
    second batch whose deletes sit close together (the shared-memory window)"""
    scale = 20
    n = 1 << scale
    src, dst, w = synth.rmat_edges(scale, 17, n=2 * n)
    g, o = pair_from_edges(h2, n, None, src, dst, w)
    deg = np.bincount(dst.astype(np.int64), minlength=n)        # vertices with in-edges
    hubs = np.argsort(-deg)[:40]
    ts = 1
    ops = []
    for v in sorted(int(x) for x in hubs) + [3, n - 5]:         # ids from 3 to n - 5
        ops.append((NODE_DELETE, v, 0, 0.0, ts))
        ts += 1
    b = Batch.of(ops).concat(synth.rmat_batch(scale, 17, 0, 5000, len(src), ts_base=ts))
    st = step(g, o, b, int(b.ts.max()), "wide node deletes")
    assert st["n_casc"] > 0
    ts = int(b.ts.max()) + 1
    live = g.export()[3]
    close = [int(x) for x in live[1000:1010]]                   # ten adjacent ids
    b2 = Batch.of([(NODE_DELETE, v, 0, 0.0, ts + i) for i, v in enumerate(close)])
    step(g, o, b2, ts + 20, "close node deletes")
