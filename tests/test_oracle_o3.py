"""Pins for O3 (oracle/o3_alg2.cpp), the Algorithm-2 flat-CSR merge on the host (CPU only).

O3 is an independent implementation of the same propagation result as O1 (the sequential
replay, itself pinned to the O2 brute force in test_oracle_pins.py): Algorithm 2's row
walk over per-node combined deltas instead of a replay onto ordered maps.
Pinned here against things other than itself:
* bit-exact equality with O1 after every batch on fuzz streams with every op kind,
  equal timestamps, out-of-order arrival, deferral, revived and sparse IDs;
* the paper's Fig. 2 worked example (tests/golden/fig2.json);
* the LDBC-shaped (node ops, sparse external IDs) and RMAT generators at small sizes;
* the special case Algorithm 2 itself states: every new ID above xid -> appended rows
  (lines 16-17), and an untouched row is a byte copy of the old one (lines 8-10, 13-15);
* create = the textbook CSR build (numpy lexsort + keep-last unique, reading A17);
* 1 thread and N threads give the same CSR; checksums = oracle.checksum's definition.
"""
import json
import os

import numpy as np
import pytest

import oracle
import synth
from oracle import O1, O3
from synth import Batch, NODE_INSERT, NODE_DELETE, EDGE_INSERT

HERE = os.path.dirname(os.path.abspath(__file__))


def same(a, b):
    for x, y in zip(a, b):
        x, y = np.asarray(x), np.asarray(y)
        if x.dtype == np.float32:
            x, y = x.view(np.uint32), y.view(np.uint32)
        if x.shape != y.shape or not np.array_equal(x, y):
            return False
    return True


def both(n, ids, src, dst, w, create_ts=0):
    return (O1.from_edges(n, ids, src, dst, w, create_ts), O3.from_edges(n, ids, src, dst, w, create_ts))


def test_fig2_worked_example():
    g = json.load(open(os.path.join(HERE, "golden", "fig2.json")))
    e = np.array(g["edges"], dtype=object)
    o = O3.from_edges(len(g["vertices"]), np.array(g["vertices"], np.uint64), np.array(e[:, 0], np.uint64),
                      np.array(e[:, 1], np.uint64), np.array(e[:, 2], np.float32), g["create_ts"])
    rc, st = o.apply(Batch.of(g["ops"]), g["snapshot_ts"])
    assert rc == 0 and st["n_visible"] == len(g["ops"])
    off, cols, w, ids = o.export()
    ex = g["expected"]
    assert ids.tolist() == ex["ext_ids"] and off.tolist() == ex["offsets"]
    assert cols.tolist() == ex["cols"] and w.tolist() == ex["weights"]


@pytest.mark.parametrize("threads", [1, 4])
def test_fuzz_vs_o1_every_batch(threads):
    oracle.set_threads(threads)
    for case in range(150):
        rng = np.random.default_rng(1000 + case)
        nid = 4 + case % 9
        ids = np.unique(rng.integers(0, 3 * nid, nid).astype(np.uint64)) if case % 3 else np.arange(nid, dtype=np.uint64)
        m = int(rng.integers(0, 4 * len(ids) + 1))
        src = ids[rng.integers(0, len(ids), m)]
        dst = ids[rng.integers(0, len(ids), m)]
        w = (rng.integers(0, 64, m) / 8).astype(np.float32)
        a, b = both(len(ids), ids, src, dst, w)
        snap = 0
        for k in range(4):
            bt = synth.fuzz_batch(seed=case, k=k, n=1 + (case * 7 + k) % 40, n_ids=3 * nid + 2, ts_lo=snap + 1,
                                  ts_span=6)
            s = snap + (3 if k % 2 else 6)   # some ops stay pending, then become visible
            ra, sa = a.apply(bt, s)
            rb, sb = b.apply(bt, s)
            assert ra == rb and sa == sb, (case, k)
            if ra == 0:
                snap = s
            assert same(a.export(), b.export()), (case, k)
            assert a.info() == b.info()
    oracle.set_threads(0)


def test_exhaustive_length3_vs_o1():
    """Every op sequence of length 3 over 3 vertices (two live, one never existed) with
    distinct timestamps, from the same initial graph as O1's exhaustive pins."""
    from test_oracle_pins import _all_ops, INIT_LIVE, INIT_EDGES
    import itertools
    ops = _all_ops(3)
    ids = np.array(INIT_LIVE, np.uint64)
    s = np.array([e[0] for e in INIT_EDGES], np.uint64)
    d = np.array([e[1] for e in INIT_EDGES], np.uint64)
    w = np.array([e[2] for e in INIT_EDGES], np.float32)
    for seq in itertools.product(ops, repeat=3):
        b = Batch.of([(k, x, y, z, t) for (k, x, y, z), t in zip(seq, (1, 2, 3))])
        o1 = O1.from_edges(len(ids), ids, s, d, w)
        o3 = O3.from_edges(len(ids), ids, s, d, w)
        assert o1.apply(b, 3)[0] == o3.apply(b, 3)[0] == 0
        assert same(o1.export(), o3.export()), seq


def test_errors_and_strong_guarantee():
    a, b = both(3, None, np.array([0, 1], np.uint64), np.array([1, 2], np.uint64), np.ones(2, np.float32), 5)
    before = b.export()
    bad = Batch.of([(EDGE_INSERT, 0, 2, 1.0, 6), (9, 0, 0, 0.0, 7)])
    assert b.apply(bad, 9)[0] == a.apply(bad, 9)[0] == oracle.E_INVAL
    stale = Batch.of([(EDGE_INSERT, 0, 2, 1.0, 5)])
    assert b.apply(stale, 9)[0] == a.apply(stale, 9)[0] == oracle.E_STALE_TS
    assert b.apply(Batch.of([]), 4)[0] == a.apply(Batch.of([]), 4)[0] == oracle.E_SNAPSHOT_REGRESSION
    assert same(b.export(), before)
    with pytest.raises(ValueError):
        O3.from_edges(2, None, np.array([0], np.uint64), np.array([5], np.uint64), np.ones(1, np.float32))


def test_ldbc_shaped_node_ops_vs_o1():
    shape = synth.LdbcShape(n_person=300, n_msg=6000, e_person=9000)
    seed = synth.seed_of("c2")
    ids = synth.ldbc_vertices(shape)
    src, dst, w = synth.ldbc_edges(shape, seed)
    a, b = both(len(ids), ids, src, dst, w)
    ts = 1
    for k in range(4):
        bt = synth.ldbc_batch(shape, seed, k, 3000, lodeg=(k == 2), ts_base=ts)
        s = int(bt.ts.max())
        assert a.apply(bt, s)[0] == b.apply(bt, s)[0] == 0
        ts = s + 1
        assert same(a.export(), b.export()), k


def test_rmat_with_weights_repeats_deferral_vs_o1():
    scale, seed = 10, synth.seed_of("c1")
    n = 1 << scale
    src, dst, w = synth.rmat_edges(scale, seed)
    a, b = both(n, None, src, dst, w)
    ts = 0
    for k in range(3):
        bt = synth.rmat_batch(scale, seed, k, 3000, len(src), p_insert=0.6, p_weight=0.2, p_repeat=0.3,
                              ops_per_txn=4, ts_base=ts)
        s = int(np.quantile(bt.ts, 0.9)) if k < 2 else int(bt.ts.max())
        assert a.apply(bt, s)[0] == b.apply(bt, s)[0] == 0
        ts = int(bt.ts.max()) + 1
        assert same(a.export(), b.export()), k


def test_append_new_ids_and_untouched_rows_copied():
    """Algorithm 2 lines 8-10 / 13-15 (untouched rows byte-identical) and 16-17 (new IDs
    above xid are appended after every old row)."""
    scale, seed = 9, 7
    n = 1 << scale
    src, dst, w = synth.rmat_edges(scale, seed)
    o = O3.from_edges(n, None, src, dst, w)
    off0, cols0, w0, ids0 = o.export()
    ops = [(NODE_INSERT, n + 5, 0, 0.0, 1), (NODE_INSERT, n + 9, 0, 0.0, 1),
           (EDGE_INSERT, n + 5, 3, 1.5, 2), (EDGE_INSERT, n + 9, n + 5, 2.5, 2), (EDGE_INSERT, 7, n + 9, 0.25, 3)]
    assert o.apply(Batch.of(ops), 3)[0] == 0
    off, cols, w1, ids = o.export()
    assert ids[:n].tolist() == ids0.tolist() and ids[n:].tolist() == [n + 5, n + 9]
    for r in range(n):
        if r == 7:
            continue
        assert cols[off[r]:off[r + 1]].tolist() == cols0[off0[r]:off0[r + 1]].tolist()
        assert w1[off[r]:off[r + 1]].view(np.uint32).tolist() == w0[off0[r]:off0[r + 1]].view(np.uint32).tolist()
    assert cols[off[n]:off[n + 1]].tolist() == [3] and cols[off[n + 1]:off[n + 2]].tolist() == [n]
    row7 = cols[off[7]:off[8]].tolist()
    assert row7 == sorted(set(cols0[off0[7]:off0[8]].tolist()) | {n + 1})


def test_create_is_textbook_csr_build():
    rng = np.random.default_rng(5)
    n = 300
    ids = np.unique(rng.integers(0, 10_000, n).astype(np.uint64))
    m = 5000
    src, dst = ids[rng.integers(0, len(ids), m)], ids[rng.integers(0, len(ids), m)]
    w = rng.random(m).astype(np.float32)
    off, cols, ww, got_ids = O3.from_edges(len(ids), ids, src, dst, w).export()
    s, d = np.searchsorted(ids, src), np.searchsorted(ids, dst)
    order = np.lexsort((np.arange(m), d, s))           # by (src, dst, arrival)
    s, d, wo = s[order], d[order], w[order]
    last = np.ones(m, bool)
    last[:-1] = (s[1:] != s[:-1]) | (d[1:] != d[:-1])  # keep the last duplicate (A17)
    assert got_ids.tolist() == ids.tolist()
    assert cols.tolist() == d[last].tolist()
    assert ww.view(np.uint32).tolist() == wo[last].view(np.uint32).tolist()
    assert off.tolist() == np.concatenate([[0], np.cumsum(np.bincount(s[last], minlength=len(ids)))]).tolist()


def test_threads_and_checksums():
    scale, seed = 11, 3
    n = 1 << scale
    src, dst, w = synth.rmat_edges(scale, seed)
    res = []
    for t in (1, 3, 8):
        oracle.set_threads(t)
        o = O3.from_edges(n, None, src, dst, w)
        bt = synth.rmat_batch(scale, seed, 0, 4000, len(src))
        assert o.apply(bt, int(bt.ts.max()))[0] == 0
        res.append((o.export(), o.checksums()))
    oracle.set_threads(0)
    for e, c in res[1:]:
        assert same(e, res[0][0]) and c == res[0][1]
    e, c = res[0]
    assert c == oracle.checksums(*e)
