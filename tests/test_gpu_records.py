"""Parity of h2tap_delta_apply_records (the paper's delta-record layout, §5.1-5.2) with the
oracle: O1 replaying the oracle's own scan of the same records (oracle.expand_records).
Bar: bit-exact offsets / cols / weights / ID map after every batch."""
import json
import os

import numpy as np
import pytest

import oracle
import synth
from oracle import O1
from synth import Batch

from test_gpu_parity import assert_same, pair_from_edges

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module")
def h2():
    import paper_conf_edbt_jibrilabs23_b200 as h2
    return h2


def rstep(g, o, rb, snap, ctx=""):
    st = g.apply_records(rb, snap)
    ops = oracle.expand_records(rb.records, rb.inserts, rb.weights, rb.deletes)
    rc, ost = o.apply(Batch.of(zip(*ops)) if ops[0] else Batch.empty(0), snap)
    assert rc == 0
    assert st["n_visible"] == ost["n_visible"] and st["n_deferred"] == ost["n_deferred"], ctx
    assert_same(g.export(), o.export(), ctx)
    return st


def test_fig2_records(h2):
    from test_oracle_pins import load_fig2_records
    g, rb = load_fig2_records()
    e = np.array(g["edges"], dtype=object)
    rep = h2.Replica.from_edges(len(g["vertices"]), np.array(g["vertices"], np.uint64),
                                np.array(e[:, 0], np.uint64), np.array(e[:, 1], np.uint64),
                                np.array(e[:, 2], np.float32), g["create_ts"])
    st = rep.apply_records(rb, g["snapshot_ts"])
    assert st["n_visible"] == 7
    off, cols, w, ids = rep.export()
    ex = g["expected"]
    assert ids.tolist() == ex["ext_ids"] and off.tolist() == ex["offsets"]
    assert cols.tolist() == ex["cols"] and w.tolist() == ex["weights"]


def test_records_fuzz_multibatch_with_invalid_and_deferred(h2):
    n = 48
    ids = np.arange(n, dtype=np.uint64) * 2 + 1
    rng = np.random.default_rng(11)
    src = ids[rng.integers(0, n, 300)]
    dst = ids[rng.integers(0, n, 300)]
    g, o = pair_from_edges(h2, n, ids, src, dst, rng.random(300).astype(np.float32))
    ts = 0
    for k in range(8):
        b = synth.fuzz_batch(seed=21, k=k, n=4000, n_ids=2 * n + 8, probs=(0.04, 0.02, 0.6, 0.34, 0.0),
                             ts_lo=ts + 1, ts_span=400)
        b = b.slice(np.lexsort((b.src, b.ts)))
        rb = synth.records_from_ops(b)
        rb.records["valid"][np.arange(len(rb)) % 17 == 3] = 0      # used in an earlier cycle
        snap = ts + 300                                            # the rest stays pending
        rstep(g, o, rb, snap, f"records batch {k}")
        ts = snap + 100


def test_records_ldbc_shaped_and_device_resident(h2):
    import torch
    shape = synth.LdbcShape(n_person=512, n_msg=20000, e_person=40000)
    seed = synth.seed_of("c2")
    ids = synth.ldbc_vertices(shape)
    src, dst, w = synth.ldbc_edges(shape, seed)
    g, o = pair_from_edges(h2, shape.n_vertices, ids, src, dst, w)
    ts = 0
    for k in range(3):
        b = synth.ldbc_batch(shape, seed, k, 5000, ts_base=ts)
        ts = int(b.ts.max())
        rb = synth.records_from_ops(b)
        assert rb.records["inserted"].any() and rb.records["deleted"].any()
        if k == 1:  # device-resident records and arrays
            dev = synth.RecordBatch(torch.from_numpy(rb.records.view(np.uint8).copy()).cuda(),
                                    torch.from_numpy(rb.inserts.view(np.int64)).cuda(),
                                    torch.from_numpy(rb.weights).cuda(), torch.from_numpy(rb.deletes.view(np.int64)).cuda())
            st = g.apply_records(dev, ts)
            ops = oracle.expand_records(rb.records, rb.inserts, rb.weights, rb.deletes)
            rc, _ = o.apply(Batch.of(zip(*ops)), ts)
            assert rc == 0 and st["h2d_bytes"] < 1024 < rb.records.nbytes  # only the counters block
            assert_same(g.export(), o.export(), "ldbc device records")
        else:
            rstep(g, o, rb, ts, f"ldbc records {k}")


def test_records_errors_leave_state(h2):
    from test_oracle_pins import load_fig2_records
    gj, rb = load_fig2_records()
    e = np.array(gj["edges"], dtype=object)
    rep = h2.Replica.from_edges(len(gj["vertices"]), np.array(gj["vertices"], np.uint64),
                                np.array(e[:, 0], np.uint64), np.array(e[:, 1], np.uint64),
                                np.array(e[:, 2], np.float32), gj["create_ts"])
    before = rep.export()
    bad = synth.RecordBatch(rb.records.copy(), rb.inserts, rb.weights, rb.deletes)
    bad.records["del_cnt"][3] = 4                                  # slice past the end of deletes
    rc, _ = rep.apply_records(bad, 20, raise_on_error=False)
    assert h2.STATUS[rc] == "E_INVAL"
    bad = synth.RecordBatch(rb.records.copy(), rb.inserts, rb.weights, rb.deletes)
    bad.records["deleted"][4] = 2                                  # flag other than 0/1
    rc, _ = rep.apply_records(bad, 20, raise_on_error=False)
    assert h2.STATUS[rc] == "E_INVAL"
    assert_same(rep.export(), before, "after refused record batches")
    assert rep.info()["snapshot_ts"] == 0
    empty = synth.records_from_ops(Batch.empty(0))
    st = rep.apply_records(empty, 1)
    assert st["n_visible"] == 0 and rep.info()["snapshot_ts"] == 1
