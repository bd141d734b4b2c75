"""Pins for OD, the dynamic-replica oracle (Algorithm 1; readings D1-D5 of
DESIGN.md §15), checked against things other than itself:

* the paper's Fig. 2 worked example in its record layout (tests/golden/fig2_records.json,
  P:L667-700), hand-derived result with the deleted node's slot kept (D3)
* O1 in tombstone mode (an independent, pinned implementation) replaying the flat-op form
  of D1-D5 on random multi-cycle record batches
* small special cases: empty cycle, invalid records, insert-then-delete, create last-wins
"""
import numpy as np
import pytest

import synth
from oracle import O1
from oracle.od_dynamic import DynamicOracle, flat_ops
from synth import Batch
from test_oracle_pins import load_fig2_records


def fig2_dyn():
    g, rb = load_fig2_records()
    e = np.array(g["edges"], dtype=object)
    return g, rb, DynamicOracle(g["vertices"], e[:, 0], e[:, 1], e[:, 2])


def test_fig2_records_dynamic():
    g, rb, o = fig2_dyn()
    st = o.apply_records(rb.records, rb.inserts, rb.weights, rb.deletes)
    off, cols, w, ids, live = o.export()
    # node 4 keeps dense id 3 with an empty entry; 5 (> xid = 4, line 8) is appended;
    # 3->5 to the node created in the same cycle is kept (D2); 3->4 and 1->4 go with node 4
    assert ids.tolist() == [1, 2, 3, 4, 5] and live.tolist() == [1, 1, 1, 0, 1]
    assert off.tolist() == [0, 0, 1, 2, 2, 3]
    assert cols.tolist() == [2, 4, 0] and w.tolist() == [0.25, 5.0, 2.0]
    assert st == dict(n_new=2, n_upd=0, n_del=3, n_casc=0, n_gated=0, n_vertex_inserted=1,
                      n_vertex_deleted=1)


def o1_tomb(ids, src, dst, w):
    return O1.from_edges(len(ids), np.asarray(ids, np.uint64), np.asarray(src, np.uint64),
                         np.asarray(dst, np.uint64), np.asarray(w, np.float32), 0, tombstone=True)


@pytest.mark.parametrize("seed", range(12))
def test_dynamic_equals_o1_tombstone_on_flat_form(seed):
    rng = np.random.default_rng(seed)
    n = 16
    ids = np.arange(n, dtype=np.uint64) * 2
    m = 40
    src, dst = ids[rng.integers(0, n, m)], ids[rng.integers(0, n, m)]
    w = rng.random(m).astype(np.float32)
    d = DynamicOracle(ids, src, dst, w)
    t = o1_tomb(ids, src, dst, w)
    for cyc in range(5):
        xid = max(d.ids)
        rb = synth.dyn_record_batch(seed, cyc, xid, 25, n_new=5, max_slice=4, p_deleted=0.08)
        ops = flat_ops(rb.records, rb.inserts, rb.weights, rb.deletes, xid)
        st = d.apply_records(rb.records, rb.inserts, rb.weights, rb.deletes)
        ts = cyc + 1
        b = Batch.of([(k, s, x, y, ts) for (k, s, x, y) in ops])
        assert t.apply(b, ts)[0] == 0
        off, cols, ww, ii, live = d.export()
        toff, tcols, tw, tids = t.export()
        assert ii.tolist() == tids.tolist() and live.tolist() == t.live().tolist()
        assert off.tolist() == toff.tolist() and cols.tolist() == tcols.tolist()
        assert ww.tolist() == tw.tolist()
        assert st["n_new"] >= 0 and st["n_vertex_deleted"] <= len(ii)


def test_empty_and_invalid_cycles_change_nothing():
    g, rb, o = fig2_dyn()
    before = o.export()
    o.apply_records([], rb.inserts, rb.weights, rb.deletes)
    rb.records["valid"] = 0
    o.apply_records(rb.records, rb.inserts, rb.weights, rb.deletes)
    assert all(np.array_equal(a, b) for a, b in zip(before, o.export()))


def rec(node, ins=(), dels=(), deleted=0, io=0, do=0):
    return dict(ts=1, node=node, ins_off=io, ins_cnt=len(ins), del_off=do, del_cnt=len(dels),
                valid=1, deleted=deleted, inserted=0)


def test_insert_then_delete_same_edge_and_last_insert_wins():
    o = DynamicOracle([1, 2, 3])
    # two records of node 1: insert 1->2 (w 1), insert 1->2 (w 4) and 1->3, delete 1->3
    recs = [rec(1, [2], io=0), rec(1, [2, 3], [3], io=1, do=0)]
    st = o.apply_records(recs, [2, 2, 3], np.float32([1, 4, 9]), [3])
    off, cols, w, _, _ = o.export()
    assert off.tolist() == [0, 1, 1, 1] and cols.tolist() == [1] and w.tolist() == [4.0]  # D1
    assert st["n_new"] == 2 and st["n_del"] == 1


def test_new_node_deleted_in_same_cycle_and_gated_edges():
    o = DynamicOracle([1, 2])
    recs = [rec(7, [1]), rec(7, deleted=1), rec(1, [7, 9], io=1), rec(5, [2], io=3)]
    st = o.apply_records(recs, [1, 7, 9, 2], np.float32([1, 2, 3, 4]), [])
    off, cols, w, ids, live = o.export()
    # 7 > xid = 2 is created and deleted by the same cycle: never inserted (D3), so 7->1 and
    # 1->7 are gated, and so is 1->9 (unknown); 5 > xid is a new node with 5->2
    assert ids.tolist() == [1, 2, 5] and live.tolist() == [1, 1, 1]
    assert off.tolist() == [0, 0, 0, 1] and cols.tolist() == [1]
    assert st["n_gated"] == 3 and st["n_casc"] == 0 and st["n_vertex_deleted"] == 0


def test_create_rejects_unknown_endpoints_and_keeps_last():
    with pytest.raises(ValueError):
        DynamicOracle([1, 2], [1], [3], [1.0])
    with pytest.raises(ValueError):
        DynamicOracle([2, 1])
    o = DynamicOracle([1, 2], [1, 1], [2, 2], [1.0, 2.0])
    assert o.export()[2].tolist() == [2.0]
