"""The append-only delta store (h2tap_ds_*, §5.1) and the propagation cycle that
scans it (h2tap_delta_apply_store, §5.2-5.3) against oracle.DeltaStoreModel + O1
(pinned in tests/test_oracle_pins.py): bit-exact CSR / ID map after every cycle, every used
delta marked invalid, invisible deltas left for a later cycle, the paper's 8-byte weights
rounded to f32 the same way on both sides, concurrent appenders, chunk release, stale
deltas refused with nothing marked; full size: configs[2]'s stream through the store equals
O3 on the same ops (whole-export checksums)."""
import threading

import numpy as np
import pytest

import oracle
import synth
from oracle import O1
from synth import Batch

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def h2():
    import paper_conf_edbt_jibrilabs23_b200 as h2
    return h2


def same(g, o, ctx=""):
    for name, a, b in zip(("offsets", "cols", "weights", "ext_ids"), g.export(), o.export()):
        a, b = np.asarray(a), np.asarray(b)
        if name == "weights":
            a, b = a.view(np.uint32), b.view(np.uint32)
        assert a.shape == b.shape and np.array_equal(a, b), f"{ctx}: {name} differs"


def cycle(g, store, o, model, snap, ctx=""):
    st = g.apply_store(store, snap)
    ops = model.cycle(snap)
    rc, ost = o.apply(Batch.of(list(zip(*ops))), snap)
    assert rc == 0 and st["n_visible"] == ost["n_visible"] == len(ops[0]), ctx
    same(g, o, ctx)
    return st


def test_fig2_two_cycles_and_validity(h2):
    from test_oracle_pins import load_fig2_records
    g0, rb = load_fig2_records()
    e = np.array(g0["edges"], dtype=object)
    args = (len(g0["vertices"]), np.array(g0["vertices"], np.uint64), np.array(e[:, 0], np.uint64),
            np.array(e[:, 1], np.uint64), np.array(e[:, 2], np.float32))
    g, o = h2.Replica.from_edges(*args), O1.from_edges(*args)
    store, model = h2.DeltaStore(0, 1024), oracle.DeltaStoreModel()
    valid = rb.records[rb.records["valid"] == 1]
    w64 = rb.weights.astype(np.float64)
    store.append_records(synth.RecordBatch(valid, rb.inserts, w64, rb.deletes))
    model.append_records(valid, rb.inserts, w64, rb.deletes)
    st = cycle(g, store, o, model, 10, "ts 10")
    assert st["n_visible"] == 3
    inf = store.info()
    assert inf["n_records"] == 5 and inf["first_pending"] == 2          # x's two deltas used
    assert store.export(2, 3)["valid"].tolist() == [1, 1, 1]
    cycle(g, store, o, model, 20, "ts 20")
    assert store.info()["first_pending"] == 5
    off, cols, w, ids = g.export()
    ex = g0["expected"]
    assert ids.tolist() == ex["ext_ids"] and cols.tolist() == ex["cols"] and w.tolist() == ex["weights"]
    st = cycle(g, store, o, model, 30, "empty")
    assert st["n_visible"] == 0
    store.join()                      # no copy outstanding: returns at once
    store.close()


def test_concurrent_appenders_interleaved_visibility_chunks(h2):
    """4 producer threads append transactions (one thread per transaction, its deltas in
    order) with small chunks; cycles take snapshots in the middle of the stream, so later
    deltas wait; chunks behind the first pending delta are released."""
    n = 300
    ids = np.arange(n, dtype=np.uint64) * 3
    rng = np.random.default_rng(9)
    src, dst = ids[rng.integers(0, n, 2000)], ids[rng.integers(0, n, 2000)]
    w = rng.random(2000).astype(np.float32)
    g, o = h2.Replica.from_edges(n, ids, src, dst, w), O1.from_edges(n, ids, src, dst, w)
    store, model = h2.DeltaStore(0, 1024), oracle.DeltaStoreModel()
    ts = 0
    for k in range(6):
        b = synth.fuzz_batch(seed=41, k=k, n=6000, n_ids=3 * n + 11, probs=(0.04, 0.02, 0.6, 0.34, 0.0),
                             ts_lo=ts + 1, ts_span=400)
        b = b.slice(np.lexsort((b.src, b.ts)))
        rb = synth.records_from_ops(b)
        w64 = rb.weights.astype(np.float64) + np.where(np.arange(len(rb.weights)) % 3 == 0, 2.0 ** -27, 0.0)
        txns = np.split(np.arange(len(rb.records)), np.flatnonzero(np.diff(rb.records["ts"])) + 1)
        # the model appends in generation order; the threads interleave whole transactions
        model.append_records(rb.records, rb.inserts, w64, rb.deletes)
        def produce(part):
            for t in part:
                for i in t:
                    r = rb.records[i]
                    io, ic, do, dc = int(r["ins_off"]), int(r["ins_cnt"]), int(r["del_off"]), int(r["del_cnt"])
                    store.append(int(r["ts"]), int(r["node"]), rb.inserts[io:io + ic], w64[io:io + ic],
                                 rb.deletes[do:do + dc], bool(r["inserted"]), bool(r["deleted"]))
        parts = [txns[i::4] for i in range(4)]
        th = [threading.Thread(target=produce, args=(p,)) for p in parts]
        for t in th:
            t.start()
        for t in th:
            t.join()
        snap = ts + 250                     # the deltas with ts in (snap, ts + 400] wait
        cycle(g, store, o, model, snap, f"cycle {k}")
        ts = snap
        inf = store.info()
        pend = store.export(inf["first_pending"], inf["n_records"] - inf["first_pending"])
        assert np.all(pend["valid"][pend["ts"] <= snap] == 0) and pend["valid"][0] == 1
    cycle(g, store, o, model, ts + 1000, "drain")
    inf = store.info()
    assert inf["first_pending"] == inf["n_records"]
    assert inf["host_bytes"] < 4 * 1024 * 48 * 4                       # consumed chunks released
    store.close()


def test_stale_delta_refused_nothing_marked(h2):
    src, dst, w = synth.rmat_edges(8, 5)
    g, o = h2.Replica.from_edges(256, None, src, dst, w), O1.from_edges(256, None, src, dst, w)
    store, model = h2.DeltaStore(0, 1024), oracle.DeltaStoreModel()
    for m in (store, model):
        m.append(5, 1, inserts=[2], weights=[0.5])
    cycle(g, store, o, model, 10, "first")
    store.append(7, 3, inserts=[4], weights=[1.5])     # committed in the past: producer error (A20)
    before = g.export(checksums=True)[4]
    rc, _ = g.apply_store(store, 20, raise_on_error=False)
    assert rc == -5
    assert g.export(checksums=True)[4] == before and g.info()["snapshot_ts"] == 10
    inf = store.info()
    assert store.export(inf["first_pending"], 1)["valid"][0] == 1
    store.close()


def test_full_size_c3_stream_through_the_store(h2):
    """configs[2] (RMAT-24, 1M-op batches): three cycles from the store, each batch appended
    one cycle ahead (read-ahead overlaps the cycle); whole-export checksums equal O3 applying
    the same ops (the records expand op for op, tests/test_oracle_pins.py)."""
    from bench import Workload
    oracle.set_threads(0)
    wl = Workload("c3")
    nv, ids, src, dst, w = wl.graph()
    o3 = oracle.O3.from_edges(nv, ids, src, dst, w)
    g = h2.Replica.from_edges(nv, ids, src, dst, w)
    del src, dst, w
    store = h2.DeltaStore(0)
    batches = [wl.batch(k) for k in range(4)]
    rbs = [synth.records_from_ops(b) for b in batches]
    store.append_records(rbs[0])
    for k in range(3):
        store.append_records(rbs[k + 1])          # the next batch is committed before this cycle
        snap = int(batches[k].ts.max())
        st = g.apply_store(store, snap)
        assert st["n_visible"] == len(batches[k])
        assert o3.apply(batches[k], snap)[0] == 0
        assert g.checksums() == o3.checksums(), f"cycle {k}"
    store.close()
