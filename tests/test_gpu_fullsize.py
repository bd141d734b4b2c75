"""Full-size parity (BASELINE.json configs[1] and [2], the sizes bench.py times).

At full size the oracle cannot replay the whole graph in seconds, so:
* sampled rows: a row's result depends only on its old row, the edge ops from its
  vertex and the node ops of its vertex and of the vertices it points to (cascades
  remove in-edges of deleted vertices from the row itself).  O1 replays exactly that
  sub-problem for a sample of rows (hubs, random rows, rows of node-op vertices)
  and the GPU rows are compared bit-exactly in external-ID space;
* whole-replica invariants at any size: monotone offsets, strictly increasing
  rows, cols < V', strictly increasing ext_ids, I6 (E' = E + NEW - DEL - CASC),
  and the live vertex set equals the replay of the node ops over the old set.
"""
import numpy as np
import pytest

import synth
from oracle import O1

pytestmark = [pytest.mark.gpu, pytest.mark.slow, pytest.mark.timeout(600)]


@pytest.fixture(scope="module")
def h2():
    import paper_conf_edbt_jibrilabs23_b200 as h2
    return h2


def check_invariants(off, cols, ids):
    V = len(ids)
    assert off[0] == 0 and off[-1] == len(cols)
    d = np.diff(off)
    assert np.all(d >= 0)
    if len(cols):
        assert int(cols.max()) < V
        starts = np.zeros(len(cols), bool)
        starts[off[:-1][d > 0]] = True
        inc = np.diff(cols.astype(np.int64)) > 0
        assert np.all(inc | starts[1:]), "row not strictly increasing"
    assert np.all(np.diff(ids) > 0)


def rows_ext(off, cols, w, ids, rows_dense):
    """{ext u: (ext dst array, weight bits)} for the given dense rows."""
    out = {}
    for u in rows_dense:
        a, b = off[u], off[u + 1]
        out[int(ids[u])] = (ids[cols[a:b]], w[a:b].view(np.uint32))
    return out


def sub_oracle(old, batch, sample_ext, snap, create_ts=0):
    """O1 on the sub-problem that determines the sampled rows."""
    off, cols, w, ids = old
    sample_ext = np.asarray(sample_ext, np.uint64)
    k = np.searchsorted(ids, sample_ext)
    kc = np.minimum(k, len(ids) - 1)
    present = ids[kc] == sample_ext
    es, ed, ew = [], [], []
    for u, kk in zip(sample_ext[present], kc[present]):
        a, b = off[kk], off[kk + 1]
        es.append(np.full(b - a, u, np.uint64)); ed.append(ids[cols[a:b]]); ew.append(w[a:b])
    es = np.concatenate(es) if es else np.array([], np.uint64)
    ed = np.concatenate(ed) if ed else np.array([], np.uint64)
    ew = np.concatenate(ew) if ew else np.array([], np.float32)
    node = batch.kind <= 1
    sel = node | np.isin(batch.src, sample_ext)
    sub = batch.slice(np.nonzero(sel)[0])
    vv = np.unique(np.concatenate([sample_ext, ed, sub.src, sub.dst[sub.kind >= 2]]))
    kk = np.minimum(np.searchsorted(ids, vv), len(ids) - 1)
    old_live = vv[ids[kk] == vv]
    o = O1.from_edges(len(old_live), old_live, es, ed, ew, create_ts)
    rc, _ = o.apply(sub, snap)
    assert rc == 0
    return o.export()


def final_live_set(old_ids, batch):
    """Replay of visible node ops (ts, seq order) over the old vertex set."""
    node = np.nonzero(batch.kind <= 1)[0]
    order = node[np.lexsort((node, batch.ts[node]))]
    live = {}
    for i in order:
        live[int(batch.src[i])] = batch.kind[i] == 0
    dead = np.array(sorted(v for v, l in live.items() if not l), np.uint64)
    born = np.array(sorted(v for v, l in live.items() if l), np.uint64)
    return np.union1d(old_ids[~np.isin(old_ids, dead)], born).astype(np.uint64)


def run_config(h2, name, n_sample=3000, records=False, tombstone=False):
    cfg = synth.CONFIGS[name]
    seed = synth.seed_of(name)
    if cfg["kind"] == "ldbc":
        shape = cfg["shape"]
        ids = synth.ldbc_vertices(shape)
        src, dst, w = synth.ldbc_edges(shape, seed)
        nv = shape.n_vertices
        batch = synth.ldbc_batch(shape, seed, 0, cfg["batch"])
    else:
        nv = 1 << cfg["scale"]
        ids = None
        src, dst, w = synth.rmat_edges(cfg["scale"], seed)
        batch = synth.rmat_batch(cfg["scale"], seed, 0, cfg["batch"], len(src), p_insert=cfg["p_insert"])
    g = h2.Replica.from_edges(nv, ids, src, dst, w, tombstone=tombstone)
    del src, dst, w
    old = g.export()
    snap = int(batch.ts.max())
    st = g.apply_records(synth.records_from_ops(batch), snap) if records else g.apply(batch, snap)
    new = g.export()
    off, cols, wn, ids_new = new
    check_invariants(off, cols, ids_new)
    assert len(cols) == len(old[1]) + st["n_new"] - st["n_del"] - st["n_casc"]       # I6
    live_set = final_live_set(old[3], batch)
    if tombstone:  # reading A23: old slots stay, the live flags say who is alive
        assert np.array_equal(ids_new, np.union1d(old[3], live_set))
        live = g.live()
        assert np.array_equal(live == 1, np.isin(ids_new, live_set))
        assert np.all(np.diff(off)[live == 0] == 0)                                # empty rows
    else:
        assert np.array_equal(ids_new, live_set)                                    # ID map
    # sample: the most-updated sources, random old rows, node-op vertices
    rng = np.random.default_rng(7)
    edge_src = batch.src[batch.kind >= 2]
    u, c = np.unique(edge_src, return_counts=True)
    rand = old[3][rng.integers(0, len(old[3]), n_sample)]
    nodev = np.unique(batch.src[batch.kind <= 1])
    cand = np.concatenate([rand, nodev[rng.permutation(len(nodev))[:300]], u[np.argsort(-c)[:200]]])
    # keep the sub-problem small: rows up to 100K old edges, 3M old edges in total
    k = np.minimum(np.searchsorted(old[3], cand), len(old[3]) - 1)
    deg = np.where(old[3][k] == cand, old[0][k + 1] - old[0][k], 0)
    deg = np.where(deg > 100_000, 0, deg)
    keep = (np.cumsum(deg) <= 3_000_000) & (np.where(old[3][k] == cand, old[0][k + 1] - old[0][k], 0) <= 100_000)
    sample = np.unique(cand[keep])
    ref = sub_oracle(old, batch, sample, snap)
    ref_rows = rows_ext(ref[0], ref[1], ref[2], ref[3], np.nonzero(np.isin(ref[3], sample))[0])
    checked = 0
    for v, (rd, rw) in ref_rows.items():
        k = int(np.searchsorted(ids_new, np.uint64(v)))
        assert k < len(ids_new) and int(ids_new[k]) == v, f"{name}: live vertex {v} missing" 
        a, b = off[k], off[k + 1]
        assert np.array_equal(ids_new[cols[a:b]], rd), f"{name}: row {v} columns differ"
        assert np.array_equal(wn[a:b].view(np.uint32), rw), f"{name}: row {v} weights differ"
        checked += 1
    # sampled vertices the oracle says are dead must be absent on the GPU too
    dead = set(int(s) for s in sample) - set(ref_rows)
    if tombstone:
        dk = np.isin(ids_new, np.array(sorted(dead), np.uint64)) if dead else np.zeros(len(ids_new), bool)
        assert np.all(g.live()[dk] == 0)
    else:
        live_gpu = set(int(x) for x in ids_new[np.isin(ids_new, np.array(sorted(dead), np.uint64))]) if dead else set()
        assert not live_gpu
    assert checked > 1000
    return st


def test_c3_rmat24_full_size(h2):
    st = run_config(h2, "c3")
    assert st["n_visible"] == synth.CONFIGS["c3"]["batch"]


def test_c2_ldbc_sf10_full_size(h2):
    st = run_config(h2, "c2")
    assert st["n_vertex_inserted"] > 0 and st["n_vertex_deleted"] > 0 and st["n_casc"] > 0


def test_c2_full_size_records_input(h2):
    """configs[1] through h2tap_delta_apply_records (the paper's delta-record layout)"""
    st = run_config(h2, "c2", records=True)
    assert st["n_vertex_inserted"] > 0 and st["n_casc"] > 0


def test_c2_full_size_tombstone_rows(h2):
    """configs[1] on a tombstone-row replica (reading A23)"""
    st = run_config(h2, "c2", tombstone=True)
    assert st["n_vertex_deleted"] > 0
