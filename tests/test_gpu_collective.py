"""Collective mode (include/h2tap.h: the library owns an NCCL communicator; SURVEY.md §8(b)
"every multi-GPU call is collective", §8(e)).  Only one GPU exists here and NCCL refuses two
ranks on one device, so this runs the library's collective path at world = 1: the slice
validation, the count all-gather, the route packing, the grouped send/recv exchange, the
two-phase status agreement and the collective BFS / SSSP / PageRank all execute through NCCL,
and the replica must stay bit-exact with O1 (and with an ordinary replica) after every batch.
The multi-rank protocol it implements is the one sharded.py runs over gloo (world 2/3, CPU
tests) and over 2 processes on one GPU (tests/test_gpu_sharded_mp.py)."""
import numpy as np
import pytest

import oracle
import synth
from oracle import O1

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def h2():
    import torch  # noqa: F401  (the process's NCCL is torch's)
    import paper_conf_edbt_jibrilabs23_b200 as h2
    return h2


def same(g, o, ctx):
    for n, a, b in zip(("offsets", "cols", "weights", "ext_ids"), g.export(), o.export()):
        a, b = np.asarray(a), np.asarray(b)
        if n == "weights":
            a, b = a.view(np.uint32), b.view(np.uint32)
        assert a.shape == b.shape and np.array_equal(a, b), f"{ctx}: {n}"


def test_collective_world1_ldbc_stream_and_checks(h2):
    shape = synth.LdbcShape(n_person=512, n_msg=20000, e_person=40000)
    seed = synth.seed_of("c2")
    ids = synth.ldbc_vertices(shape)
    src, dst, w = synth.ldbc_edges(shape, seed)
    nid = h2.nccl_unique_id()
    assert len(nid) == h2.NCCL_ID_BYTES
    g = h2.Replica.from_edges(shape.n_vertices, ids, src, dst, w, nccl_id=nid)
    plain = h2.Replica.from_edges(shape.n_vertices, ids, src, dst, w)
    o = O1.from_edges(shape.n_vertices, ids, src, dst, w)
    ts, seq = 0, 0
    for k in range(4):
        b = synth.ldbc_batch(shape, seed, k, 6000, lodeg=(k == 2), ts_base=ts)
        ts = int(b.ts.max())
        st = g.apply(b, ts)                       # this rank's slice = the whole batch
        plain.apply(b, ts)
        rc, ost = o.apply(b, ts)
        assert rc == 0 and st["n_visible"] == ost["n_visible"]
        same(g, o, f"collective batch {k}")
        seq += len(b)
        cs = g.collective_stats()
        assert cs["global_seq"] == seq and cs["route_bytes"] == 0   # world 1: nothing leaves
        inf = g.info()
        assert inf["shard_vertex_base"] == 0 and inf["shard_edge_base"] == 0
    off, cols, ww, ext = g.export()
    for d in (0, len(ext) // 2):
        assert np.array_equal(g.bfs(int(ext[d])), oracle.bfs(off, cols, d))
        assert np.array_equal(g.sssp(int(ext[d])), oracle.sssp(off, cols, ww, d))
    pr, ref = g.pagerank(), oracle.pagerank(off, cols)
    assert np.max(np.abs(pr - ref) / np.maximum(ref, 1e-300)) <= 1e-6
    assert np.array_equal(g.bfs(int(ext[3])), plain.bfs(int(ext[3])))


def test_collective_agreed_refusal_and_no_prepare(h2):
    n = 1 << 10
    src, dst, w = synth.rmat_edges(10, 3, n=8 * n)
    g = h2.Replica.from_edges(n, None, src, dst, w, nccl_id=h2.nccl_unique_id())
    b = synth.rmat_batch(10, 3, 0, 500, len(src))
    snap = int(b.ts.max())
    g.apply(b, snap)
    before = g.export(checksums=True)[4]
    stale = synth.rmat_batch(10, 3, 1, 200, len(src))
    stale.ts[:] = 1                               # <= the snapshot: every rank refuses
    rc, _ = g.apply(stale, snap + 5, raise_on_error=False)
    assert rc == -5
    assert g.export(checksums=True)[4] == before and g.info()["snapshot_ts"] == snap
    rc, _ = g.prepare(b, snap + 10)               # the collective call agrees and swaps itself
    assert rc == -1
    b2 = synth.rmat_batch(10, 3, 2, 300, len(src))
    b2.ts += snap
    g.apply(b2, int(b2.ts.max()))                 # still usable after both refusals
    o = O1.from_edges(n, None, src, dst, w)
    o.apply(b, snap)
    o.apply(b2, int(b2.ts.max()))
    same(g, o, "after refusals")
