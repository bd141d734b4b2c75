"""Vertex-range sharding — several shards of one graph on one GPU.

The host routes ops the way the exchange step does (edge ops to the shard owning
their source, node ops to every shard, global rank-major arrival numbers); the
shards' exports, concatenated in shard order with their edge bases, must equal the
unsharded oracle bit-exactly after every batch.
"""
import numpy as np
import pytest

import synth
from oracle import O1
from synth import Batch

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def h2():
    import paper_conf_edbt_jibrilabs23_b200 as h2
    return h2


def route(batch: Batch, seq0: int, bounds: np.ndarray, p: int):
    """Ops for shard p: node ops (all shards) + edge ops whose source p owns; explicit seq."""
    seq = np.arange(seq0, seq0 + len(batch), dtype=np.uint64)
    hi = bounds[p + 1] if p + 1 < len(bounds) - 1 else np.iinfo(np.uint64).max
    own = (batch.src >= bounds[p]) & ((batch.src < hi) | (p + 1 == len(bounds) - 1))
    sel = (batch.kind <= 1) | own
    b = batch.slice(np.nonzero(sel)[0])
    b.seq = seq[sel]
    return b


def gather(shards):
    offs, cols, ws, ids = [], [], [], []
    base = 0
    for g in shards:
        o, c, w, i = g.export()
        offs.append(o[:-1] + base)
        base += int(o[-1])
        cols.append(c); ws.append(w); ids.append(i)
    return (np.concatenate(offs + [np.array([base], np.int64)]), np.concatenate(cols),
            np.concatenate(ws), np.concatenate(ids))


def assert_same(a, b, ctx):
    for n, x, y in zip(("offsets", "cols", "weights", "ext_ids"), a, b):
        x, y = np.asarray(x), np.asarray(y)
        if n == "weights":
            x, y = x.view(np.uint32), y.view(np.uint32)
        assert x.shape == y.shape and np.array_equal(x, y), f"{ctx}: {n} differs"


def run(h2, P, n_vertices, ids, src, dst, w, batches, bounds):
    o = O1.from_edges(n_vertices, ids, src, dst, w)
    shards = []
    for p in range(P):
        hi = bounds[p + 1] if p + 1 < P else np.iinfo(np.uint64).max
        mine = (src >= bounds[p]) & ((src < hi) | (p == P - 1))
        shards.append(h2.Replica.from_edges(n_vertices, ids, src[mine], dst[mine], w[mine],
                                            rank=p, world=P, shard_bounds=bounds))
    assert_same(gather(shards), o.export(), f"P={P} create")
    seq0 = 0
    for k, (b, snap) in enumerate(batches):
        for p in range(P):
            shards[p].apply(route(b, seq0, bounds, p), snap)
        seq0 += len(b)
        rc, _ = o.apply(b, snap)
        assert rc == 0
        assert_same(gather(shards), o.export(), f"P={P} batch {k}")
    bases = [g.info()["shard_vertex_base"] for g in shards]
    assert bases == sorted(bases) and bases[0] == 0


@pytest.mark.parametrize("P", [2, 3, 5])
def test_sharded_rmat_edges_and_deferral(h2, P):
    scale = 12
    src, dst, w = synth.rmat_edges(scale, 40 + P)
    n = 1 << scale
    bounds = h2.balanced_bounds(src, P)
    batches, ts = [], 0
    for k in range(3):
        b = synth.rmat_batch(scale, 40 + P, k, 6000, len(src), p_insert=0.6, p_weight=0.1,
                             p_repeat=0.2, ops_per_txn=3, ts_base=ts)
        ts = int(b.ts.max())
        batches.append((b, int(np.quantile(b.ts, 0.9))))
    batches.append((Batch.empty(0), ts))
    run(h2, P, n, None, src, dst, w, batches, bounds)


@pytest.mark.parametrize("P", [2, 4])
def test_sharded_node_ops_ldbc(h2, P):
    shape = synth.LdbcShape(n_person=512, n_msg=20000, e_person=40000)
    seed = synth.seed_of("c2") + P
    ids = synth.ldbc_vertices(shape)
    src, dst, w = synth.ldbc_edges(shape, seed)
    bounds = h2.balanced_bounds(src, P)
    batches, ts = [], 0
    for k in range(3):
        b = synth.ldbc_batch(shape, seed, k, 4000, ts_base=ts)
        ts = int(b.ts.max())
        batches.append((b, ts))
    run(h2, P, shape.n_vertices, ids, src, dst, w, batches, bounds)


def test_sharded_fuzz_node_ops_every_kind(h2):
    """Sparse external ids, node inserts/deletes anywhere (ids move between shard row ranges)."""
    P = 3
    n = 600
    ids = (np.arange(n, dtype=np.uint64) * 7 + 3)
    rng = np.random.default_rng(5)
    src = ids[rng.integers(0, n, 4000)]
    dst = ids[rng.integers(0, n, 4000)]
    w = rng.random(4000).astype(np.float32)
    bounds = np.array([0, 7 * 200, 7 * 400, np.iinfo(np.uint64).max], np.uint64)
    batches, ts = [], 0
    for k in range(4):
        b = synth.fuzz_batch(seed=77, k=k, n=3000, n_ids=7 * n + 10, probs=(0.05, 0.03, 0.5, 0.25, 0.17),
                             ts_lo=ts + 1, ts_span=500)
        hit = np.arange(len(b)) % 2 == 0
        b.src[hit] = ids[b.src[hit] % n]
        b.dst[hit] = ids[b.dst[hit] % n]
        batches.append((b, ts + 400))
        ts += 500
    run(h2, P, n, ids, src, dst, w, batches, bounds)


def test_wrong_shard_is_rejected(h2):
    src, dst, w = synth.rmat_edges(8, 1)
    bounds = np.array([0, 128, np.iinfo(np.uint64).max], np.uint64)
    g = h2.Replica.from_edges(256, None, src[src < 128], dst[src < 128], w[src < 128], rank=0, world=2,
                              shard_bounds=bounds)
    bad = Batch.of([(synth.EDGE_INSERT, 200, 3, 1.0, 5)])
    bad.seq = np.array([0], np.uint64)
    with pytest.raises(h2.H2tapError):
        g.apply(bad, 5)


# ------------------------------------------------------- library routing (a8)
REC = np.dtype([("src", "<u8"), ("dst", "<u8"), ("ts", "<u8"), ("seq", "<u8"), ("w", "<f4"),
                ("kind", "u1"), ("pad", "u1", 3)])


def np_pack(b: Batch, seq0: int, bounds: np.ndarray):
    """Independent host routing: per destination, node ops + owned edge ops, in op order."""
    P = len(bounds) - 1
    own = np.searchsorted(bounds[1:P], b.src, side="right")
    out = []
    for d in range(P):
        sel = np.nonzero((b.kind <= 1) | (own == d))[0]
        r = np.zeros(len(sel), REC)
        r["src"], r["dst"], r["ts"], r["seq"] = b.src[sel], b.dst[sel], b.ts[sel], seq0 + sel.astype(np.uint64)
        r["w"], r["kind"] = b.w[sel], b.kind[sel]
        out.append(r)
    return out


def to_dev(b: Batch):
    import torch
    return Batch(*(torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a).cuda()
                   for a in (b.kind, b.src, b.dst, b.w, b.ts)))


@pytest.mark.parametrize("P", [2, 3])
def test_routed_pack_and_apply(h2, P):
    """h2tap_route_pack on every source rank's slice (bit-exact against host routing),
    the all-to-all emulated by concatenating segments in source-rank order, then
    h2tap_delta_apply_routed on every shard; gathered shards == unsharded oracle."""
    from paper_conf_edbt_jibrilabs23_b200.sharded import LibEngine
    n = 700
    ids = np.arange(n, dtype=np.uint64) * 3 + 1
    rng = np.random.default_rng(9 + P)
    src, dst = ids[rng.integers(0, n, 5000)], ids[rng.integers(0, n, 5000)]
    w = rng.random(5000).astype(np.float32)
    bounds = h2.balanced_bounds(src, P)
    o = O1.from_edges(n, ids, src, dst, w)
    shards = []
    for p in range(P):
        mine = np.searchsorted(bounds[1:P], src, side="right") == p
        shards.append(h2.Replica.from_edges(n, ids, src[mine], dst[mine], w[mine], rank=p, world=P,
                                            shard_bounds=bounds))
    eng = [LibEngine(s, "cuda:0") for s in shards]
    ts, seq = 0, 0
    for k in range(4):
        g = synth.fuzz_batch(seed=21, k=k, n=3000 + 517 * k, n_ids=3 * n + 5, probs=(0.05, 0.03, 0.5, 0.25, 0.17),
                             ts_lo=ts + 1, ts_span=400)
        hit = np.arange(len(g)) % 3 != 0
        g.src[hit], g.dst[hit] = ids[g.src[hit] % n], ids[g.dst[hit] % n]
        snap = ts + 300
        inbox = [[] for _ in range(P)]
        for p in range(P):
            lo, hi = p * len(g) // P, (p + 1) * len(g) // P
            sl = g.slice(slice(lo, hi))
            assert eng[p].validate(to_dev(sl)) == 0
            recs, counts = eng[p].pack(to_dev(sl), seq + lo)
            host = recs.cpu().numpy()
            want = np_pack(sl, seq + lo, bounds)
            assert counts == [len(x) for x in want]
            off = 0
            for d in range(P):
                seg = host[off * 40:(off + counts[d]) * 40]
                assert np.array_equal(seg, want[d].view(np.uint8)), f"batch {k} src {p} dst {d}: records differ"
                inbox[d].append(recs[off * 40:(off + counts[d]) * 40])
                off += counts[d]
        import torch
        for d in range(P):
            recv = torch.cat(inbox[d]) if inbox[d] else torch.empty(0, dtype=torch.uint8, device="cuda")
            eng[d].apply_routed(recv, recv.numel() // 40, snap)
        seq += len(g)
        rc, _ = o.apply(g, snap)
        assert rc == 0
        assert_same(gather(shards), o.export(), f"routed P={P} batch {k}")
        ts += 400
    # a stale op is reported by validate (before anything is applied)
    stale = Batch.of([(synth.EDGE_INSERT, int(ids[0]), int(ids[1]), 1.0, 3)])
    assert h2.STATUS[eng[0].validate(to_dev(stale))] == "E_STALE_TS"


def test_sharded_checks_logical_shards(h2):
    """BFS / SSSP / PageRank over P = 3 shards through the per-shard C-ABI steps, the
    collectives emulated on the host (MAX / SUM / MIN across shards)."""
    import torch
    import oracle
    P = 3
    n = 1 << 11
    src, dst, w = synth.rmat_edges(11, 17, n=10 * n)
    ids = np.arange(n, dtype=np.uint64) * 7 + 3
    src, dst = ids[src], ids[dst]
    bounds = h2.balanced_bounds(src, P)
    own = np.searchsorted(bounds[1:P], src, side="right")
    shards = [h2.Replica.from_edges(n, ids, src[own == p], dst[own == p], w[own == p], rank=p, world=P,
                                    shard_bounds=bounds) for p in range(P)]
    off, cols, ww, gid = O1.from_edges(n, ids, src, dst, w).export()
    dev = torch.device("cuda")
    s_ext = int(gid[int(np.argmax(np.diff(off)))])
    s = shards[0].lookup(s_ext)
    assert all(g.lookup(s_ext) == s for g in shards)
    # BFS
    level = torch.full((n,), -1, dtype=torch.int32, device=dev)
    level[s] = 0
    depth = 0
    while True:
        marks = [torch.zeros(n, dtype=torch.uint8, device=dev) for _ in shards]
        for g, m in zip(shards, marks):
            g.shard_bfs_expand(level, depth, m)
        mark = torch.stack(marks).amax(0)
        if shards[0].shard_bfs_settle(level, mark, depth) == 0:
            break
        depth += 1
    assert np.array_equal(level.cpu().numpy(), oracle.bfs(off, cols, s))
    # PageRank
    pr = torch.full((n,), 1.0 / n, dtype=torch.float64, device=dev)
    for _ in range(20):
        accs = [torch.zeros(n, dtype=torch.float64, device=dev) for _ in shards]
        dangs = [torch.zeros(1, dtype=torch.float64, device=dev) for _ in shards]
        for g, a, d in zip(shards, accs, dangs):
            g.shard_pr_push(pr, a, d)
        acc, dang = torch.stack(accs).sum(0), torch.stack(dangs).sum(0)
        shards[0].shard_pr_finish(acc, dang, 0.85)
        pr = acc
    ref = oracle.pagerank(off, cols, 0.85, 20)
    assert np.max(np.abs(pr.cpu().numpy() - ref) / ref) < 1e-6
    # SSSP
    assert all(g.shard_check_weights() == 0 for g in shards)
    d = torch.full((n,), float("inf"), dtype=torch.float64, device=dev)
    d[s] = 0.0
    fr = torch.zeros(n, dtype=torch.uint8, device=dev)
    fr[s] = 1
    while True:
        nds = [d.clone() for _ in shards]
        for g, x in zip(shards, nds):
            g.shard_sssp_relax(fr, d, x)
        nd = torch.stack(nds).amin(0)
        if shards[0].shard_sssp_settle(d, nd, fr) == 0:
            break
    assert np.array_equal(d.cpu().numpy(), oracle.sssp(off, cols, ww, s))
