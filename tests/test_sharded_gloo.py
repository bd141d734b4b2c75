"""Multi-process sharded apply over gloo (CPU; world_size 2 and 3).

Exercises the exchange protocol of paper_conf_edbt_jibrilabs23_b200.sharded (status
agreement, rank-major arrival numbers, routing of edge ops to the owner of their
source and of node ops to every shard, variable all-to-all, two-phase prepare /
agree / commit-or-abort, shard bases) with an oracle-backed shard engine standing in
for the GPU replica.  The shards' rows, gathered in shard order, must equal the
unsharded oracle after every batch; a prepare failure injected on ONE rank must leave
every shard unchanged (no rank commits), and the next batch must apply normally.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

REC = np.dtype([("src", "<u8"), ("dst", "<u8"), ("ts", "<u8"), ("seq", "<u8"), ("w", "<f4"),
                ("kind", "u1"), ("pad", "u1", 3)])
assert REC.itemsize == 40


class OracleShard:
    """Test double for LibEngine: O1 over the global vertex set with this shard's rows."""

    def __init__(self, n, ids, src, dst, w, bounds, rank):
        from oracle import O1
        self.bounds, self.rank, self.P = bounds, rank, len(bounds) - 1
        self.snap = 0
        mine = self.owner(src) == rank
        self.o = O1.from_edges(n, ids, src[mine], dst[mine], w[mine])

    def owner(self, x):
        return np.searchsorted(self.bounds[1:self.P], np.asarray(x, np.uint64), side="right")

    def validate(self, b):
        if len(b.kind) and int(b.kind.max()) > 4:
            return -1
        if len(b.kind) and int(b.ts.min()) <= self.snap:
            return -5
        return 0

    def pack(self, b, seq0):
        n = len(b.kind)
        own = np.where(b.kind <= 1, -1, self.owner(b.src))
        parts, counts = [], []
        for d in range(self.P):
            sel = np.nonzero((own == -1) | (own == d))[0]
            r = np.zeros(len(sel), REC)
            r["src"], r["dst"], r["ts"] = b.src[sel], b.dst[sel], b.ts[sel]
            r["seq"] = seq0 + sel.astype(np.uint64)
            r["w"], r["kind"] = b.w[sel], b.kind[sel]
            parts.append(r)
            counts.append(len(sel))
        buf = np.concatenate(parts) if n else np.zeros(0, REC)
        return torch.from_numpy(buf.view(np.uint8).copy()), counts

    def route_count(self, b):
        own = np.where(b.kind <= 1, -1, self.owner(b.src))
        return [int(np.count_nonzero((own == -1) | (own == d))) for d in range(self.P)]

    fail_next = False   # inject a prepare failure (as if the GPU ran out of memory)
    prepared = None

    def prepare_routed(self, recs, n, snap):
        from synth import Batch
        r = recs.numpy().view(REC)
        assert len(r) == n and (n < 2 or np.all(np.diff(r["seq"].astype(np.int64)) > 0))
        assert self.prepared is None
        if self.fail_next:
            self.fail_next = False
            return -2, {}
        self.prepared = (Batch(r["kind"].copy(), r["src"].copy(), r["dst"].copy(), r["w"].copy(),
                               r["ts"].copy()), snap)
        return 0, {"n_visible": n}

    def commit(self):
        b, snap = self.prepared
        self.prepared = None
        rc, st = self.o.apply(b, snap)
        assert rc == 0
        self.snap = snap

    def abort(self):
        assert self.prepared is not None
        self.prepared = None

    def own_rows(self):
        off, cols, w, ids = self.o.export()
        rows = np.nonzero(self.owner(ids) == self.rank)[0]
        lo = int(rows[0]) if len(rows) else int(np.searchsorted(self.owner(ids), self.rank))
        hi = lo + len(rows)
        return off[lo:hi + 1] - off[lo], cols[off[lo]:off[hi]], w[off[lo]:off[hi]], ids[lo:hi], lo

    def local_sizes(self):
        off, cols, w, ids, lo = self.own_rows()
        return len(ids), len(cols), lo

    # one shard's part of a check step, plain numpy on CPU tensors (in place)
    def lookup(self, x):
        ids = self.o.export()[3]
        k = int(np.searchsorted(ids, np.uint64(x)))
        assert k < len(ids) and ids[k] == x
        return k

    def _rows(self):
        off, cols, w, ids, lo = self.own_rows()
        for i in range(len(ids)):
            yield lo + i, cols[off[i]:off[i + 1]], w[off[i]:off[i + 1]]

    def bfs_expand(self, level, depth, mark):
        lv, mk = level.numpy(), mark.numpy()
        for u, cs, _ in self._rows():
            if lv[u] == depth:
                for v in cs:
                    if lv[v] < 0:
                        mk[v] = 1

    def bfs_settle(self, level, mark, depth):
        lv, mk = level.numpy(), mark.numpy()
        new = (mk == 1) & (lv < 0)
        lv[new] = depth + 1
        return int(new.sum())

    def pr_push(self, pr, acc, dang):
        p, a, d = pr.numpy(), acc.numpy(), dang.numpy()
        for u, cs, _ in self._rows():
            if len(cs) == 0:
                d[0] += p[u]
            for v in cs:
                a[v] += p[u] / len(cs)

    def pr_finish(self, acc, dang, damping):
        a, V = acc.numpy(), len(acc)
        a[:] = (1 - damping) / V + damping * (a + dang.numpy()[0] / V)

    def check_weights(self):
        return int(any((ws < 0).any() or np.isnan(ws).any() for _, _, ws in self._rows()))

    def sssp_relax(self, frontier, dist_, nd):
        f, d, n = frontier.numpy(), dist_.numpy(), nd.numpy()
        for u, cs, ws in self._rows():
            if f[u]:
                for v, x in zip(cs, ws):
                    n[v] = min(n[v], d[u] + float(x))

    def sssp_settle(self, dist_, nd, frontier):
        d, n, f = dist_.numpy(), nd.numpy(), frontier.numpy()
        ch = n < d
        f[:] = ch
        d[ch] = n[ch]
        return int(ch.sum())


def _worker(rank, world, port, out):
    os.environ["MASTER_ADDR"], os.environ["MASTER_PORT"] = "127.0.0.1", str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        from paper_conf_edbt_jibrilabs23_b200.sharded import ShardedReplica
        from paper_conf_edbt_jibrilabs23_b200 import H2tapError, balanced_bounds

        n = 400
        ids = np.arange(n, dtype=np.uint64) * 5 + 2
        rng = np.random.default_rng(3)
        src, dst = ids[rng.integers(0, n, 3000)], ids[rng.integers(0, n, 3000)]
        w = rng.random(3000).astype(np.float32)
        bounds = balanced_bounds(src, world)
        sh = ShardedReplica(OracleShard(n, ids, src, dst, w, bounds, rank), rank, world, "cpu")
        results, ts = [], 0
        for k in range(4):
            g = synth.fuzz_batch(seed=11, k=k, n=1200, n_ids=5 * n + 9, probs=(0.05, 0.03, 0.5, 0.25, 0.17),
                                 ts_lo=ts + 1, ts_span=300)
            hit = np.arange(len(g)) % 2 == 0
            g.src[hit], g.dst[hit] = ids[g.src[hit] % n], ids[g.dst[hit] % n]
            sl = g.slice(slice(rank * len(g) // world, (rank + 1) * len(g) // world))  # rank-major slices
            st = sh.apply(sl, ts + 250)
            assert st["global_batch"] == len(g)
            off, cols, ww, own_ids, lo = sh.engine.own_rows()
            results.append((off, cols, ww, own_ids, sh.bases()))
            ts += 300
        # a prepare failure on the last rank only: nobody commits, every shard unchanged
        before = sh.engine.own_rows()
        g = synth.fuzz_batch(seed=12, k=0, n=600, n_ids=5 * n + 9, ts_lo=ts + 1, ts_span=50)
        sl = g.slice(slice(rank * len(g) // world, (rank + 1) * len(g) // world))
        sh.engine.fail_next = rank == world - 1
        try:
            sh.apply(sl, ts + 40)
            aborted = False
        except H2tapError as e:
            aborted = e.status == -2
        after = sh.engine.own_rows()
        aborted = aborted and all(np.array_equal(np.asarray(a), np.asarray(b)) for a, b in zip(before, after))
        aborted = aborted and sh.engine.prepared is None
        # a stale op on one rank must make every rank refuse the batch
        from synth import Batch
        bad = Batch.of([(2, int(ids[0]), int(ids[1]), 1.0, 5 if rank == world - 1 else ts + 10)])
        try:
            sh.apply(bad, ts + 20)
            refused = False
        except H2tapError as e:
            refused = e.status == -5
        # freshness checks through the sharded orchestration (one collective per step)
        src0 = int(sh.engine.o.export()[3][0])
        checks = (src0, sh.bfs(src0).numpy().copy(), sh.sssp(src0).numpy().copy(), sh.pagerank(0.85, 20).numpy().copy())
        gathered = [None] * world
        dist.all_gather_object(gathered, (results, refused and aborted, checks))
        if rank == 0:
            out.put(gathered)
    finally:
        dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_exchange_over_gloo(world):
    import synth
    from oracle import O1
    from paper_conf_edbt_jibrilabs23_b200 import balanced_bounds  # noqa: F401 (library loads on CPU)

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    gathered = q.get(timeout=240)
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    # global reference
    n = 400
    ids = np.arange(n, dtype=np.uint64) * 5 + 2
    rng = np.random.default_rng(3)
    src, dst = ids[rng.integers(0, n, 3000)], ids[rng.integers(0, n, 3000)]
    w = rng.random(3000).astype(np.float32)
    o = O1.from_edges(n, ids, src, dst, w)
    ts = 0
    for k in range(4):
        g = synth.fuzz_batch(seed=11, k=k, n=1200, n_ids=5 * n + 9, probs=(0.05, 0.03, 0.5, 0.25, 0.17),
                             ts_lo=ts + 1, ts_span=300)
        hit = np.arange(len(g)) % 2 == 0
        g.src[hit], g.dst[hit] = ids[g.src[hit] % n], ids[g.dst[hit] % n]
        rc, _ = o.apply(g, ts + 250)
        assert rc == 0
        off, cols, ww, gid = o.export()
        parts = [gathered[r][0][k] for r in range(world)]
        # shard bases are consistent with the concatenation
        row_base = np.cumsum([0] + [len(p[3]) for p in parts])[:-1]
        edge_base = np.cumsum([0] + [len(p[1]) for p in parts])[:-1]
        assert [p[4][0] for p in parts] == list(row_base)
        assert [p[4][1] for p in parts] == list(edge_base)
        cat_off = np.concatenate([p[0][:-1] + eb for p, eb in zip(parts, edge_base)] + [np.array([len(cols)])])
        assert np.array_equal(np.concatenate([p[3] for p in parts]), gid)
        assert np.array_equal(cat_off, off)
        assert np.array_equal(np.concatenate([p[1] for p in parts]), cols)
        assert np.array_equal(np.concatenate([p[2] for p in parts]).view(np.uint32), ww.view(np.uint32))
        ts += 300
    assert all(gathered[r][1] for r in range(world))  # every rank aborted / refused the bad batches
    import oracle
    src0, lv, dd, pr = gathered[0][2]
    for r in range(1, world):
        assert all(np.array_equal(a, b) for a, b in zip(gathered[r][2][1:], (lv, dd, pr)))
    d0 = int(np.searchsorted(gid, np.uint64(src0)))
    assert np.array_equal(lv, oracle.bfs(off, cols, d0))
    assert np.array_equal(dd, oracle.sssp(off, cols, ww, d0))
    ref = oracle.pagerank(off, cols, 0.85, 20)
    assert np.max(np.abs(pr - ref) / ref) < 1e-9
