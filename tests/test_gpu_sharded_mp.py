"""Two processes, one shard each, on one GPU: the complete sharded path
(ShardedReplica + LibEngine: validate, status agreement, rank-major numbering,
h2tap_route_pack, all-to-all, h2tap_delta_apply_routed) over a gloo group.  The
shards' exports, gathered in rank order, must equal the unsharded oracle bit-exactly
after every batch.  (NCCL refuses two ranks on one device; the protocol code is the
same, only the collectives' transport differs.)"""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _worker(rank, world, port, q, exchange="alltoall"):
    os.environ["MASTER_ADDR"], os.environ["MASTER_PORT"] = "127.0.0.1", str(port)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        import paper_conf_edbt_jibrilabs23_b200 as h2
        from paper_conf_edbt_jibrilabs23_b200.sharded import LibEngine, ShardedReplica
        torch.cuda.set_device(0)
        shape = synth.LdbcShape(n_person=300, n_msg=12000, e_person=20000)
        seed = synth.seed_of("c2") + 99
        ids = synth.ldbc_vertices(shape)
        src, dst, w = synth.ldbc_edges(shape, seed)
        bounds = h2.balanced_bounds(src, world)
        mine = np.searchsorted(bounds[1:world], src, side="right") == rank
        rep = h2.Replica.from_edges(shape.n_vertices, ids, src[mine], dst[mine], w[mine], rank=rank,
                                    world=world, shard_bounds=bounds)
        shr = ShardedReplica(LibEngine(rep, "cuda:0"), rank, world, "cuda:0", exchange=exchange)
        outs, ts = [], 0
        for k in range(4):
            g = synth.ldbc_batch(shape, seed, k, 5000, ts_base=ts)
            ts = int(g.ts.max())
            sl = g.slice(slice(rank * len(g) // world, (rank + 1) * len(g) // world))
            if k % 2:  # device slice; even batches go in as host arrays (staged by LibEngine)
                sl = synth.Batch(*(torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a).cuda()
                                   for a in (sl.kind, sl.src, sl.dst, sl.w, sl.ts)))
            shr.apply(sl, ts if k != 2 else int(np.quantile(g.ts, 0.7)))
            outs.append((rep.export(), shr.bases()))
        # freshness checks on the sharded replica (one collective per step)
        source = None
        for c in ids[:64]:
            try:
                rep.lookup(int(c))   # replicated ID map: the same answer on every rank
                source = int(c)
                break
            except h2.H2tapError:
                pass
        checks = (source, shr.bfs(source).cpu().numpy(), shr.sssp(source).cpu().numpy(),
                  shr.pagerank(0.85, 20).cpu().numpy())
        gathered = [None] * world
        dist.all_gather_object(gathered, (outs, checks))
        if rank == 0:
            q.put(gathered)
        dist.barrier()
        shr.close()
        rep.close()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("exchange", ["alltoall", "p2p"])
def test_two_process_sharded_apply(exchange):
    import torch.multiprocessing as mp
    import oracle
    import synth
    from oracle import O1

    world = 2
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, exchange)) for r in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=300)
    gathered = [g[0] for g in got]
    checks = [g[1] for g in got]
    for p in procs:
        p.join(120)
        assert p.exitcode == 0

    shape = synth.LdbcShape(n_person=300, n_msg=12000, e_person=20000)
    seed = synth.seed_of("c2") + 99
    ids = synth.ldbc_vertices(shape)
    src, dst, w = synth.ldbc_edges(shape, seed)
    o = O1.from_edges(shape.n_vertices, ids, src, dst, w)
    ts = 0
    for k in range(4):
        g = synth.ldbc_batch(shape, seed, k, 5000, ts_base=ts)
        ts = int(g.ts.max())
        rc, _ = o.apply(g, ts if k != 2 else int(np.quantile(g.ts, 0.7)))
        assert rc == 0
        off, cols, ww, gid = o.export()
        parts = [gathered[r][k] for r in range(world)]
        e_base = 0
        cat_off, cat_cols, cat_w, cat_ids = [], [], [], []
        for (po, pc, pw, pi), (row_lo, eb, vr, e) in parts:
            assert eb == e_base and vr == len(pi) and e == len(pc)
            assert row_lo == sum(len(x) for x in cat_ids)
            cat_off.append(po[:-1] + e_base)
            e_base += int(po[-1])
            cat_cols.append(pc); cat_w.append(pw); cat_ids.append(pi)
        assert np.array_equal(np.concatenate(cat_off + [np.array([e_base])]), off), f"batch {k}: offsets"
        assert np.array_equal(np.concatenate(cat_cols), cols), f"batch {k}: cols"
        assert np.array_equal(np.concatenate(cat_w).view(np.uint32), ww.view(np.uint32)), f"batch {k}: weights"
        assert np.array_equal(np.concatenate(cat_ids), gid), f"batch {k}: ext ids"

    # checks: identical on both ranks, equal to the oracle on the unsharded graph
    source = checks[0][0]
    for c in checks[1:]:
        assert c[0] == source and all(np.array_equal(a, b) for a, b in zip(c[1:], checks[0][1:]))
    d = int(np.searchsorted(gid, np.uint64(source)))
    assert gid[d] == source
    assert np.array_equal(checks[0][1], oracle.bfs(off, cols, d))
    assert np.array_equal(checks[0][2], oracle.sssp(off, cols, ww, d))
    ref = oracle.pagerank(off, cols, 0.85, 20)
    assert np.max(np.abs(checks[0][3] - ref) / ref) < 1e-6
