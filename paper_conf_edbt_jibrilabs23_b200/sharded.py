"""Sharded (multi-GPU) apply: one process per GPU, 1D external-ID ranges.

The exchange step a8 around the per-shard pipeline:

1. every rank validates its slice of the global batch and counts its records per
   destination (an edge op goes to the shard owning its source, a node op to every
   shard); ONE all-gather of (status, slice size, counts[world]) gives every rank the
   agreed validity, the rank-major global arrival numbers (reading A5) and the whole
   world x world count matrix (host round trip 1);
2. the library packs the slice into 40-byte route records grouped by destination;
3. the records are exchanged with an all-to-all whose splits every rank already knows
   (NCCL over NVLink on GPUs; gloo in the CPU tests);
4. two-phase apply: the library runs the whole cycle on what it received but leaves
   the result in its back buffers (h2tap_delta_apply_routed_prepare); the ranks agree on
   the prepare statuses with an all-reduce(MIN) (host round trip 2) and then ALL commit
   (h2tap_delta_commit, the swap) or ALL abort (h2tap_delta_abort) - a failure on one
   rank (e.g. out of memory) leaves every shard at the old snapshot;
5. shard bases (first global row, first global edge) come from an all-gather of the
   shards' row and edge counts.

Freshness checks on the sharded replica (SURVEY.md §8(e) "Checks"): every shard keeps the
whole ID map, so per-vertex state is a GLOBAL device array replicated on every rank; each
step runs one library kernel per shard over the rows it owns and one collective combines
the shards — BFS: MAX of the next-frontier marks per level; PageRank: SUM of the pushed
contributions and of the dangling mass per iteration; SSSP: MIN of the relaxed distances
per round.  The loops stop on counts that are identical on every rank.

The compute runs in the library's kernels (route packing included); this module is
orchestration only.  The engine is anything with validate / pack / apply_routed /
local_sizes (the CUDA replica here, an oracle-backed shard in the CPU tests).
"""
from __future__ import annotations

from types import SimpleNamespace

import numpy as np
import torch
import torch.distributed as dist

from . import ROUTE_REC_BYTES, H2tapError, IpcWindow, Replica


class LibEngine:
    """A shard of the CUDA replica (libh2tap.so)."""

    def __init__(self, replica: Replica, device):
        self.rep = replica
        self.device = torch.device(device)
        self.buf = torch.empty(0, dtype=torch.uint8, device=self.device)
        self.launches = 0   # validate / pack kernels (apply_routed reports its own)
        self.h2d = 0

    def stage(self, batch):
        """Device copy of a host batch slice (route packing reads device memory)."""
        if getattr(batch.kind, "is_cuda", False):
            return batch
        cols = []
        for a in (batch.kind, batch.src, batch.dst, batch.w, batch.ts):
            t = a if isinstance(a, torch.Tensor) else torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a)
            self.h2d += t.numel() * t.element_size()
            cols.append(t.to(self.device, non_blocking=True))
        return SimpleNamespace(kind=cols[0], src=cols[1], dst=cols[2], w=cols[3], ts=cols[4])

    def validate(self, batch) -> int:
        self.launches += 1 if len(batch.kind) else 0
        return self.rep.validate(batch)

    def pack(self, batch, seq0: int):
        n = len(batch.kind)
        cap = max(1024, int(n * 1.3) + 1024)
        for _ in range(2):
            if self.buf.numel() < cap * ROUTE_REC_BYTES:
                self.buf = torch.empty(cap * ROUTE_REC_BYTES, dtype=torch.uint8, device=self.device)
            rc, counts = self.rep.route_pack(batch, seq0, self.buf, cap)
            self.launches += 1 + (len(counts) if rc == 0 and n else 0)
            if rc == 0:
                return self.buf[: sum(counts) * ROUTE_REC_BYTES], counts
            if rc != -7:  # not E_CAPACITY
                raise H2tapError(rc, "h2tap_route_pack", "")
            cap = sum(counts)
        raise H2tapError(-7, "h2tap_route_pack", "capacity")

    def apply_routed(self, recs, n: int, snapshot_ts: int):
        return self.rep.apply_routed(recs, n, snapshot_ts)

    def prepare_routed(self, recs, n: int, snapshot_ts: int):
        return self.rep.prepare_routed(recs, n, snapshot_ts)

    def commit(self):
        self.rep.commit()

    def abort(self):
        self.rep.abort()

    # fused exchange (peer-memory windows)
    def route_count(self, batch):
        self.launches += 1 if len(batch.kind) else 0
        return self.rep.route_count(batch)

    def pack_p2p(self, batch, seq0: int, windows, offsets):
        self.launches += 1 if len(batch.kind) else 0
        self.rep.route_pack_p2p(batch, seq0, windows, offsets)

    def local_sizes(self):
        inf = self.rep.info()
        return inf["n_vertices"], inf["n_edges"], inf["shard_vertex_base"]

    # one shard's part of a check step (library kernels)
    def lookup(self, ext_id):
        return self.rep.lookup(ext_id)

    def bfs_expand(self, level, depth, mark):
        self.rep.shard_bfs_expand(level, depth, mark)

    def bfs_settle(self, level, mark, depth):
        return self.rep.shard_bfs_settle(level, mark, depth)

    def pr_push(self, pr, acc, dangling):
        self.rep.shard_pr_push(pr, acc, dangling)

    def pr_finish(self, acc, dangling, damping):
        self.rep.shard_pr_finish(acc, dangling, damping)

    def check_weights(self):
        return self.rep.shard_check_weights()

    def sssp_relax(self, frontier, dist, nd):
        self.rep.shard_sssp_relax(frontier, dist, nd)

    def sssp_settle(self, dist, nd, frontier):
        return self.rep.shard_sssp_settle(dist, nd, frontier)


class _Ptr:
    """device pointer with the data_ptr() interface the engine expects"""

    def __init__(self, p):
        self.p = p

    def data_ptr(self):
        return self.p


class ShardedReplica:
    def __init__(self, engine, rank: int, world: int, device, group=None, exchange: str = "alltoall",
                 time_exchange: bool = False):
        """exchange: "alltoall" (pack, then all-to-all over the process group) or "p2p"
        (h2tap_route_pack_p2p stores every record straight into its destination's
        CUDA-IPC window: the fused pack-and-exchange kernel; world <= 16)."""
        self.engine, self.rank, self.world, self.group = engine, rank, world, group
        self.device = torch.device(device)
        if exchange not in ("alltoall", "p2p"):
            raise ValueError("exchange must be 'alltoall' or 'p2p'")
        self.exchange = exchange
        self.win = None          # this rank's receive window (IpcWindow)
        self.win_caps = None     # every rank's window capacity (records)
        self.peers = None        # every rank's window, mapped here (device pointers)
        # gloo moves host tensors only: collectives on a CUDA engine then go through host
        # copies (tests / several ranks sharing one GPU); NCCL works on device memory
        self.coll = torch.device("cpu") if dist.get_backend(group) == "gloo" else self.device
        self.next_seq = 0
        # CUDA events around pack + exchange (stats["ms_exchange"]; CUDA engines only)
        self.time_exchange = time_exchange and self.device.type == "cuda"

    def _i64(self, vals):
        return torch.tensor(vals, dtype=torch.int64, device=self.coll)

    def apply(self, batch, snapshot_ts: int):
        """Apply this rank's slice of one global batch (every rank calls with the same
        snapshot_ts; slices are taken rank-major from the global batch)."""
        if hasattr(self.engine, "stage"):
            batch = self.engine.stage(batch)
        n = len(batch.kind)
        # 1. validity + slice size + destination counts of every rank: one all-gather
        st = int(self.engine.validate(batch))
        counts = [int(c) for c in self.engine.route_count(batch)] if st == 0 else [0] * self.world
        mine = self._i64([st, n] + counts)
        allv = torch.empty(self.world * (2 + self.world), dtype=torch.int64, device=self.coll)
        dist.all_gather_into_tensor(allv, mine, group=self.group)
        M = allv.view(self.world, 2 + self.world).cpu().numpy()          # host round trip 1
        if int(M[:, 0].min()) != 0:
            raise H2tapError(int(M[:, 0].min()), "sharded apply", "a rank rejected its batch slice")
        sizes = [int(x) for x in M[:, 1]]
        C = M[:, 2:]                                                      # C[s][d]
        seq0 = self.next_seq + sum(sizes[: self.rank])
        self.last_route_bytes = int(C[self.rank].sum() - C[self.rank][self.rank]) * ROUTE_REC_BYTES
        if self.time_exchange:
            ex0, ex1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ex0.record()
        if self.exchange == "p2p":
            recv, n_recv = self._exchange_p2p(batch, seq0, C)
        else:
            # 2./3. pack by destination, exchange with splits known from C
            recs, sent = self.engine.pack(batch, seq0)
            assert [int(x) for x in sent] == [int(x) for x in C[self.rank]], "route counts changed"
            rc = [int(x) for x in C[:, self.rank]]
            recv = torch.empty(sum(rc) * ROUTE_REC_BYTES, dtype=torch.uint8, device=self.coll)
            dist.all_to_all_single(recv, recs.to(self.coll), [c * ROUTE_REC_BYTES for c in rc],
                                   [int(c) * ROUTE_REC_BYTES for c in C[self.rank]], group=self.group)
            recv, n_recv = recv.to(recs.device), sum(rc)
        if self.time_exchange:
            ex1.record()
        # 4. two-phase apply: prepare everywhere, agree, then all commit or all abort
        try:
            status, stats = self.engine.prepare_routed(recv, n_recv, snapshot_ts)
        except Exception:   # an engine that raises counts as a failed prepare
            status, stats = -3, {}
        agree = self._i64([status])
        dist.all_reduce(agree, op=dist.ReduceOp.MIN, group=self.group)
        agreed = int(agree.item())                                        # host round trip 2
        if agreed != 0:
            if status == 0:
                self.engine.abort()
            raise H2tapError(agreed, "sharded apply", "a rank failed to prepare; every rank aborted")
        self.engine.commit()
        self.next_seq += sum(sizes)
        stats["global_batch"] = sum(sizes)
        stats["route_bytes"] = self.last_route_bytes
        if self.time_exchange:
            ex1.synchronize()
            stats["ms_exchange"] = ex0.elapsed_time(ex1)
        return stats

    def _windows(self, need):
        """(re)create receive windows so that rank d's holds need[d] records; collective,
        and every rank takes the same decision (all know the whole count matrix)"""
        if self.win_caps is not None and all(n <= c for n, c in zip(need, self.win_caps)):
            return
        mine_cap = self.win_caps[self.rank] if self.win_caps is not None else 0
        if self.win is None or need[self.rank] > mine_cap:
            if self.win is not None:
                self.win.free()
            mine_cap = max(1024, int(need[self.rank] * 1.5) + 1024)
            self.win = IpcWindow(self.device.index or 0, mine_cap * ROUTE_REC_BYTES)
        info = [None] * self.world
        dist.all_gather_object(info, (self.win.handle_bytes(), mine_cap), group=self.group)
        if self.peers is not None:
            for r, p in enumerate(self.peers):
                if r != self.rank and p:
                    IpcWindow.close_peer(p)
        self.peers = [self.win.ptr.value if r == self.rank else IpcWindow.open(self.device.index or 0, h)
                      for r, (h, _) in enumerate(info)]
        self.win_caps = [c for _, c in info]

    def _exchange_p2p(self, batch, seq0: int, C):
        need = C.sum(axis=0)
        self._windows([int(x) for x in need])
        offsets = C[: self.rank].sum(axis=0) if self.rank else np.zeros(self.world, np.int64)
        # one kernel packs and stores into the peers' windows; the barrier orders the
        # stores before the owners read their windows
        self.engine.pack_p2p(batch, seq0, self.peers, [int(x) for x in offsets])
        dist.barrier(group=self.group)
        return _Ptr(self.peers[self.rank]), int(need[self.rank])

    def close(self):
        if self.peers is not None:
            for r, p in enumerate(self.peers):
                if r != self.rank and p:
                    IpcWindow.close_peer(p)
            self.peers = None
        if self.win is not None:
            self.win.free()
            self.win = None

    def _allreduce(self, t, op):
        """collective on a device tensor (gloo: through a host copy)"""
        if t.device == self.coll:
            dist.all_reduce(t, op=op, group=self.group)
            return t
        h = t.to(self.coll)
        dist.all_reduce(h, op=op, group=self.group)
        t.copy_(h)
        return t

    def n_vertices(self) -> int:
        """global vertex count = the shards' rows summed"""
        v = self._i64([self.engine.local_sizes()[0]])
        dist.all_reduce(v, group=self.group)
        return int(v.item())

    def bfs(self, source_ext: int):
        """BFS levels (int32, global dense order, -1 unreachable) on every rank."""
        V = self.n_vertices()
        src = self.engine.lookup(source_ext)
        level = torch.full((V,), -1, dtype=torch.int32, device=self.device)
        level[src] = 0
        mark = torch.empty(V, dtype=torch.uint8, device=self.device)
        depth = 0
        while True:
            mark.zero_()
            self.engine.bfs_expand(level, depth, mark)
            self._allreduce(mark, dist.ReduceOp.MAX)
            if self.engine.bfs_settle(level, mark, depth) == 0:
                return level
            depth += 1

    def pagerank(self, damping: float = 0.85, iterations: int = 20):
        """PageRank (fp64, Graphalytics, reading A18) on every rank."""
        V = self.n_vertices()
        pr = torch.full((V,), 1.0 / V if V else 0.0, dtype=torch.float64, device=self.device)
        for _ in range(iterations):
            acc = torch.zeros(V, dtype=torch.float64, device=self.device)
            dang = torch.zeros(1, dtype=torch.float64, device=self.device)
            self.engine.pr_push(pr, acc, dang)
            self._allreduce(acc, dist.ReduceOp.SUM)
            self._allreduce(dang, dist.ReduceOp.SUM)
            self.engine.pr_finish(acc, dang, damping)
            pr = acc
        return pr

    def sssp(self, source_ext: int):
        """SSSP distances (fp64, +inf unreachable, reading A21) on every rank."""
        bad = self._i64([self.engine.check_weights()])
        dist.all_reduce(bad, op=dist.ReduceOp.MAX, group=self.group)
        if int(bad.item()):
            raise H2tapError(-1, "sharded sssp", "negative or NaN edge weight")
        V = self.n_vertices()
        src = self.engine.lookup(source_ext)
        d = torch.full((V,), float("inf"), dtype=torch.float64, device=self.device)
        d[src] = 0.0
        frontier = torch.zeros(V, dtype=torch.uint8, device=self.device)
        frontier[src] = 1
        while True:
            nd = d.clone()
            self.engine.sssp_relax(frontier, d, nd)
            self._allreduce(nd, dist.ReduceOp.MIN)
            if self.engine.sssp_settle(d, nd, frontier) == 0:
                return d

    def bases(self):
        """(row base, edge base, rows, edges) of this shard in the global CSR."""
        vr, e, row_lo = self.engine.local_sizes()
        allc = [self._i64([0, 0]) for _ in range(self.world)]
        dist.all_gather(allc, self._i64([vr, e]), group=self.group)
        e_base = sum(int(c[1].item()) for c in allc[: self.rank])
        return row_lo, e_base, vr, e
