"""O2 - brute-force replay for tiny inputs (ORACLE; test infrastructure only).

An implementation of the same definition as O1 that shares nothing with it: the
graph is a flat Python list of (u, w, x) triples plus a set of live vertices,
every rule is a linear scan, and the CSR is rebuilt from scratch by sorting.
It exists to pin O1 (tests/test_oracle_pins.py): a dropped term, a wrong index
or a transposed operand in either shows up as a mismatch on exhaustive tiny
cases.

Rules (§5.1 P:L550-581 update types; §5.3 P:L755-769 visibility;
§5.4 P:L879-887 merge; readings A1-A13 of DESIGN.md):
  NODE_INSERT v      : v joins the live set (no-op if live)
  NODE_DELETE v      : v leaves the live set; every triple with u == v or w == v
                       is dropped (no-op if not live)
  EDGE_INSERT u,w,x  : if u and w are live: drop any (u, w, *) triple, add (u, w, x)
  EDGE_DELETE u,w    : drop any (u, w, *) triple
  EDGE_WEIGHT u,w,x  : if a (u, w, *) triple exists, replace it by (u, w, x)
"""
from __future__ import annotations

import numpy as np

NODE_INSERT, NODE_DELETE, EDGE_INSERT, EDGE_DELETE, EDGE_WEIGHT = 0, 1, 2, 3, 4
OK, E_INVAL, E_STALE_TS, E_SNAPSHOT_REGRESSION = 0, -1, -5, -6


class BruteForce:
    def __init__(self, live=(), edges=(), snap_ts=0):
        self.live = set(int(v) for v in live)
        self.edges = []  # flat list of [u, w, x]
        for (u, w, x) in edges:
            u, w = int(u), int(w)
            assert u in self.live and w in self.live
            self.edges = [e for e in self.edges if not (e[0] == u and e[1] == w)]
            self.edges.append([u, w, np.float32(x)])
        self.snap_ts = snap_ts
        self.next_seq = 0
        self.pending = []  # (ts, seq, kind, u, w, x)

    def _step(self, kind, u, w, x):
        if kind == NODE_INSERT:
            self.live.add(u)
        elif kind == NODE_DELETE:
            if u in self.live:
                self.live.discard(u)
                self.edges = [e for e in self.edges if e[0] != u and e[1] != u]
        elif kind == EDGE_INSERT:
            if u in self.live and w in self.live:
                self.edges = [e for e in self.edges if not (e[0] == u and e[1] == w)]
                self.edges.append([u, w, np.float32(x)])
        elif kind == EDGE_DELETE:
            self.edges = [e for e in self.edges if not (e[0] == u and e[1] == w)]
        elif kind == EDGE_WEIGHT:
            for e in self.edges:
                if e[0] == u and e[1] == w:
                    e[2] = np.float32(x)

    def apply(self, kind, src, dst, w, ts, snapshot_ts):
        if snapshot_ts < self.snap_ts:
            return E_SNAPSHOT_REGRESSION
        if any(int(k) > EDGE_WEIGHT for k in kind):
            return E_INVAL
        if any(int(t) <= self.snap_ts for t in ts):
            return E_STALE_TS
        ops = list(self.pending)
        for i in range(len(kind)):
            ops.append((int(ts[i]), self.next_seq + i, int(kind[i]), int(src[i]), int(dst[i]),
                        np.float32(w[i])))
        self.next_seq += len(kind)
        visible = [o for o in ops if o[0] <= snapshot_ts]
        self.pending = [o for o in ops if o[0] > snapshot_ts]
        # replay in commit order: sort by (ts, seq) by repeated minimum extraction
        while visible:
            m = min(range(len(visible)), key=lambda i: (visible[i][0], visible[i][1]))
            t, s, k, u, d, x = visible.pop(m)
            self._step(k, u, d, x)
        self.snap_ts = snapshot_ts
        return OK

    def export(self):
        ids = sorted(self.live)
        rank = {v: i for i, v in enumerate(ids)}
        trip = sorted((rank[e[0]], rank[e[1]], e[2]) for e in self.edges)
        off = np.zeros(len(ids) + 1, np.int64)
        for (r, _, _) in trip:
            off[r + 1] += 1
        off = np.cumsum(off).astype(np.int64)
        cols = np.array([t[1] for t in trip], np.uint32)
        w = np.array([t[2] for t in trip], np.float32)
        return off, cols, w, np.array(ids, np.uint64)
