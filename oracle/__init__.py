"""ORACLE - test infrastructure only.

Plain, slow, obviously correct CPU implementation of what the hot path
computes.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py`` (its ``cpu_baseline`` leg and ``--impl reference`` arm) may
import this package.  The product package ``paper_conf_edbt_jibrilabs23_b200``
never imports it and shares no code with it (the only common module is the
input generator ``synth``, which holds none of the method's arithmetic).

* ``O1``  (o1_replay.cpp): sequential replay of visible ops in (ts, seq)
  order onto std::map adjacency, compact sorted CSR export; BFS and PageRank
  by their textbook definitions.
* ``O2``  (o2_bruteforce.py): independent brute force on a flat edge list,
  used to pin O1 on exhaustive tiny cases.
* ``O3``  (o3_alg2.cpp): the paper's own method on the host - a flat CSR
  updated by Algorithm 2 + merge(), 1 thread or OpenMP; pinned
  bit-exact to O1 and used as the whole-export checksum reference at full
  size and as the CPU baseline.
* ``OD``  (od_dynamic.py): the dynamic replica's update (Algorithm 1).
* ``expand_records``: the delta-store scan of the paper's record layout
  (§5.1-5.2) into the flat op sequence O1 replays.
* ``DeltaStoreModel``: the append-only delta store and its per-cycle consistency
  check (§5.1-5.3) as a plain Python list (valid + visible deltas are used once).
* ``checksum``: position-keyed 64-bit checksum of an exported array (the
  comparison key for large exports; written here independently of the CUDA
  export's own checksum kernel).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from .o2_bruteforce import BruteForce  # noqa: F401

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "o1_replay.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")
_SRC3 = os.path.join(_HERE, "o3_alg2.cpp")
_LIB3 = os.path.join(_HERE, "libo3.so")

OK, E_INVAL, E_STALE_TS, E_SNAPSHOT_REGRESSION = 0, -1, -5, -6


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-fPIC", "-shared", "-o", _LIB, _SRC])
    if force or not os.path.exists(_LIB3) or os.path.getmtime(_LIB3) < os.path.getmtime(_SRC3):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-fopenmp", "-fPIC", "-shared", "-o", _LIB3,
                               _SRC3])
    return _LIB


class _Stats(ctypes.Structure):
    _fields_ = [("n_visible", ctypes.c_uint64), ("n_deferred", ctypes.c_uint64)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        P, u64, sz = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_size_t
        L.o1_new.restype = P
        L.o1_new.argtypes = [u64]
        L.o1_set_tombstone.argtypes = [P]
        L.o1_live.argtypes = [P, P]
        L.o1_destroy.argtypes = [P]
        L.o1_load_edges.restype = ctypes.c_int
        L.o1_load_edges.argtypes = [P, sz, P, sz, P, P, P]
        L.o1_load_csr.restype = ctypes.c_int
        L.o1_load_csr.argtypes = [P, sz, P, P, P, P]
        L.o1_apply.restype = ctypes.c_int
        L.o1_apply.argtypes = [P, sz, P, P, P, P, P, u64, ctypes.POINTER(_Stats)]
        L.o1_info.argtypes = [P, P, P, P, P]
        L.o1_export.argtypes = [P, P, P, P, P]
        L.o1_pending.restype = u64
        L.o1_pending.argtypes = [P, P, P, P, P, P, P]
        L.o1_bfs.argtypes = [u64, P, P, u64, P]
        L.o1_pagerank.argtypes = [u64, P, P, ctypes.c_double, ctypes.c_int, P]
        L.o1_sssp.restype = ctypes.c_int
        L.o1_sssp.argtypes = [u64, P, P, P, u64, P]
        _lib = L
    return _lib


def _p(a):
    return None if a is None else ctypes.c_void_p(a.ctypes.data)


def _c(a, dt):
    return None if a is None else np.ascontiguousarray(a, dtype=dt)


class O1:
    """Sequential-replay oracle replica (std::map adjacency)."""

    def __init__(self, create_ts: int = 0, tombstone: bool = False):
        self.h = lib().o1_new(create_ts)
        if tombstone:  # reading A23: deleted nodes keep their id and an empty row
            lib().o1_set_tombstone(self.h)

    def __del__(self):
        if getattr(self, "h", None):
            lib().o1_destroy(self.h)
            self.h = None

    @staticmethod
    def from_edges(n_vertices, vertex_ids, src, dst, w, create_ts=0, tombstone=False) -> "O1":
        g = O1(create_ts, tombstone)
        ids = _c(vertex_ids, np.uint64)
        src, dst, w = _c(src, np.uint64), _c(dst, np.uint64), _c(w, np.float32)
        rc = lib().o1_load_edges(g.h, n_vertices, _p(ids), len(src), _p(src), _p(dst), _p(w))
        if rc != OK:
            raise ValueError(f"o1_load_edges: {rc}")
        return g

    @staticmethod
    def from_csr(offsets, cols, w, ext_ids=None, create_ts=0) -> "O1":
        g = O1(create_ts)
        off, cols, w = _c(offsets, np.int64), _c(cols, np.uint32), _c(w, np.float32)
        ids = _c(ext_ids, np.uint64)
        lib().o1_load_csr(g.h, len(off) - 1, _p(off), _p(cols), _p(w), _p(ids))
        return g

    def apply(self, batch, snapshot_ts: int):
        k = _c(batch.kind, np.uint8)
        s, d = _c(batch.src, np.uint64), _c(batch.dst, np.uint64)
        w, t = _c(batch.w, np.float32), _c(batch.ts, np.uint64)
        st = _Stats()
        rc = lib().o1_apply(self.h, len(k), _p(k), _p(s), _p(d), _p(w), _p(t), snapshot_ts,
                            ctypes.byref(st))
        return rc, {"n_visible": st.n_visible, "n_deferred": st.n_deferred}

    def live(self) -> np.ndarray:
        """u8 liveness of every exported vertex (all 1 unless tombstone mode)"""
        out = np.empty(self.info()["n_vertices"], np.uint8)
        lib().o1_live(self.h, _p(out))
        return out

    def info(self):
        v = [ctypes.c_uint64() for _ in range(4)]
        lib().o1_info(self.h, *(ctypes.byref(x) for x in v))
        return dict(n_vertices=v[0].value, n_edges=v[1].value, snapshot_ts=v[2].value,
                    n_pending=v[3].value)

    def export(self):
        inf = self.info()
        off = np.empty(inf["n_vertices"] + 1, np.int64)
        cols = np.empty(inf["n_edges"], np.uint32)
        w = np.empty(inf["n_edges"], np.float32)
        ids = np.empty(inf["n_vertices"], np.uint64)
        lib().o1_export(self.h, _p(off), _p(cols), _p(w), _p(ids))
        return off, cols, w, ids

    def pending(self):
        n = lib().o1_pending(self.h, None, None, None, None, None, None)
        a = [np.empty(n, dt) for dt in (np.uint8, np.uint64, np.uint64, np.float32, np.uint64,
                                        np.uint64)]
        lib().o1_pending(self.h, *(_p(x) for x in a))
        return a


_lib3 = None


def lib3():
    global _lib3
    if _lib3 is None:
        build()
        L = ctypes.CDLL(_LIB3)
        P, u64 = ctypes.c_void_p, ctypes.c_uint64
        L.o3_new.restype = P
        L.o3_new.argtypes = [u64]
        L.o3_destroy.argtypes = [P]
        L.o3_set_threads.argtypes = [ctypes.c_int]
        L.o3_max_threads.restype = ctypes.c_int
        L.o3_create_edges.restype = ctypes.c_int
        L.o3_create_edges.argtypes = [P, u64, P, u64, P, P, P]
        L.o3_apply.restype = ctypes.c_int
        L.o3_apply.argtypes = [P, u64, P, P, P, P, P, u64, ctypes.POINTER(_Stats)]
        L.o3_info.argtypes = [P, P, P, P, P]
        L.o3_export.argtypes = [P, P, P, P, P]
        L.o3_checksums.argtypes = [P, P]
        _lib3 = L
    return _lib3


def set_threads(n: int = 0) -> int:
    """OpenMP threads O3 uses (0 = every host thread); returns the count in effect."""
    lib3().o3_set_threads(int(n))
    return lib3().o3_max_threads()


class O3:
    """Algorithm-2 flat-CSR merge on the host (oracle/o3_alg2.cpp)."""

    def __init__(self, create_ts: int = 0):
        self.h = lib3().o3_new(create_ts)

    def __del__(self):
        if getattr(self, "h", None):
            lib3().o3_destroy(self.h)
            self.h = None

    @staticmethod
    def from_edges(n_vertices, vertex_ids, src, dst, w, create_ts=0) -> "O3":
        g = O3(create_ts)
        ids = _c(vertex_ids, np.uint64)
        src, dst, w = _c(src, np.uint64), _c(dst, np.uint64), _c(w, np.float32)
        rc = lib3().o3_create_edges(g.h, n_vertices, _p(ids), len(src), _p(src), _p(dst), _p(w))
        if rc != OK:
            raise ValueError(f"o3_create_edges: {rc}")
        return g

    def apply(self, batch, snapshot_ts: int):
        k = _c(batch.kind, np.uint8)
        s, d = _c(batch.src, np.uint64), _c(batch.dst, np.uint64)
        w, t = _c(batch.w, np.float32), _c(batch.ts, np.uint64)
        st = _Stats()
        rc = lib3().o3_apply(self.h, len(k), _p(k), _p(s), _p(d), _p(w), _p(t), snapshot_ts,
                             ctypes.byref(st))
        return rc, {"n_visible": st.n_visible, "n_deferred": st.n_deferred}

    def info(self):
        v = [ctypes.c_uint64() for _ in range(4)]
        lib3().o3_info(self.h, *(ctypes.byref(x) for x in v))
        return dict(n_vertices=v[0].value, n_edges=v[1].value, snapshot_ts=v[2].value,
                    n_pending=v[3].value)

    def export(self):
        inf = self.info()
        off = np.empty(inf["n_vertices"] + 1, np.int64)
        cols = np.empty(inf["n_edges"], np.uint32)
        w = np.empty(inf["n_edges"], np.float32)
        ids = np.empty(inf["n_vertices"], np.uint64)
        lib3().o3_export(self.h, _p(off), _p(cols), _p(w), _p(ids))
        return off, cols, w, ids

    def checksums(self):
        out = np.zeros(4, np.uint64)
        lib3().o3_checksums(self.h, _p(out))
        return [int(x) for x in out]


def expand_records(records, inserts, weights, deletes):
    """Delta-store scan (§5.1-§5.2) of a delta-record batch into
    the flat ops O1 replays, plain loops in record order.  Per VALID record (
    invalid records were used in an earlier cycle and are skipped), in the order of
    reading A22: NODE_INSERT if the record created its node, an EDGE_DELETE per entry
    of its deletes slice, an EDGE_INSERT per entry of its inserts / weights slices
    (P:L627-646), NODE_DELETE if its deleted flag is set.  All ops carry the
    record's transaction timestamp.  A slice outside its array -> ValueError.
    Returns (kind, src, dst, w, ts) lists."""
    kind, src, dst, w, ts = [], [], [], [], []

    def op(k, s, d, x, t):
        kind.append(k); src.append(s); dst.append(d); w.append(x); ts.append(t)

    for r in records:
        if not r["valid"]:
            continue
        t, v = int(r["ts"]), int(r["node"])
        io, ic, do, dc = int(r["ins_off"]), int(r["ins_cnt"]), int(r["del_off"]), int(r["del_cnt"])
        if io + ic > len(inserts) or io + ic > len(weights) or do + dc > len(deletes):
            raise ValueError("delta record slice outside its array")
        if r["inserted"]:
            op(0, v, 0, 0.0, t)                                  # NODE_INSERT
        for j in range(dc):
            op(3, v, int(deletes[do + j]), 0.0, t)               # EDGE_DELETE
        for j in range(ic):
            op(2, v, int(inserts[io + j]), float(weights[io + j]), t)  # EDGE_INSERT
        if r["deleted"]:
            op(1, v, 0, 0.0, t)                                  # NODE_DELETE
    return kind, src, dst, w, ts


class DeltaStoreModel:
    """The delta store of §5.1 and the scan's consistency check of §5.2-5.3
    (P:L702-769), written out plainly: an append-only list of delta records (ts, node,
    inserted / deleted flags, validity flag, slices of the inserts / weights / deletes
    arrays; the weights are 8-byte).  A propagation cycle with snapshot S
    takes, in append order, every record that is valid and visible (ts <= S; an invisible
    one waits for a later cycle), expands them (expand_records, reading A22;
    the 8-byte weights rounded to the replica's f32 by round-to-nearest-even, reading A15)
    and marks them invalid (each delta is used once)."""

    def __init__(self):
        self.records, self.inserts, self.weights, self.deletes = [], [], [], []

    def append(self, ts, node, inserts=(), weights=(), deletes=(), inserted=False, deleted=False):
        self.records.append(dict(ts=int(ts), node=int(node), ins_off=len(self.inserts), ins_cnt=len(inserts),
                                 del_off=len(self.deletes), del_cnt=len(deletes), valid=1,
                                 inserted=int(bool(inserted)), deleted=int(bool(deleted))))
        self.inserts += [int(x) for x in inserts]
        self.weights += [float(x) for x in weights]
        self.deletes += [int(x) for x in deletes]

    def append_records(self, recs, inserts, weights, deletes):
        for r in recs:
            io, ic, do, dc = int(r["ins_off"]), int(r["ins_cnt"]), int(r["del_off"]), int(r["del_cnt"])
            self.append(r["ts"], r["node"], inserts[io:io + ic], [float(x) for x in weights[io:io + ic]],
                        deletes[do:do + dc], r["inserted"], r["deleted"])

    def cycle(self, snapshot_ts):
        """the valid and visible deltas of this cycle as flat ops (kind, src, dst, w, ts);
        they are marked invalid"""
        used = [r for r in self.records if r["valid"] and r["ts"] <= snapshot_ts]
        w32 = np.asarray(self.weights, np.float64).astype(np.float32)  # RN-even narrowing
        ops = expand_records(used, self.inserts, w32, self.deletes)
        for r in used:
            r["valid"] = 0
        return ops


def bfs(offsets, cols, source_dense: int) -> np.ndarray:
    off, cols = _c(offsets, np.int64), _c(cols, np.uint32)
    lvl = np.empty(len(off) - 1, np.int32)
    lib().o1_bfs(len(off) - 1, _p(off), _p(cols), source_dense, _p(lvl))
    return lvl


def sssp(offsets, cols, weights, source_dense: int) -> np.ndarray:
    """Dijkstra distances (fp64, +inf unreachable); ValueError on a negative or NaN weight."""
    off, cols, w = _c(offsets, np.int64), _c(cols, np.uint32), _c(weights, np.float32)
    dist = np.empty(len(off) - 1, np.float64)
    if lib().o1_sssp(len(off) - 1, _p(off), _p(cols), _p(w), source_dense, _p(dist)) != 0:
        raise ValueError("sssp: negative or NaN edge weight")
    return dist


def pagerank(offsets, cols, damping: float = 0.85, iterations: int = 20) -> np.ndarray:
    off, cols = _c(offsets, np.int64), _c(cols, np.uint32)
    pr = np.empty(len(off) - 1, np.float64)
    lib().o1_pagerank(len(off) - 1, _p(off), _p(cols), damping, iterations, _p(pr))
    return pr


# ------------------------------------------------------------- checksum ----
_M = np.uint64(0xFFFFFFFFFFFFFFFF)


def _sm64(x: np.ndarray) -> np.ndarray:
    x = x + np.uint64(0x9E3779B97F4A7C15)
    x = (x ^ (x >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    x = (x ^ (x >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return x ^ (x >> np.uint64(31))


SALT = {"offsets": 1, "cols": 2, "weights": 3, "ext_ids": 4}


def checksum(a: np.ndarray, salt: int) -> int:
    """sum_i sm64(bits(a_i) ^ sm64(i ^ salt)) mod 2^64; bits = raw pattern, zero-extended."""
    a = np.ascontiguousarray(a)
    if a.dtype == np.float32:
        bits = a.view(np.uint32).astype(np.uint64)
    elif a.dtype.itemsize == 4:
        bits = a.view(np.uint32).astype(np.uint64)
    else:
        bits = a.view(np.uint64)
    total = np.uint64(0)
    step = 1 << 24
    with np.errstate(over="ignore"):
        for s in range(0, len(bits), step):
            i = np.arange(s, min(s + step, len(bits)), dtype=np.uint64)
            h = _sm64(bits[s:s + step] ^ _sm64(i ^ np.uint64(salt)))
            total = total + np.sum(h, dtype=np.uint64)
    return int(total)


def checksums(off, cols, w, ids):
    return [checksum(off, SALT["offsets"]), checksum(cols, SALT["cols"]),
            checksum(w, SALT["weights"]), checksum(ids, SALT["ext_ids"])]
