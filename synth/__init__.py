"""Seeded synthetic inputs (graphs and timestamped update streams).

The one module both the CUDA path's tests/bench and the oracle draw inputs
from.  It holds none of the method's arithmetic: it only generates edge lists,
vertex-ID lists and op streams from a counter-based generator (``synth.c``).
See DESIGN.md "Input recipe" and SURVEY.md §8(d).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "synth.c")
_LIB = os.path.join(_HERE, "libsynth.so")

NODE_INSERT, NODE_DELETE, EDGE_INSERT, EDGE_DELETE, EDGE_WEIGHT = 0, 1, 2, 3, 4
MASTER_SEED = 0x48325441  # master seed + config index


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", _LIB, _SRC])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u64, i32, f64, P = ctypes.c_uint64, ctypes.c_int, ctypes.c_double, ctypes.c_void_p
        L.synth_rand.restype = u64
        L.synth_rand.argtypes = [u64, u64, u64]
        L.synth_scramble.restype = u64
        L.synth_scramble.argtypes = [i32, u64, u64]
        L.synth_rmat_edges.argtypes = [i32, u64, u64, u64, P, P, P]
        L.synth_rmat_batch.argtypes = [i32, u64, u64, u64, u64, f64, f64, f64, u64, u64,
                                       P, P, P, P, P]
        L.synth_ldbc_vertices.argtypes = [u64, u64, P]
        L.synth_ldbc_edges.argtypes = [u64, u64, u64, u64, u64, u64, P, P, P]
        L.synth_ldbc_batch.restype = u64
        L.synth_ldbc_batch.argtypes = [u64, u64, u64, u64, u64, u64, i32, u64, P, P, P, P, P]
        L.synth_fuzz_batch.argtypes = [u64, u64, u64, u64, P, u64, u64, P, P, P, P, P]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


@dataclass
class Batch:
    """SoA op batch (h2tap_batch layout): kind u8, src u64, dst u64, w f32, ts u64."""
    kind: np.ndarray
    src: np.ndarray
    dst: np.ndarray
    w: np.ndarray
    ts: np.ndarray

    def __len__(self) -> int:
        return int(self.kind.shape[0])

    @staticmethod
    def empty(n: int = 0) -> "Batch":
        return Batch(np.zeros(n, np.uint8), np.zeros(n, np.uint64), np.zeros(n, np.uint64),
                     np.zeros(n, np.float32), np.zeros(n, np.uint64))

    @staticmethod
    def of(ops) -> "Batch":
        """ops: iterable of (kind, src, dst, w, ts)."""
        ops = list(ops)
        b = Batch.empty(len(ops))
        for i, (k, s, d, w, t) in enumerate(ops):
            b.kind[i], b.src[i], b.dst[i], b.w[i], b.ts[i] = k, s, d, w, t
        return b

    def slice(self, sl) -> "Batch":
        return Batch(self.kind[sl], self.src[sl], self.dst[sl], self.w[sl], self.ts[sl])

    def concat(self, other: "Batch") -> "Batch":
        return Batch(*(np.concatenate([a, b]) for a, b in zip(
            (self.kind, self.src, self.dst, self.w, self.ts),
            (other.kind, other.src, other.dst, other.w, other.ts))))

    def nbytes(self) -> int:
        return sum(a.nbytes for a in (self.kind, self.src, self.dst, self.w, self.ts))


# ------------------------------------------------------------------ RMAT ----
def rmat_edges(scale: int, seed: int, n: int | None = None, first: int = 0, weights: bool = True):
    """Initial RMAT edge list (Graph500 A,B,C,D; scrambled labels; f32 weights)."""
    if n is None:
        n = 16 << scale
    src = np.empty(n, np.uint64)
    dst = np.empty(n, np.uint64)
    w = np.empty(n, np.float32) if weights else None
    lib().synth_rmat_edges(scale, seed, first, n, _p(src), _p(dst), _p(w) if weights else None)
    return src, dst, w


def rmat_batch(scale: int, seed: int, k: int, n: int, m_initial: int, p_insert: float = 0.8,
               p_weight: float = 0.0, p_repeat: float = 0.0, ops_per_txn: int = 1,
               ts_base: int = 0) -> Batch:
    b = Batch.empty(n)
    lib().synth_rmat_batch(scale, seed, k, n, m_initial, p_insert, p_weight, p_repeat,
                           ops_per_txn, ts_base, _p(b.kind), _p(b.src), _p(b.dst), _p(b.w),
                           _p(b.ts))
    return b


# ------------------------------------------------------------- LDBC-SNB ----
@dataclass
class LdbcShape:
    n_person: int
    n_msg: int
    e_person: int

    @property
    def n_vertices(self) -> int:
        return self.n_person + self.n_msg

    @property
    def n_edges(self) -> int:
        return self.e_person + 4 * self.n_msg


# SF10-shaped: ~30.0 M vertices, ~176.6 M directed edges, 65,536 Person hubs
LDBC_SF10 = LdbcShape(n_person=65536, n_msg=30_000_000 - 65536,
                      e_person=176_600_000 - 4 * (30_000_000 - 65536))


def ldbc_vertices(shape: LdbcShape) -> np.ndarray:
    ids = np.empty(shape.n_vertices, np.uint64)
    lib().synth_ldbc_vertices(shape.n_person, shape.n_msg, _p(ids))
    return ids


def ldbc_edges(shape: LdbcShape, seed: int, first: int = 0, n: int | None = None):
    if n is None:
        n = shape.n_edges - first
    src = np.empty(n, np.uint64)
    dst = np.empty(n, np.uint64)
    w = np.empty(n, np.float32)
    lib().synth_ldbc_edges(shape.n_person, shape.n_msg, shape.e_person, seed, first, n,
                           _p(src), _p(dst), _p(w))
    return src, dst, w


def ldbc_batch(shape: LdbcShape, seed: int, k: int, n_cap: int, lodeg: bool = False,
               ts_base: int = 0) -> Batch:
    b = Batch.empty(n_cap)
    n = lib().synth_ldbc_batch(shape.n_person, shape.n_msg, shape.e_person, seed, k, n_cap,
                               int(lodeg), ts_base, _p(b.kind), _p(b.src), _p(b.dst), _p(b.w),
                               _p(b.ts))
    return b.slice(slice(0, int(n)))


# ------------------------------------------------------------------ fuzz ----
def fuzz_batch(seed: int, k: int, n: int, n_ids: int, probs=(0.1, 0.05, 0.5, 0.2, 0.15),
               ts_lo: int = 1, ts_span: int = 8) -> Batch:
    b = Batch.empty(n)
    p = np.asarray(probs, np.float64)
    p = p / p.sum()
    lib().synth_fuzz_batch(seed, k, n, n_ids, _p(p), ts_lo, ts_span, _p(b.kind), _p(b.src),
                           _p(b.dst), _p(b.w), _p(b.ts))
    return b


# ----------------------------------------------------------- configs ----
CONFIGS = {
    # name: description (BASELINE.json configs[i]) and generator parameters
    "c1": dict(index=0, kind="rmat", scale=16, edge_factor=16, batch=10_000, p_insert=0.8),
    "c2": dict(index=1, kind="ldbc", shape=LDBC_SF10, batch=100_000),
    "c3": dict(index=2, kind="rmat", scale=24, edge_factor=16, batch=1_000_000, p_insert=0.8),
    # configs[3] at P = 1 (the single-GPU reference point of the sharded scaling runs)
    "c4": dict(index=3, kind="rmat", scale=26, edge_factor=16, batch=8_000_000, p_insert=0.8),
}


def seed_of(name: str) -> int:
    return MASTER_SEED + CONFIGS[name]["index"]


# ------------------------------------------------- delta-record batches ----
# The paper's delta-store layout (§5.1): fixed-size delta records
# (transaction timestamp, node ID, validity and deleted flags, offsets + counts
# into the inserts / weights / deletes arrays).  This module only PACKS op
# sequences into that layout (input production); the expansion back into ops is
# the method's scan and lives on each side separately (oracle/, the CUDA path).
RECORD_DTYPE = np.dtype([("ts", "<u8"), ("node", "<u8"), ("ins_off", "<u8"), ("del_off", "<u8"),
                         ("ins_cnt", "<u4"), ("del_cnt", "<u4"), ("valid", "u1"), ("deleted", "u1"),
                         ("inserted", "u1"), ("pad", "u1", (5,))])
assert RECORD_DTYPE.itemsize == 48


@dataclass
class RecordBatch:
    """h2tap_record_batch layout: records (RECORD_DTYPE) + inserts u64 / weights f32 / deletes u64."""
    records: np.ndarray
    inserts: np.ndarray
    weights: np.ndarray
    deletes: np.ndarray

    def __len__(self) -> int:
        return int(self.records.shape[0])

    def nbytes(self) -> int:
        return sum(a.nbytes for a in (self.records, self.inserts, self.weights, self.deletes))


_PHASE = {NODE_INSERT: 0, EDGE_DELETE: 1, EDGE_INSERT: 2, NODE_DELETE: 3}


def records_from_ops(b: Batch) -> RecordBatch:
    """Pack consecutive ops of one transaction (same ts) on one node into one record,
    in the order a record expands to (reading A22): [NODE_INSERT] EDGE_DELETE* EDGE_INSERT*
    [NODE_DELETE], each destination at most once per record.  A new record starts
    wherever that order would break, so expanding the records yields `b` op for op.
    EDGE_WEIGHT has no record form (the paper's four update types)."""
    n = len(b)
    if n and np.any(b.kind == EDGE_WEIGHT):
        raise ValueError("EDGE_WEIGHT ops have no delta-record form")
    kind = b.kind.astype(np.int64)
    ph = np.zeros(n, np.int64)
    for k, p in _PHASE.items():
        ph[kind == k] = p
    cut = np.ones(n, bool)
    if n > 1:
        cut[1:] = ((b.ts[1:] != b.ts[:-1]) | (b.src[1:] != b.src[:-1]) | (ph[1:] < ph[:-1]) |
                   ((ph[1:] == ph[:-1]) & ((ph[1:] == 0) | (ph[1:] == 3))))
    edge = (kind == EDGE_INSERT) | (kind == EDGE_DELETE)
    while True:  # split a record where a destination repeats
        gid = np.cumsum(cut) - 1
        e = np.flatnonzero(edge)
        o = e[np.lexsort((e, b.dst[e], gid[e]))]
        dup = (gid[o[1:]] == gid[o[:-1]]) & (b.dst[o[1:]] == b.dst[o[:-1]])
        if not dup.any():
            break
        cut[o[1:][dup]] = True
    gid = np.cumsum(cut) - 1
    nr = int(cut.sum())
    rec = np.zeros(nr, RECORD_DTYPE)
    starts = np.flatnonzero(cut)
    rec["ts"] = b.ts[starts]
    rec["node"] = b.src[starts]
    rec["valid"] = 1
    ins = np.flatnonzero(kind == EDGE_INSERT)
    dl = np.flatnonzero(kind == EDGE_DELETE)
    rec["ins_cnt"] = np.bincount(gid[ins], minlength=nr)
    rec["del_cnt"] = np.bincount(gid[dl], minlength=nr)
    rec["ins_off"] = np.concatenate([[0], np.cumsum(rec["ins_cnt"].astype(np.uint64))[:-1]]) if nr else []
    rec["del_off"] = np.concatenate([[0], np.cumsum(rec["del_cnt"].astype(np.uint64))[:-1]]) if nr else []
    rec["inserted"][gid[kind == NODE_INSERT]] = 1
    rec["deleted"][gid[kind == NODE_DELETE]] = 1
    return RecordBatch(rec, b.dst[ins].copy(), b.w[ins].copy(), b.dst[dl].copy())


def dyn_record_batch(seed: int, k: int, xid: int, n_records: int, n_new: int = 4, max_slice: int = 6,
                     p_deleted: float = 0.05, p_new: float = 0.1, p_invalid: float = 0.03) -> RecordBatch:
    """Random delta records for the dynamic replica (Algorithm 1): each record's
    node is a new ID in (xid, xid + n_new] with probability p_new, otherwise an ID in [0, xid];
    inserts go to IDs in [0, xid + n_new], deletes to IDs in [0, xid]; slices are laid out
    back to back.  Random numbers only (no update rule here)."""
    rng = np.random.default_rng([seed, k, 0x44594E])
    rec = np.zeros(n_records, RECORD_DTYPE)
    new = rng.random(n_records) < p_new
    rec["node"] = np.where(new, xid + 1 + rng.integers(0, max(n_new, 1), n_records),
                           rng.integers(0, xid + 1, n_records)).astype(np.uint64)
    rec["deleted"] = rng.random(n_records) < p_deleted
    rec["valid"] = rng.random(n_records) >= p_invalid
    rec["inserted"] = new
    rec["ts"] = 1
    ic = rng.integers(0, max_slice + 1, n_records)
    dc = rng.integers(0, max_slice + 1, n_records)
    rec["ins_cnt"], rec["del_cnt"] = ic, dc
    rec["ins_off"] = np.concatenate([[0], np.cumsum(ic)[:-1]]).astype(np.uint64) if n_records else []
    rec["del_off"] = np.concatenate([[0], np.cumsum(dc)[:-1]]).astype(np.uint64) if n_records else []
    ni, nd = int(ic.sum()), int(dc.sum())
    ins = rng.integers(0, xid + 1 + n_new, ni).astype(np.uint64)
    wts = rng.integers(1, 1 << 16, ni).astype(np.float32) / np.float32(1 << 10)
    dl = rng.integers(0, xid + 1, nd).astype(np.uint64)
    return RecordBatch(rec, ins, wts, dl)
