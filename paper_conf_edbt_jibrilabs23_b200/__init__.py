"""B200-native update propagation into a GPU-resident CSR replica (graph H2TAP).

Thin ctypes binding over ``libh2tap.so`` (include/h2tap.h).  Argument
marshalling only: every step of the propagation path runs in the library's
sm_100a kernels.  There is no CPU fallback — importing this package raises if
the shared library is missing.  PyTorch is used only for device memory (the
caching allocator backs the library's allocations) and streams.

Arrays may be numpy arrays (host memory; copied in by the library) or torch
CUDA tensors (device memory of the replica's device).
"""
from __future__ import annotations

import atexit
import ctypes
import os
import weakref

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("H2TAP_LIB") or os.path.join(_HERE, "libh2tap.so")  # override: build-variant experiments

OK = 0
STATUS = {0: "OK", -1: "E_INVAL", -2: "E_NOMEM", -3: "E_CUDA", -4: "E_NCCL", -5: "E_STALE_TS",
          -6: "E_SNAPSHOT_REGRESSION", -7: "E_CAPACITY", -8: "E_POISONED"}
NODE_INSERT, NODE_DELETE, EDGE_INSERT, EDGE_DELETE, EDGE_WEIGHT = 0, 1, 2, 3, 4

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build the CUDA library first (`make lib` or "
                      "`python -c 'import __graft_entry__ as g; g.build()'`). There is no CPU fallback.")


class H2tapError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        self.status = status
        self.name = STATUS.get(status, str(status))
        super().__init__(f"{where}: {self.name}: {detail}")


_P = ctypes.c_void_p
_u64 = ctypes.c_uint64
_ALLOC = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p)
_FREE = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p)


class _Allocator(ctypes.Structure):
    _fields_ = [("ctx", _P), ("alloc", _ALLOC), ("free", _FREE)]


class _Config(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("rank", ctypes.c_int), ("world", ctypes.c_int),
                ("nccl_unique_id", _P), ("shard_bounds", _P), ("expected_batch", _u64),
                ("alloc", _Allocator), ("stream", _P), ("id_mode", ctypes.c_int)]


class _Batch(ctypes.Structure):
    _fields_ = [("n", ctypes.c_size_t), ("on_device", ctypes.c_int), ("kind", _P), ("src", _P),
                ("dst", _P), ("weight", _P), ("ts", _P), ("seq", _P)]


class _RecordBatch(ctypes.Structure):
    _fields_ = [("n_records", ctypes.c_size_t), ("on_device", ctypes.c_int), ("records", _P),
                ("inserts", _P), ("weights", _P), ("n_inserts", ctypes.c_size_t),
                ("deletes", _P), ("n_deletes", ctypes.c_size_t), ("weights64", _P)]


RECORD_BYTES = 48  # sizeof(h2tap_delta_record)


def _is_f64(a) -> bool:
    if a is None:
        return False
    if _is_torch(a):
        import torch
        return a.dtype == torch.float64
    return np.asarray(a).dtype == np.float64


def _record_batch(rb):
    """(h2tap_record_batch, keepalive) for rb (.records .inserts .weights .deletes); f64
    weights go through weights64 (the paper's 8-byte weights), f32 through weights."""
    w64 = _is_f64(rb.weights)
    pr, pi, pd = _ptr(rb.records), _ptr(rb.inserts, np.uint64), _ptr(rb.deletes, np.uint64)
    pw = _ptr(rb.weights, np.float64 if w64 else np.float32)
    b = _RecordBatch()
    recs = pr[2]
    nbytes = recs.numel() * recs.element_size() if _is_torch(recs) else recs.nbytes
    if nbytes % RECORD_BYTES:
        raise ValueError("records buffer is not a whole number of 48-byte records")
    b.n_records = nbytes // RECORD_BYTES
    b.on_device = _on_device(pr, pi, pw, pd)
    b.records, b.inserts, b.deletes = pr[0], pi[0], pd[0]
    b.weights, b.weights64 = (None, pw[0]) if w64 else (pw[0], None)
    b.n_inserts = len(pi[2]) if pi[2] is not None else 0
    b.n_deletes = len(pd[2]) if pd[2] is not None else 0
    return b, (pr, pi, pw, pd)


class ApplyStats(ctypes.Structure):
    _fields_ = [(n, _u64) for n in ("n_visible", "n_deferred", "n_gated", "n_new", "n_del", "n_upd",
                                    "n_casc", "n_vertex_inserted", "n_vertex_deleted")] + \
               [(n, ctypes.c_float) for n in ("ms_ingest", "ms_nodeops", "ms_sort_reduce",
                                              "ms_degree_scan", "ms_merge", "ms_route", "ms_total")] + \
               [(n, _u64) for n in ("bytes_alg", "bytes_merge", "n_launches", "h2d_bytes", "d2h_bytes")]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


_lib = ctypes.CDLL(LIB_PATH)
_lib.h2tap_replica_create_from_edges.restype = ctypes.c_int
_lib.h2tap_replica_create_from_edges.argtypes = [ctypes.POINTER(_Config), ctypes.c_size_t, _P,
                                                 ctypes.c_size_t, _P, _P, _P, ctypes.c_int, _u64,
                                                 ctypes.POINTER(_P)]
_lib.h2tap_replica_create_from_csr.restype = ctypes.c_int
_lib.h2tap_replica_create_from_csr.argtypes = [ctypes.POINTER(_Config), ctypes.c_size_t, _P, _P, _P,
                                               _P, ctypes.c_int, _u64, ctypes.POINTER(_P)]
_lib.h2tap_delta_apply.restype = ctypes.c_int
_lib.h2tap_delta_apply.argtypes = [_P, ctypes.POINTER(_Batch), _u64, ctypes.POINTER(ApplyStats)]
_lib.h2tap_delta_apply_records.restype = ctypes.c_int
_lib.h2tap_delta_apply_records.argtypes = [_P, ctypes.POINTER(_RecordBatch), _u64, ctypes.POINTER(ApplyStats)]
_lib.h2tap_batch_validate.restype = ctypes.c_int
_lib.h2tap_batch_validate.argtypes = [_P, ctypes.POINTER(_Batch)]
_lib.h2tap_route_pack.restype = ctypes.c_int
_lib.h2tap_route_pack.argtypes = [_P, ctypes.POINTER(_Batch), _u64, _P, _u64, ctypes.POINTER(_u64)]
_lib.h2tap_delta_apply_routed.restype = ctypes.c_int
_lib.h2tap_delta_apply_routed.argtypes = [_P, _P, ctypes.c_size_t, _u64, ctypes.POINTER(ApplyStats)]
ROUTE_REC_BYTES = 40  # sizeof(h2tap_route_rec)
_lib.h2tap_replica_info.restype = ctypes.c_int
_lib.h2tap_replica_info.argtypes = [_P] + [ctypes.POINTER(_u64)] * 6
_lib.h2tap_replica_export.restype = ctypes.c_int
_lib.h2tap_replica_export.argtypes = [_P, _P, _P, _P, _P, ctypes.c_int, ctypes.POINTER(_u64)]
_lib.h2tap_bfs.restype = ctypes.c_int
_lib.h2tap_bfs.argtypes = [_P, _u64, _P, ctypes.c_int]
_lib.h2tap_sssp.restype = ctypes.c_int
_lib.h2tap_sssp.argtypes = [_P, _u64, _P, ctypes.c_int]
for _n, _a in (("h2tap_batch_stage", [_P, ctypes.POINTER(_Batch), ctypes.POINTER(_Batch)]),
               ("h2tap_route_count", [_P, ctypes.POINTER(_Batch), _P]),
               ("h2tap_delta_apply_prepare", [_P, ctypes.POINTER(_Batch), _u64, ctypes.POINTER(ApplyStats)]),
               ("h2tap_delta_apply_routed_prepare", [_P, _P, ctypes.c_size_t, _u64, ctypes.POINTER(ApplyStats)]),
               ("h2tap_delta_commit", [_P]),
               ("h2tap_delta_apply_async", [_P, ctypes.POINTER(_Batch), _u64, ctypes.POINTER(ApplyStats),
                                            ctypes.POINTER(ctypes.c_int)]),
               ("h2tap_replica_sync", [_P, ctypes.POINTER(ApplyStats), ctypes.POINTER(ctypes.c_int)]),
               ("h2tap_pending_export", [_P, _P, _P, _P, _P, _P, _P, ctypes.c_int]),
               ("h2tap_ds_create", [ctypes.c_int, ctypes.c_size_t, ctypes.POINTER(_P)]),
               ("h2tap_ds_append", [_P, _u64, _u64, ctypes.c_int, ctypes.c_int, _P, _P, ctypes.c_uint32, _P,
                                    ctypes.c_uint32]),
               ("h2tap_ds_append_records", [_P, _P, ctypes.c_size_t, _P, _P, ctypes.c_size_t, _P, ctypes.c_size_t]),
               ("h2tap_ds_info", [_P] + [ctypes.POINTER(_u64)] * 5),
               ("h2tap_ds_export", [_P, _u64, ctypes.c_size_t, _P]),
               ("h2tap_delta_apply_store", [_P, _P, _u64, ctypes.POINTER(ApplyStats)]),
               ("h2tap_ds_join", [_P, _P]),
               ("h2tap_dyn_pagerank", [_P, ctypes.c_double, ctypes.c_int, _P]),
               ("h2tap_dyn_sssp", [_P, _u64, _P]),
               ("h2tap_dyn_stage", [_P, ctypes.POINTER(_RecordBatch), ctypes.POINTER(_RecordBatch)]),
               ("h2tap_delta_abort", [_P]),
               ("h2tap_route_pack_p2p", [_P, ctypes.POINTER(_Batch), _u64, _P, _P]),
               ("h2tap_ipc_alloc", [ctypes.c_int, ctypes.c_size_t, ctypes.POINTER(_P), _P]),
               ("h2tap_ipc_open", [ctypes.c_int, _P, ctypes.POINTER(_P)]),
               ("h2tap_ipc_close", [_P]),
               ("h2tap_ipc_free", [_P]),
               ("h2tap_replica_lookup", [_P, _u64, ctypes.POINTER(_u64)]),
               ("h2tap_shard_bfs_expand", [_P, _P, ctypes.c_int32, _P]),
               ("h2tap_shard_bfs_settle", [_P, _P, _P, ctypes.c_int32, ctypes.POINTER(_u64)]),
               ("h2tap_shard_pr_push", [_P, _P, _P, _P]),
               ("h2tap_shard_pr_finish", [_P, _P, _P, ctypes.c_double]),
               ("h2tap_shard_check_weights", [_P, ctypes.POINTER(ctypes.c_int)]),
               ("h2tap_shard_sssp_relax", [_P, _P, _P, _P]),
               ("h2tap_shard_sssp_settle", [_P, _P, _P, _P, ctypes.POINTER(_u64)])):
    getattr(_lib, _n).restype = ctypes.c_int
    getattr(_lib, _n).argtypes = _a
_lib.h2tap_replica_liveness.restype = ctypes.c_int
_lib.h2tap_replica_liveness.argtypes = [_P, _P, ctypes.c_int]
_lib.h2tap_pagerank.restype = ctypes.c_int
_lib.h2tap_pagerank.argtypes = [_P, ctypes.c_double, ctypes.c_int, _P, ctypes.c_int]
_lib.h2tap_ds_destroy.restype = None
_lib.h2tap_ds_destroy.argtypes = [_P]
_lib.h2tap_replica_destroy.restype = None
_lib.h2tap_replica_destroy.argtypes = [_P]
_lib.h2tap_status_str.restype = ctypes.c_char_p
_lib.h2tap_status_str.argtypes = [ctypes.c_int]
_lib.h2tap_last_error.restype = ctypes.c_char_p
_lib.h2tap_version.restype = ctypes.c_char_p


def version() -> str:
    return _lib.h2tap_version().decode()


class StagedBatch:
    """device batch in a library staging slot (h2tap_batch_stage); keeps the host arrays alive"""

    def __init__(self, b, keep):
        self.b, self.keep = b, keep

    def __len__(self):
        return int(self.b.n)


class IpcWindow:
    """A cudaMalloc'ed receive window shared with peer processes through CUDA IPC."""

    def __init__(self, device: int, nbytes: int):
        self.device, self.nbytes = device, int(nbytes)
        self.ptr = _P()
        self.handle = (ctypes.c_ubyte * 64)()
        _check(_lib.h2tap_ipc_alloc(device, self.nbytes, ctypes.byref(self.ptr), self.handle), "h2tap_ipc_alloc")

    def handle_bytes(self) -> bytes:
        return bytes(self.handle)

    @staticmethod
    def open(device: int, handle: bytes) -> int:
        p = _P()
        h = (ctypes.c_ubyte * 64).from_buffer_copy(handle)
        _check(_lib.h2tap_ipc_open(device, h, ctypes.byref(p)), "h2tap_ipc_open")
        return int(p.value)

    @staticmethod
    def close_peer(ptr: int):
        _check(_lib.h2tap_ipc_close(_P(ptr)), "h2tap_ipc_close")

    def free(self):
        if self.ptr:
            _lib.h2tap_ipc_free(self.ptr)
            self.ptr = _P()


def balanced_bounds(src_ext, world: int) -> np.ndarray:
    """world + 1 external-ID split points that balance the edges (rows are owned by their
    source): quantiles of the edge sources' external IDs.  Host-side planning only."""
    s = np.sort(np.asarray(src_ext, dtype=np.uint64))
    b = np.zeros(world + 1, np.uint64)
    for p in range(1, world):
        b[p] = s[min(len(s) - 1, (len(s) * p) // world)] if len(s) else p
    b[world] = np.iinfo(np.uint64).max
    return np.maximum.accumulate(b)


def _check(rc: int, where: str):
    if rc != OK:
        raise H2tapError(rc, where, (_lib.h2tap_last_error() or b"").decode())


def _is_torch(x) -> bool:
    return hasattr(x, "data_ptr") and hasattr(x, "is_cuda")


def _ptr(x, dtype=None):
    """(pointer, on_device, keepalive) for a numpy array or a torch tensor (or None)."""
    if x is None:
        return None, None, None
    if _is_torch(x):
        if not x.is_contiguous():
            x = x.contiguous()
        return ctypes.c_void_p(x.data_ptr()), bool(x.is_cuda), x
    a = np.ascontiguousarray(x, dtype=dtype)
    return ctypes.c_void_p(a.ctypes.data), False, a


def _on_device(*ptrs):
    flags = {p[1] for p in ptrs if p[0] is not None}
    if len(flags) > 1:
        raise ValueError("mix of host and device arrays in one call")
    return int(flags.pop()) if flags else 0


def _torch_allocator(device: int):
    import torch

    def _alloc(ctx, nbytes, stream):
        try:
            return torch.cuda.caching_allocator_alloc(int(nbytes), device, int(stream or 0))
        except Exception:  # out of memory: NULL makes the library return H2TAP_E_NOMEM
            return None

    def _free(ctx, p, stream):
        torch.cuda.caching_allocator_delete(int(p))

    return _ALLOC(_alloc), _FREE(_free)


# replicas still open at interpreter exit are destroyed before torch's module
# teardown (their memory goes back through torch's caching allocator)
_LIVE = weakref.WeakSet()


@atexit.register
def _close_live():
    for r in list(_LIVE):
        r.close()


NCCL_ID_BYTES = 128  # sizeof(ncclUniqueId)


def nccl_unique_id() -> bytes:
    """h2tap_nccl_unique_id: a fresh NCCL id (call on one rank, broadcast the bytes)"""
    buf = ctypes.create_string_buffer(NCCL_ID_BYTES)
    _check(_lib.h2tap_nccl_unique_id(buf, NCCL_ID_BYTES), "h2tap_nccl_unique_id")
    return buf.raw


class Replica:
    """A CSR replica in device memory (opaque h2tap_replica*)."""

    def __init__(self, handle, keep):
        self._h = handle
        self._keep = keep
        _LIVE.add(self)

    # ---------------------------------------------------------------- create
    @staticmethod
    def _config(device, stream, torch_allocator, rank=0, world=1, shard_bounds=None, tombstone=False,
                nccl_id=None):
        cfg = _Config()
        cfg.device = device
        cfg.id_mode = 1 if tombstone else 0  # H2TAP_ID_TOMBSTONE / H2TAP_ID_COMPACT
        cfg.rank, cfg.world = rank, world
        keep = []
        if nccl_id is not None:  # collective mode: the library owns an NCCL communicator
            idb = ctypes.create_string_buffer(bytes(nccl_id), NCCL_ID_BYTES)
            cfg.nccl_unique_id = ctypes.cast(idb, ctypes.c_void_p)
            keep.append(idb)
        if world > 1 or (nccl_id is not None and shard_bounds is not None):
            sb = np.ascontiguousarray(shard_bounds, dtype=np.uint64)
            if sb.shape != (world + 1,):
                raise ValueError("shard_bounds must have world + 1 entries")
            cfg.shard_bounds = ctypes.c_void_p(sb.ctypes.data)
            keep.append(sb)
        if torch_allocator:
            a, f = _torch_allocator(device)
            cfg.alloc.alloc, cfg.alloc.free = a, f
            keep += [a, f]
        if stream is None:
            try:
                import torch
                stream = torch.cuda.current_stream(device).cuda_stream
            except Exception:  # pragma: no cover
                stream = 0
        cfg.stream = ctypes.c_void_p(int(stream))
        return cfg, keep

    @classmethod
    def from_edges(cls, n_vertices, vertex_ids, src, dst, w, create_ts=0, device=0, stream=None,
                   torch_allocator=True, rank=0, world=1, shard_bounds=None, tombstone=False,
                   nccl_id=None) -> "Replica":
        """Create a replica (world > 1: shard `rank` of a vertex-range sharded graph; pass
        the GLOBAL vertex set and only the edges whose source this shard owns).  nccl_id
        (bytes from nccl_unique_id() on one rank, the same on every rank): collective mode -
        apply() takes this rank's slice of the global batch and routes / agrees inside the
        library; bfs / sssp / pagerank are collective (include/h2tap.h)."""
        cfg, keep = cls._config(device, stream, torch_allocator, rank, world, shard_bounds, tombstone, nccl_id)
        pi, ps, pd, pw = (_ptr(vertex_ids, np.uint64), _ptr(src, np.uint64), _ptr(dst, np.uint64),
                          _ptr(w, np.float32))
        ond = _on_device(pi, ps, pd, pw)
        n_e = len(src) if src is not None else 0
        h = ctypes.c_void_p()
        rc = _lib.h2tap_replica_create_from_edges(ctypes.byref(cfg), int(n_vertices), pi[0], n_e,
                                                  ps[0], pd[0], pw[0], ond, int(create_ts),
                                                  ctypes.byref(h))
        _check(rc, "h2tap_replica_create_from_edges")
        return cls(h, keep + [cfg])

    @classmethod
    def from_csr(cls, offsets, cols, w, ext_ids=None, create_ts=0, device=0, stream=None,
                 torch_allocator=True, tombstone=False) -> "Replica":
        cfg, keep = cls._config(device, stream, torch_allocator, tombstone=tombstone)
        po, pc, pw, pi = (_ptr(offsets, np.int64), _ptr(cols, np.uint32), _ptr(w, np.float32),
                          _ptr(ext_ids, np.uint64))
        ond = _on_device(po, pc, pw, pi)
        h = ctypes.c_void_p()
        rc = _lib.h2tap_replica_create_from_csr(ctypes.byref(cfg), len(offsets) - 1, po[0], pc[0],
                                                pw[0], pi[0], ond, int(create_ts), ctypes.byref(h))
        _check(rc, "h2tap_replica_create_from_csr")
        return cls(h, keep + [cfg])

    # ----------------------------------------------------------------- apply
    @staticmethod
    def _batch(batch):
        pk, ps, pd, pw, pt = (_ptr(batch.kind, np.uint8), _ptr(batch.src, np.uint64),
                              _ptr(batch.dst, np.uint64), _ptr(batch.w, np.float32),
                              _ptr(batch.ts, np.uint64))
        pq = _ptr(getattr(batch, "seq", None), np.uint64)
        b = _Batch()
        b.n = len(batch.kind)
        b.on_device = _on_device(pk, ps, pd, pw, pt, pq)
        b.kind, b.src, b.dst, b.weight, b.ts, b.seq = pk[0], ps[0], pd[0], pw[0], pt[0], pq[0]
        return b, (pk, ps, pd, pw, pt, pq)

    def validate(self, batch) -> int:
        """h2tap_batch_validate: status code of a batch slice (0 = OK)."""
        b, keep = self._batch(batch)
        return _lib.h2tap_batch_validate(self._h, ctypes.byref(b))

    def route_pack(self, batch, seq0: int, out, capacity_records: int):
        """h2tap_route_pack into `out` (torch CUDA uint8, >= capacity*40 bytes); returns
        (status, counts[world])."""
        b, keep = self._batch(batch)
        world = self._keep[-1].world if self._keep else 1
        counts = (_u64 * max(1, world))()
        rc = _lib.h2tap_route_pack(self._h, ctypes.byref(b), int(seq0), ctypes.c_void_p(out.data_ptr()),
                                   int(capacity_records), counts)
        return rc, [int(x) for x in counts]

    def apply_routed(self, recs, n: int, snapshot_ts: int):
        """h2tap_delta_apply_routed on `n` received route records (torch CUDA uint8)."""
        st = ApplyStats()
        _check(_lib.h2tap_delta_apply_routed(self._h, ctypes.c_void_p(recs.data_ptr()) if n else None, int(n),
                                             int(snapshot_ts), ctypes.byref(st)), "h2tap_delta_apply_routed")
        return st.as_dict()

    def prepare_routed(self, recs, n: int, snapshot_ts: int):
        """h2tap_delta_apply_routed_prepare: the whole cycle except the swap; returns
        (status, stats).  Follow with commit() or abort()."""
        st = ApplyStats()
        rc = _lib.h2tap_delta_apply_routed_prepare(self._h, ctypes.c_void_p(recs.data_ptr()) if n else None,
                                                   int(n), int(snapshot_ts), ctypes.byref(st))
        return rc, st.as_dict()

    def prepare(self, batch, snapshot_ts: int):
        """h2tap_delta_apply_prepare: (status, stats); follow with commit() or abort()."""
        b, keep = self._batch(batch)
        st = ApplyStats()
        rc = _lib.h2tap_delta_apply_prepare(self._h, ctypes.byref(b), int(snapshot_ts), ctypes.byref(st))
        return rc, st.as_dict()

    def commit(self):
        """h2tap_delta_commit: swap in the prepared cycle (a7)."""
        _check(_lib.h2tap_delta_commit(self._h), "h2tap_delta_commit")

    def abort(self):
        """h2tap_delta_abort: drop the prepared cycle (the replica is unchanged)."""
        _check(_lib.h2tap_delta_abort(self._h), "h2tap_delta_abort")

    def stage(self, batch) -> "StagedBatch":
        """h2tap_batch_stage: start the host->device copy of the next batch (pinned host
        arrays for an asynchronous copy); apply() the returned handle later."""
        b, keep = self._batch(batch)
        out = _Batch()
        _check(_lib.h2tap_batch_stage(self._h, ctypes.byref(b), ctypes.byref(out)), "h2tap_batch_stage")
        return StagedBatch(out, keep)

    def apply(self, batch, snapshot_ts: int, raise_on_error: bool = True):
        """h2tap_delta_apply; batch has .kind .src .dst .w .ts (numpy or torch CUDA), or is
        a StagedBatch from stage()."""
        if isinstance(batch, StagedBatch):
            b, keep = batch.b, batch.keep
        else:
            b, keep = self._batch(batch)
        st = ApplyStats()
        rc = _lib.h2tap_delta_apply(self._h, ctypes.byref(b), int(snapshot_ts), ctypes.byref(st))
        if raise_on_error:
            _check(rc, "h2tap_delta_apply")
            return st.as_dict()
        return rc, st.as_dict()

    def apply_async(self, batch, snapshot_ts: int):
        """h2tap_delta_apply_async: enqueue the cycle and return; returns the stats dict of the
        cycle completed during this call (the previous one) or None."""
        if isinstance(batch, StagedBatch):
            b, keep = batch.b, batch.keep
        else:
            b, keep = self._batch(batch)
        st, has = ApplyStats(), ctypes.c_int(0)
        _check(_lib.h2tap_delta_apply_async(self._h, ctypes.byref(b), int(snapshot_ts), ctypes.byref(st),
                                            ctypes.byref(has)), "h2tap_delta_apply_async")
        return st.as_dict() if has.value else None

    def pending(self):
        """h2tap_pending_export: (kind, src, dst, w, ts, seq) numpy arrays of the pending ops"""
        n = self.info()["n_pending"]
        a = [np.empty(n, dt) for dt in (np.uint8, np.uint64, np.uint64, np.float32, np.uint64, np.uint64)]
        _check(_lib.h2tap_pending_export(self._h, *(ctypes.c_void_p(x.ctypes.data) for x in a), 0),
               "h2tap_pending_export")
        return a

    def sync(self):
        """h2tap_replica_sync: complete the last asynchronous cycle; its stats dict or None."""
        st, has = ApplyStats(), ctypes.c_int(0)
        _check(_lib.h2tap_replica_sync(self._h, ctypes.byref(st), ctypes.byref(has)), "h2tap_replica_sync")
        return st.as_dict() if has.value else None

    def apply_records(self, rb, snapshot_ts: int, raise_on_error: bool = True):
        """h2tap_delta_apply_records; rb has .records (48-byte records: a numpy structured
        array, or a torch CUDA uint8 tensor) .inserts .weights (f32, or f64 = the paper's
        8-byte weights) .deletes."""
        b, keep = _record_batch(rb)
        st = ApplyStats()
        rc = _lib.h2tap_delta_apply_records(self._h, ctypes.byref(b), int(snapshot_ts), ctypes.byref(st))
        if raise_on_error:
            _check(rc, "h2tap_delta_apply_records")
            return st.as_dict()
        return rc, st.as_dict()

    def apply_store(self, store: "DeltaStore", snapshot_ts: int, raise_on_error: bool = True):
        """h2tap_delta_apply_store: one propagation cycle from an append-only delta store."""
        st = ApplyStats()
        rc = _lib.h2tap_delta_apply_store(self._h, store._h, int(snapshot_ts), ctypes.byref(st))
        if raise_on_error:
            _check(rc, "h2tap_delta_apply_store")
            return st.as_dict()
        return rc, st.as_dict()

    def collective_stats(self):
        """h2tap_collective_stats: {global_seq, route_bytes} of a collective-mode replica"""
        a, b = _u64(), _u64()
        _check(_lib.h2tap_collective_stats(self._h, ctypes.byref(a), ctypes.byref(b)), "h2tap_collective_stats")
        return dict(global_seq=a.value, route_bytes=b.value)

    # ------------------------------------------------------------- read back
    def info(self):
        v = [_u64() for _ in range(6)]
        _check(_lib.h2tap_replica_info(self._h, *(ctypes.byref(x) for x in v)), "h2tap_replica_info")
        return dict(n_vertices=v[0].value, n_edges=v[1].value, snapshot_ts=v[2].value,
                    n_pending=v[3].value, shard_vertex_base=v[4].value, shard_edge_base=v[5].value)

    def export(self, on_device: bool = False, checksums: bool = False):
        """(offsets, cols, w, ext_ids[, checksums]) as numpy (host) or torch CUDA tensors."""
        inf = self.info()
        V, E = inf["n_vertices"], inf["n_edges"]
        if on_device:
            import torch
            dev = torch.device("cuda", torch.cuda.current_device())
            out = (torch.empty(V + 1, dtype=torch.int64, device=dev),
                   torch.empty(E, dtype=torch.int32, device=dev),
                   torch.empty(E, dtype=torch.float32, device=dev),
                   torch.empty(V, dtype=torch.int64, device=dev))
            ptrs = [ctypes.c_void_p(t.data_ptr()) for t in out]
        else:
            out = (np.empty(V + 1, np.int64), np.empty(E, np.uint32), np.empty(E, np.float32),
                   np.empty(V, np.uint64))
            ptrs = [ctypes.c_void_p(a.ctypes.data) for a in out]
        cs = (_u64 * 4)()
        _check(_lib.h2tap_replica_export(self._h, *ptrs, int(on_device), cs if checksums else None),
               "h2tap_replica_export")
        return (*out, [int(x) for x in cs]) if checksums else out

    def checksums(self):
        cs = (_u64 * 4)()
        _check(_lib.h2tap_replica_export(self._h, None, None, None, None, 0, cs), "h2tap_replica_export")
        return [int(x) for x in cs]

    def bfs(self, source_ext: int) -> np.ndarray:
        lvl = np.empty(self.info()["n_vertices"], np.int32)
        _check(_lib.h2tap_bfs(self._h, int(source_ext), ctypes.c_void_p(lvl.ctypes.data), 0), "h2tap_bfs")
        return lvl

    def live(self) -> np.ndarray:
        """u8 liveness per dense id (all 1 unless the replica keeps tombstones)"""
        out = np.empty(self.info()["n_vertices"], np.uint8)
        _check(_lib.h2tap_replica_liveness(self._h, ctypes.c_void_p(out.ctypes.data), 0), "h2tap_replica_liveness")
        return out

    # ---- fused exchange (peer-memory windows; sharded.py runs the protocol)
    def route_count(self, batch):
        b, keep = self._batch(batch)
        world = self._keep[-1].world if self._keep else 1
        counts = (_u64 * max(1, world))()
        _check(_lib.h2tap_route_count(self._h, ctypes.byref(b), counts), "h2tap_route_count")
        return [int(x) for x in counts]

    def route_pack_p2p(self, batch, seq0: int, windows, offsets):
        b, keep = self._batch(batch)
        ptrs = (_P * len(windows))(*[_P(int(x)) for x in windows])
        offs = (_u64 * len(offsets))(*[int(x) for x in offsets])
        _check(_lib.h2tap_route_pack_p2p(self._h, ctypes.byref(b), int(seq0), ptrs, offs), "h2tap_route_pack_p2p")

    # ---- one shard's part of a check step (device tensors; sharded.py combines shards)
    def lookup(self, ext_id: int) -> int:
        d = _u64()
        _check(_lib.h2tap_replica_lookup(self._h, int(ext_id), ctypes.byref(d)), "h2tap_replica_lookup")
        return d.value

    def shard_bfs_expand(self, level, depth: int, mark):
        _check(_lib.h2tap_shard_bfs_expand(self._h, _P(level.data_ptr()), int(depth), _P(mark.data_ptr())),
               "h2tap_shard_bfs_expand")

    def shard_bfs_settle(self, level, mark, depth: int) -> int:
        n = _u64()
        _check(_lib.h2tap_shard_bfs_settle(self._h, _P(level.data_ptr()), _P(mark.data_ptr()), int(depth),
                                           ctypes.byref(n)), "h2tap_shard_bfs_settle")
        return n.value

    def shard_pr_push(self, pr, acc, dangling):
        _check(_lib.h2tap_shard_pr_push(self._h, _P(pr.data_ptr()), _P(acc.data_ptr()), _P(dangling.data_ptr())),
               "h2tap_shard_pr_push")

    def shard_pr_finish(self, acc, dangling, damping: float):
        _check(_lib.h2tap_shard_pr_finish(self._h, _P(acc.data_ptr()), _P(dangling.data_ptr()), float(damping)),
               "h2tap_shard_pr_finish")

    def shard_check_weights(self) -> int:
        b = ctypes.c_int()
        _check(_lib.h2tap_shard_check_weights(self._h, ctypes.byref(b)), "h2tap_shard_check_weights")
        return b.value

    def shard_sssp_relax(self, frontier, dist, nd):
        _check(_lib.h2tap_shard_sssp_relax(self._h, _P(frontier.data_ptr()), _P(dist.data_ptr()), _P(nd.data_ptr())),
               "h2tap_shard_sssp_relax")

    def shard_sssp_settle(self, dist, nd, frontier) -> int:
        n = _u64()
        _check(_lib.h2tap_shard_sssp_settle(self._h, _P(dist.data_ptr()), _P(nd.data_ptr()), _P(frontier.data_ptr()),
                                            ctypes.byref(n)), "h2tap_shard_sssp_settle")
        return n.value

    def sssp(self, source_ext: int) -> np.ndarray:
        dist = np.empty(self.info()["n_vertices"], np.float64)
        _check(_lib.h2tap_sssp(self._h, int(source_ext), ctypes.c_void_p(dist.ctypes.data), 0), "h2tap_sssp")
        return dist

    def pagerank(self, damping: float = 0.85, iterations: int = 20) -> np.ndarray:
        pr = np.empty(self.info()["n_vertices"], np.float64)
        _check(_lib.h2tap_pagerank(self._h, damping, iterations, ctypes.c_void_p(pr.ctypes.data), 0),
               "h2tap_pagerank")
        return pr

    def close(self):
        if getattr(self, "_h", None):
            _lib.h2tap_replica_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


for _n, _a, _r in (("h2tap_dyn_create", [ctypes.POINTER(_Config), ctypes.c_size_t, _P, ctypes.c_size_t, _P, _P, _P,
                                         ctypes.c_int, ctypes.POINTER(_P)], ctypes.c_int),
                   ("h2tap_dyn_apply_records", [_P, ctypes.POINTER(_RecordBatch), ctypes.POINTER(ApplyStats)],
                    ctypes.c_int),
                   ("h2tap_dyn_info", [_P] + [ctypes.POINTER(_u64)] * 3, ctypes.c_int),
                   ("h2tap_dyn_export", [_P, _P, _P, _P, _P, _P], ctypes.c_int),
                   ("h2tap_dyn_bfs", [_P, _u64, _P], ctypes.c_int),
                   ("h2tap_dyn_destroy", [_P], None)):
    getattr(_lib, _n).restype = _r
    getattr(_lib, _n).argtypes = _a


class StagedRecords:
    """A record batch staged by DynReplica.stage (device view of a library slot)."""

    def __init__(self, b, keep):
        self.b, self.keep = b, keep


class DynReplica:
    """The dynamic (hash-table) replica: Algorithm 1, §5.4
    (opaque h2tap_dyn*; include/h2tap.h documents the semantics)."""

    def __init__(self, handle, keep):
        self._h = handle
        self._keep = keep
        _LIVE.add(self)

    @classmethod
    def from_edges(cls, n_vertices, vertex_ids, src, dst, w, device=0, stream=None,
                   torch_allocator=True) -> "DynReplica":
        cfg, keep = Replica._config(device, stream, torch_allocator)
        pi, ps, pd, pw = (_ptr(vertex_ids, np.uint64), _ptr(src, np.uint64), _ptr(dst, np.uint64),
                          _ptr(w, np.float32))
        ond = _on_device(pi, ps, pd, pw)
        n_e = len(src) if src is not None else 0
        h = ctypes.c_void_p()
        _check(_lib.h2tap_dyn_create(ctypes.byref(cfg), int(n_vertices), pi[0], n_e, ps[0], pd[0], pw[0], ond,
                                     ctypes.byref(h)), "h2tap_dyn_create")
        return cls(h, keep + [cfg])

    def stage(self, rb) -> "StagedRecords":
        """h2tap_dyn_stage: start the H2D copy of a host record batch (pinned for an
        asynchronous copy) into a library slot; apply_records() the returned handle later."""
        b, keep = _record_batch(rb)
        out = _RecordBatch()
        _check(_lib.h2tap_dyn_stage(self._h, ctypes.byref(b), ctypes.byref(out)), "h2tap_dyn_stage")
        return StagedRecords(out, keep)

    def apply_records(self, rb, raise_on_error: bool = True):
        """h2tap_dyn_apply_records on rb (.records .inserts .weights .deletes, host or device),
        or on a StagedRecords from stage()."""
        b, keep = (rb.b, rb.keep) if isinstance(rb, StagedRecords) else _record_batch(rb)
        st = ApplyStats()
        rc = _lib.h2tap_dyn_apply_records(self._h, ctypes.byref(b), ctypes.byref(st))
        if raise_on_error:
            _check(rc, "h2tap_dyn_apply_records")
            return st.as_dict()
        return rc, st.as_dict()

    def info(self):
        v = [_u64() for _ in range(3)]
        _check(_lib.h2tap_dyn_info(self._h, *(ctypes.byref(x) for x in v)), "h2tap_dyn_info")
        return dict(n_vertices=v[0].value, n_edges=v[1].value, table_slots=v[2].value)

    def export(self):
        """(offsets i64, cols u32, w f32, ext_ids u64, live u8) as numpy arrays (the CSR
        materialised on the GPU)."""
        inf = self.info()
        V, E = inf["n_vertices"], inf["n_edges"]
        out = (np.empty(V + 1, np.int64), np.empty(E, np.uint32), np.empty(E, np.float32),
               np.empty(V, np.uint64), np.empty(V, np.uint8))
        _check(_lib.h2tap_dyn_export(self._h, *[ctypes.c_void_p(a.ctypes.data) for a in out]),
               "h2tap_dyn_export")
        return out

    def bfs(self, source_ext: int) -> np.ndarray:
        """BFS levels (int32 per dense id, -1 unreachable / dead) from a live ext id."""
        lv = np.empty(self.info()["n_vertices"], np.int32)
        _check(_lib.h2tap_dyn_bfs(self._h, int(source_ext), ctypes.c_void_p(lv.ctypes.data)), "h2tap_dyn_bfs")
        return lv

    def pagerank(self, damping: float = 0.85, iterations: int = 20) -> np.ndarray:
        """PageRank (fp64) over the live vertices, 0 for a dead one, tables read in place."""
        pr = np.empty(self.info()["n_vertices"], np.float64)
        _check(_lib.h2tap_dyn_pagerank(self._h, float(damping), int(iterations), ctypes.c_void_p(pr.ctypes.data)),
               "h2tap_dyn_pagerank")
        return pr

    def sssp(self, source_ext: int) -> np.ndarray:
        """SSSP distances (fp64, +inf unreachable) from a live ext id, tables read in place."""
        dist = np.empty(self.info()["n_vertices"], np.float64)
        _check(_lib.h2tap_dyn_sssp(self._h, int(source_ext), ctypes.c_void_p(dist.ctypes.data)), "h2tap_dyn_sssp")
        return dist

    def close(self):
        if getattr(self, "_h", None):
            _lib.h2tap_dyn_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


class DeltaStore:
    """The paper's append-only delta store (§5.1, Fig. 2; h2tap_ds_*): a chunked table of
    delta records + inserts / 8-byte weights / deletes arrays on the host, mirrored to the GPU
    by the propagation cycle (Replica.apply_store)."""

    def __init__(self, device: int = 0, chunk_records: int = 1 << 20):
        h = _P()
        _check(_lib.h2tap_ds_create(int(device), int(chunk_records), ctypes.byref(h)), "h2tap_ds_create")
        self._h = h

    def append(self, ts: int, node: int, inserts=(), weights=(), deletes=(), inserted=False, deleted=False):
        """one delta: transaction ts, node, its inserted (dst, 8-byte weight) and deleted dsts"""
        i = np.ascontiguousarray(inserts, np.uint64)
        w = np.ascontiguousarray(weights, np.float64)
        d = np.ascontiguousarray(deletes, np.uint64)
        if len(i) != len(w):
            raise ValueError("inserts and weights differ in length")
        _check(_lib.h2tap_ds_append(self._h, int(ts), int(node), int(bool(inserted)), int(bool(deleted)),
                                    ctypes.c_void_p(i.ctypes.data), ctypes.c_void_p(w.ctypes.data), len(i),
                                    ctypes.c_void_p(d.ctypes.data), len(d)), "h2tap_ds_append")

    def append_records(self, rb):
        """a bulk commit of host records (rb.records with valid = 1; weights f32 or f64)"""
        rec = np.ascontiguousarray(rb.records)
        i = np.ascontiguousarray(rb.inserts, np.uint64)
        w = np.ascontiguousarray(rb.weights, np.float64)
        d = np.ascontiguousarray(rb.deletes, np.uint64)
        _check(_lib.h2tap_ds_append_records(self._h, ctypes.c_void_p(rec.ctypes.data), len(rec),
                                            ctypes.c_void_p(i.ctypes.data), ctypes.c_void_p(w.ctypes.data), len(i),
                                            ctypes.c_void_p(d.ctypes.data), len(d)), "h2tap_ds_append_records")

    def info(self):
        v = [_u64() for _ in range(5)]
        _check(_lib.h2tap_ds_info(self._h, *(ctypes.byref(x) for x in v)), "h2tap_ds_info")
        return dict(n_records=v[0].value, first_pending=v[1].value, n_mirrored=v[2].value,
                    host_bytes=v[3].value, device_bytes=v[4].value)

    def join(self, stream=None):
        """h2tap_ds_join: `stream` (a torch.cuda.Stream or raw handle; None = the current torch
        stream) waits for the store's outstanding host-to-device copies (the read-ahead)"""
        if stream is None:
            import torch
            stream = torch.cuda.current_stream()
        h = getattr(stream, "cuda_stream", stream)
        _check(_lib.h2tap_ds_join(self._h, ctypes.c_void_p(int(h or 0))), "h2tap_ds_join")

    def export(self, first: int, n: int):
        """records [first, first + n) of the live window, current validity flags"""
        from synth import RECORD_DTYPE
        out = np.zeros(n, RECORD_DTYPE)
        _check(_lib.h2tap_ds_export(self._h, int(first), int(n), ctypes.c_void_p(out.ctypes.data)), "h2tap_ds_export")
        return out

    def close(self):
        if getattr(self, "_h", None):
            _lib.h2tap_ds_destroy(self._h)
            self._h = None

    def __del__(self):
        self.close()

