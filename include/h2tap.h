/*
 * h2tap.h - C ABI of the B200-native update-propagation path for graph H2TAP.
 *
 * The path: a batch of committed, timestamped delta-store updates is propagated
 * into a CSR replica resident in GPU memory (§4.2, §5.2-5.4
 * P:L702-890).  Implemented by hand-written sm_100a kernels in libh2tap.so; no
 * CPU fallback.  Every entry point returns a status code (no exception crosses
 * the ABI); detail text for the last failure on the calling thread comes from
 * h2tap_last_error().
 *
 * Replica layout: offsets int64[V+1], cols uint32[E] (dense IDs),
 * weights float32[E] (carried bit-exactly), ext_ids uint64[V] (strictly
 * increasing external IDs; dense ID = rank of the external ID among live
 * vertices, reading A9).  Rows are sorted by column and duplicate-free
 * (reading A1).
 *
 * Ownership: caller buffers are only read (or, for export/bfs/pagerank,
 * written) during the call and never retained.  The replica owns all device
 * state; it allocates through h2tap_config.alloc (e.g. the torch caching
 * allocator) or cudaMallocAsync when alloc.alloc is NULL.
 *
 * Strong guarantee: on any error the replica's CSR, ID map, snapshot_ts and
 * pending set are unchanged.  A sticky CUDA error marks the handle POISONED;
 * then only h2tap_replica_destroy is valid.
 *
 * Streams: all work is ordered on h2tap_config.stream; calls return after the
 * work has completed.
 */
#ifndef H2TAP_H
#define H2TAP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct h2tap_replica h2tap_replica; /* opaque; owns all device state */

typedef enum {
    H2TAP_OK = 0,
    H2TAP_E_INVAL = -1,               /* bad argument, unknown op kind, malformed CSR */
    H2TAP_E_NOMEM = -2,               /* device allocation failed */
    H2TAP_E_CUDA = -3,                /* CUDA error (sticky ones poison the handle) */
    H2TAP_E_NCCL = -4,                /* collective failed (multi-GPU) */
    H2TAP_E_STALE_TS = -5,            /* an op has ts <= current snapshot_ts (reading A7) */
    H2TAP_E_SNAPSHOT_REGRESSION = -6, /* snapshot_ts < current snapshot_ts */
    H2TAP_E_CAPACITY = -7,            /* size beyond the 32-bit dense-ID / op-index limits */
    H2TAP_E_POISONED = -8             /* handle unusable after a sticky CUDA error */
} h2tap_status;

/* op kinds (uint8_t), §5.1; EDGE_WEIGHT is reading A3 */
enum {
    H2TAP_NODE_INSERT = 0, /* src = vertex; no-op if live (A12)                     */
    H2TAP_NODE_DELETE = 1, /* src = vertex; removes it and all in/out edges (A8)     */
    H2TAP_EDGE_INSERT = 2, /* src->dst, weight; upsert if both endpoints live (A2)   */
    H2TAP_EDGE_DELETE = 3, /* src->dst; no-op if absent (A4)                         */
    H2TAP_EDGE_WEIGHT = 4  /* src->dst, weight; update-if-present (A3)               */
};

/* A batch of ops, structure of arrays, all arrays of length n (29 B/op).
 * Caller-owned, read-only, not retained.  on_device: 0 = host memory (pinned
 * preferred; copied in), 1 = device memory of the replica's device. */
typedef struct {
    size_t n;
    int on_device;
    const uint8_t* kind;
    const uint64_t* src;
    const uint64_t* dst;    /* ignored for NODE_* */
    const float* weight;    /* ignored for NODE_* and EDGE_DELETE; may be NULL if unused */
    const uint64_t* ts;     /* commit timestamps (MVTO txn timestamps) */
    const uint64_t* seq;    /* arrival numbers (reading A5); NULL = assigned by the library in
                               batch order.  Sharded replicas without a communicator receive
                               routed ops and must pass their global (rank-major) numbers. */
} h2tap_batch;

/* Filled by h2tap_delta_apply (counts are global over all ranks). */
typedef struct {
    uint64_t n_visible;   /* ops with ts <= snapshot_ts applied this call (incl. earlier pending) */
    uint64_t n_deferred;  /* ops with ts > snapshot_ts kept pending for a later call (A6) */
    uint64_t n_gated;     /* edge ops dropped: endpoint not live at the op's point (A13) or
                             superseded by a later node delete of an endpoint (A8) */
    uint64_t n_new;       /* keys inserted that were absent from the old CSR */
    uint64_t n_del;       /* old edges removed by EDGE_DELETE */
    uint64_t n_upd;       /* old edges whose weight was overwritten (upsert or EDGE_WEIGHT) */
    uint64_t n_casc;      /* old edges removed by a node delete of an endpoint (A8) */
    uint64_t n_vertex_inserted, n_vertex_deleted;
    float ms_ingest, ms_nodeops, ms_sort_reduce, ms_degree_scan, ms_merge, ms_route, ms_total;
    uint64_t bytes_alg;   /* algorithmic bytes of this call */
    uint64_t bytes_merge; /* algorithmic bytes of the merge kernel launch */
    uint64_t n_launches;  /* kernels launched by this call */
    uint64_t h2d_bytes, d2h_bytes; /* host<->device bytes copied by this call */
} h2tap_apply_stats;

enum { H2TAP_ID_COMPACT = 0, H2TAP_ID_TOMBSTONE = 1 };

typedef struct {
    void* ctx;
    void* (*alloc)(void* ctx, size_t bytes, void* stream); /* NULL -> cudaMallocAsync */
    void (*free)(void* ctx, void* p, void* stream);
} h2tap_allocator;

/* Sharding (world > 1): 1D ranges of EXTERNAL vertex IDs.  Shard `rank` owns the rows
 * of the live vertices with shard_bounds[rank] <= id < shard_bounds[rank+1] (the last
 * bound is inclusive of UINT64_MAX); columns hold GLOBAL dense IDs (rank among all live
 * vertices) and every shard keeps the global ID map.  Without a communicator
 * (nccl_unique_id == NULL) the caller routes: each shard receives the edge ops whose
 * source it owns plus every node op, with explicit global seq numbers, and combines
 * shard bases itself; h2tap_replica_info reports the shard's rows/edges and its
 * global row base. */
typedef struct {
    int device;                  /* CUDA device ordinal */
    int rank, world;             /* world == 1 for a single replica */
    const void* nccl_unique_id;  /* ncclUniqueId bytes (collective mode, see below), else NULL */
    const uint64_t* shard_bounds;/* world + 1 non-decreasing external-ID split points (host),
                                    NULL if world == 1; world <= 4096, else H2TAP_E_INVAL */
    uint64_t expected_batch;     /* capacity hint (ops per batch); 0 = none */
    h2tap_allocator alloc;
    void* stream;                /* cudaStream_t; NULL = legacy default stream */
    int id_mode;                 /* H2TAP_ID_COMPACT (0): a deleted node leaves the ID map and the
                                    dense IDs are compacted (reading A9); H2TAP_ID_TOMBSTONE (1):
                                    the paper's merge() semantics, P:L879-881 — a deleted node
                                    keeps its slot with an empty row, flagged dead (reading A23);
                                    single replica only */
} h2tap_config;

/* Create from an edge list (reading A17): the vertex set is vertex_ids
 * (strictly increasing; NULL = identity 0..n_vertices-1), then the edges are
 * inserted in order, the last duplicate (src,dst) winning.  An edge endpoint
 * outside the vertex set, or non-increasing vertex_ids -> E_INVAL.
 * snapshot_ts = create_ts.  Arrays host (on_device=0) or device (1). */
h2tap_status h2tap_replica_create_from_edges(const h2tap_config* cfg, size_t n_vertices,
        const uint64_t* vertex_ids, size_t n_edges, const uint64_t* src, const uint64_t* dst,
        const float* w, int on_device, uint64_t create_ts, h2tap_replica** out);

/* Create from a CSR (checkpoint restore): offsets int64[n_vertices+1], cols
 * uint32[offsets[n]], w float[offsets[n]] (NULL = zeros), ext_ids uint64[n]
 * (NULL = identity).  Requires offsets[0]=0 and monotone, rows strictly
 * increasing, cols < n_vertices, ext_ids strictly increasing; else E_INVAL. */
h2tap_status h2tap_replica_create_from_csr(const h2tap_config* cfg, size_t n_vertices,
        const int64_t* offsets, const uint32_t* cols, const float* w, const uint64_t* ext_ids,
        int on_device, uint64_t create_ts, h2tap_replica** out);

/* One propagation cycle (the hot path; §5.2-5.4, Algorithm 2
 * P:L845-887): ops of this batch and earlier pending ops with ts <= snapshot_ts
 * are applied as if replayed in (ts, seq) order (seq = arrival order, reading
 * A5); the rest stay pending (A6).  Result: a new compact sorted CSR + ID map,
 * swapped in atomically at snapshot_ts.
 * Errors: snapshot_ts < current -> E_SNAPSHOT_REGRESSION; unknown kind ->
 * E_INVAL; any batch op with ts <= current snapshot_ts -> E_STALE_TS. */
h2tap_status h2tap_delta_apply(h2tap_replica* r, const h2tap_batch* batch, uint64_t snapshot_ts,
        h2tap_apply_stats* stats /* nullable */);

/* Stage the NEXT host batch: its host->device copy starts now on the replica's copy
 * stream (pinned host memory makes it asynchronous) and `staged` receives a device
 * batch in one of two library-owned slots.  Passing `staged` to h2tap_delta_apply
 * orders the apply after the copy.  Typical pipeline — the copy of batch k+1 overlaps
 * the apply of batch k (apply returns only when its cycle is done):
 *     stage(b0, &s0); for k: { stage(b[k+1], &s[k+1]); apply(&s[k]); }
 * At most two staged batches may be outstanding (the slots alternate); the host arrays
 * must stay valid until the batch has been applied.  seq must be NULL (arrival order).
 * The staged bytes are reported in the h2d_bytes of the apply that consumes them. */
h2tap_status h2tap_batch_stage(h2tap_replica* r, const h2tap_batch* host, h2tap_batch* staged);

/* ---- the paper's delta-store layout as a second input format ----
 * Delta records (§5.1 "Delta Store Architecture"): fixed-size records of
 * (transaction timestamp, node ID, validity flag, deleted flag, offset + count into the
 * inserts / weights arrays, offset + count into the deletes array); the destinations and
 * weights of a record's inserted relationships, and the destinations of its deleted ones,
 * live in three shared arrays (the CSR-like layout of Fig. 2).  `inserted` marks a record
 * whose transaction created its node (the paper implies it by a record for a new node ID,
 * P:L670-676; reading A22). */
typedef struct {
    uint64_t ts;                /* commit timestamp of the appending transaction */
    uint64_t node;              /* external ID of the updated node */
    uint64_t ins_off, del_off;  /* first index in inserts[]/weights[] and in deletes[] */
    uint32_t ins_cnt, del_cnt;  /* slice lengths */
    uint8_t valid;              /* 0: used in an earlier cycle, skipped */
    uint8_t deleted;            /* node deleted: all its relationships go */
    uint8_t inserted;           /* node created by this transaction (reading A22) */
    uint8_t pad[5];
} h2tap_delta_record;           /* 48 bytes */

typedef struct {  /* all arrays caller-owned, read-only, not retained; host or device */
    size_t n_records; int on_device;
    const h2tap_delta_record* records;
    const uint64_t* inserts; const float* weights; size_t n_inserts;
    const uint64_t* deletes; size_t n_deletes;
    /* the paper's 8-byte weights: when non-NULL they are used instead of
     * `weights` and narrowed to the replica's f32 by round-to-nearest-even (reading A15) */
    const double* weights64;
} h2tap_record_batch;

/* One propagation cycle from delta records: the delta-store scan (§5.2)
 * runs on the GPU — every valid record expands, at its timestamp and in record order,
 * into [NODE_INSERT] EDGE_DELETE* EDGE_INSERT* [NODE_DELETE] (reading A22) — and the
 * resulting ops are applied exactly as h2tap_delta_apply applies a flat batch (same
 * visibility, pending and error rules; each expanded op is one update in the stats).
 * The caller marks the records it passed as used; records with ts >
 * snapshot_ts stay pending inside the replica.  A record slice outside its array or a
 * flag other than 0/1 -> E_INVAL (nothing applied). */
h2tap_status h2tap_delta_apply_records(h2tap_replica* r, const h2tap_record_batch* batch,
        uint64_t snapshot_ts, h2tap_apply_stats* stats /* nullable */);

/* ---- the append-only delta store (§5.1 "Delta Store Architecture"; Fig. 2)
 * and the propagation cycle that scans it (§5.2-§5.3) — SURVEY.md §8(f) NEXT-1.
 * Host side: a delta table of fixed-size chunks of h2tap_delta_record plus the inserts /
 * weights (8-byte) / deletes arrays, chunked alike, in pinned memory.  A
 * committing transaction appends one delta per node it changed (append-only: no lookups of
 * other deltas, no updates); appends are thread-safe and published in index order.  The
 * store keeps a device mirror of its unconsumed tail on `device` (copied asynchronously on
 * the store's own copy stream).  Ownership: the store owns all its memory; appended arrays
 * are copied in and not retained.  Errors: E_INVAL (null / bad flags / bad slices),
 * E_NOMEM, E_CAPACITY (more than 65536 chunks), E_CUDA. */
typedef struct h2tap_delta_store h2tap_delta_store;
/* chunk_records: records per chunk (rounded up to a power of two, >= 1024, <= 2^24);
 * payload chunks hold 4 x chunk_records elements. */
h2tap_status h2tap_ds_create(int device, size_t chunk_records, h2tap_delta_store** out);
/* one delta: transaction ts, node, inserted / deleted flags (0/1), n_ins destination IDs with
 * their 8-byte weights, n_del deleted destination IDs; valid = 1 */
h2tap_status h2tap_ds_append(h2tap_delta_store* s, uint64_t ts, uint64_t node, int inserted, int deleted,
        const uint64_t* inserts, const double* weights, uint32_t n_ins, const uint64_t* deletes, uint32_t n_del);
/* n deltas at once (one bulk commit, host arrays): records[i].ins_off / del_off index the
 * given arrays (rebased to the store's positions); every record must have valid = 1 */
h2tap_status h2tap_ds_append_records(h2tap_delta_store* s, const h2tap_delta_record* records, size_t n,
        const uint64_t* inserts, const double* weights, size_t n_inserts, const uint64_t* deletes,
        size_t n_deletes);
/* n_records = published deltas; first_pending = index of the first delta that may still be
 * valid (everything before it was used and its host chunks may be released); n_mirrored =
 * deltas copied to the device; host_bytes / device_bytes = memory held (any may be NULL) */
h2tap_status h2tap_ds_info(const h2tap_delta_store* s, uint64_t* n_records, uint64_t* first_pending,
        uint64_t* n_mirrored, uint64_t* host_bytes, uint64_t* device_bytes);
/* copy deltas [first, first + n) of the live window [first_pending, n_records) with their
 * current validity flags and absolute array offsets into `out` (host) */
h2tap_status h2tap_ds_export(h2tap_delta_store* s, uint64_t first, size_t n, h2tap_delta_record* out);
void h2tap_ds_destroy(h2tap_delta_store* s);
/* One propagation cycle from the store: the scan covers every published delta from
 * first_pending on (trailing 1024-delta blocks whose deltas all have ts > snapshot_ts are
 * invisible and left for later; their copy to the device starts now and overlaps this
 * cycle), keeps the valid and visible ones (valid flag set, ts <= snapshot_ts),
 * expands them as h2tap_delta_apply_records does (reading A22; weights narrowed to f32 by
 * round-to-nearest-even) and applies them.  On success every delta it used is marked invalid
 * ("by the end of the delta store scan" P:L721-725) and first_pending advances; on
 * any error nothing is marked and the replica is unchanged (strong guarantee).  A valid
 * delta with ts <= the replica's current snapshot -> E_STALE_TS (reading A20).  stats:
 * h2d_bytes = the store's bytes copied to the device by this call. */
h2tap_status h2tap_delta_apply_store(h2tap_replica* r, h2tap_delta_store* s, uint64_t snapshot_ts,
        h2tap_apply_stats* stats /* nullable */);
/* Make `stream` (a cudaStream_t of the store's device; NULL = the legacy default stream) wait
 * for every host-to-device copy the store has issued so far - the read-ahead of the deltas a
 * cycle left for later keeps running after h2tap_delta_apply_store returns; an event recorded
 * on `stream` after this call completes only when those copies have.  Nothing blocks the host. */
h2tap_status h2tap_ds_join(h2tap_delta_store* s, void* stream);

/* ---- exchange step of a sharded apply ----------------------
 * A rank holding a slice of the global batch (i) validates it (every rank must agree
 * before anything is applied), (ii) packs its ops into 40-byte route records grouped
 * by destination shard — an edge op goes to the shard owning its source, a node op to
 * every shard — (iii) exchanges them with an all-to-all (NCCL over NVLink; the caller's
 * process group), and (iv) applies what it received. */
typedef struct {
    uint64_t src, dst, ts, seq;  /* seq: global rank-major arrival number (reading A5) */
    float w;
    uint8_t kind;
    uint8_t pad[3];
} h2tap_route_rec;

/* ---- collective mode ("every multi-GPU call is collective"; north_star:
 * ops routed to the owner of their source with an NCCL all-to-all, global offsets from
 * all-gathered per-shard counts).  A replica created with cfg.nccl_unique_id != NULL (the
 * same 128-byte id on every rank, from h2tap_nccl_unique_id on one rank; world >= 1,
 * shard_bounds may be NULL when world == 1) owns an NCCL communicator; creating it is
 * collective.  On such a replica:
 *   h2tap_delta_apply(slice, snapshot_ts): every rank passes ITS slice of the global batch
 *     (rank-major arrival order, reading A5; host or device) and the same snapshot_ts.  Inside:
 *     validation + destination counts, one ncclAllGather (host round trip 1: any rank's bad
 *     slice -> every rank returns the same E_INVAL / E_STALE_TS, nothing applied), the
 *     route records exchanged with grouped ncclSend/ncclRecv, the cycle prepared in the back
 *     buffers, one ncclAllGather of the prepare statuses and shard edge counts (round trip 2):
 *     every rank commits, or every rank aborts and returns the lowest (worst) status.
 *     h2tap_replica_info's ebase is then the shard's first global edge.  Prepare / async are
 *     refused (E_INVAL) on a collective replica: the call agrees and swaps itself.
 *   h2tap_bfs / h2tap_sssp / h2tap_pagerank: collective; the per-shard kernels plus one
 *     ncclAllReduce per step (MAX of the u8 frontier marks, SUM of the PageRank
 *     contributions and dangling mass, MIN of the fp64 distances); results are global
 *     (V entries, dense order) on every rank.
 * NCCL is loaded at run time (dlopen libnccl.so.2); unavailable -> E_INVAL at create.
 * A failure inside an NCCL call is E_NCCL. */
h2tap_status h2tap_nccl_unique_id(void* id_out /* >= 128 bytes */, size_t cap);
/* global arrival number of the next slice base; route bytes this rank sent to other
 * ranks in the last collective apply (40 B per record).  E_INVAL without a communicator. */
h2tap_status h2tap_collective_stats(const h2tap_replica* r, uint64_t* global_seq, uint64_t* route_bytes);

/* E_INVAL (unknown kind) / E_STALE_TS (ts <= snapshot) / OK for a batch slice. */
h2tap_status h2tap_batch_validate(const h2tap_replica* r, const h2tap_batch* batch);

/* ---- fused exchange over peer memory (pack-and-store into peers'
 * windows instead of pack + all-to-all).  Protocol per sharded apply (sharded.py):
 * (1) h2tap_route_count -> this rank's counts[world]; (2) the caller all-gathers the
 * world x world count matrix C and places, for every destination d, this rank's records
 * at offset sum_{s < rank} C[s][d] of d's receive window (rank-major global order, A5);
 * (3) h2tap_route_pack_p2p writes them there directly — one kernel, its stores go over
 * NVLink/NVSwitch to the peer-mapped windows — and returns when they are complete;
 * (4) a barrier; (5) each rank applies its window with h2tap_delta_apply_routed.
 * Windows are CUDA IPC allocations (h2tap_ipc_alloc on the owner, h2tap_ipc_open on the
 * peers; the 64-byte handles travel through the caller's process group).  world <= 16. */
h2tap_status h2tap_route_count(const h2tap_replica* r, const h2tap_batch* batch, uint64_t* counts);
h2tap_status h2tap_route_pack_p2p(const h2tap_replica* r, const h2tap_batch* batch, uint64_t seq0,
        h2tap_route_rec* const* peer_window /* host array [world] of device pointers */,
        const uint64_t* peer_offset /* host [world], records */);
h2tap_status h2tap_ipc_alloc(int device, size_t bytes, void** dptr, void* handle64);
h2tap_status h2tap_ipc_open(int device, const void* handle64, void** dptr);
h2tap_status h2tap_ipc_close(void* dptr);
h2tap_status h2tap_ipc_free(void* dptr);

/* Pack `batch` (on_device must be 1) into `out` (device, `capacity` records), grouped
 * by destination rank 0..world-1; counts[world] (host) receives the records per
 * destination.  Op i gets seq = seq0 + i.  Needs n_edge + world * n_node records; if
 * capacity is smaller, returns E_CAPACITY with counts filled (retry with more). */
h2tap_status h2tap_route_pack(const h2tap_replica* r, const h2tap_batch* batch, uint64_t seq0,
        h2tap_route_rec* out, uint64_t capacity, uint64_t* counts);

/* h2tap_delta_apply on received route records (device, n records, any order). */
h2tap_status h2tap_delta_apply_routed(h2tap_replica* r, const h2tap_route_rec* recs, size_t n,
        uint64_t snapshot_ts, h2tap_apply_stats* stats /* nullable */);

/* Two-phase apply (all-or-nothing across the shards of a sharded replica, SURVEY.md
 * §8(b) "the status is agreed with an all-reduce before commit").
 * h2tap_delta_apply_prepare / h2tap_delta_apply_routed_prepare run the whole cycle of
 * h2tap_delta_apply / h2tap_delta_apply_routed (a1-a6) but stop before the swap (a7):
 * the new CSR, ID map and pending set wait in the back buffers and every read
 * (export, info, checks) still sees the old snapshot.  The caller then agrees on the
 * status with its peers and calls h2tap_delta_commit (the swap at snapshot_ts, O(1),
 * cannot fail on a healthy handle) or h2tap_delta_abort (drops the prepared cycle; the
 * replica stays exactly as before the prepare).  While a cycle is prepared, every
 * other apply/create call returns H2TAP_E_INVAL.  h2tap_delta_apply = prepare + commit.
 * Errors of prepare: those of the one-phase call; nothing is prepared then. */
h2tap_status h2tap_delta_apply_prepare(h2tap_replica* r, const h2tap_batch* batch, uint64_t snapshot_ts,
        h2tap_apply_stats* stats /* nullable */);
h2tap_status h2tap_delta_apply_routed_prepare(h2tap_replica* r, const h2tap_route_rec* recs, size_t n,
        uint64_t snapshot_ts, h2tap_apply_stats* stats /* nullable */);
h2tap_status h2tap_delta_commit(h2tap_replica* r);  /* E_INVAL if nothing is prepared */
h2tap_status h2tap_delta_abort(h2tap_replica* r);   /* no-op if nothing is prepared */

/* Asynchronous apply (throughput mode): the whole cycle of h2tap_delta_apply is enqueued on
 * the replica's stream and the call returns after the cycle's first read-back (a1), without
 * waiting for the merge; the new snapshot is visible to every later call, which completes the
 * cycle first (export / info / checks synchronise; the next apply reads the cycle's final sizes
 * when its own first read-back has passed them, so consecutive cycles leave the GPU no idle gap).
 * *has_completed = 1 and *completed = the stats of the cycle completed during this call (the
 * previous one), else 0.  h2tap_replica_sync completes the last cycle and hands out its stats.
 * Errors detected before the return are those of h2tap_delta_apply (strong guarantee); the
 * asynchronous path is not taken for sharded replicas or two-phase cycles (they run
 * synchronously). */
h2tap_status h2tap_delta_apply_async(h2tap_replica* r, const h2tap_batch* batch, uint64_t snapshot_ts,
        h2tap_apply_stats* completed /* nullable */, int* has_completed /* nullable */);
h2tap_status h2tap_replica_sync(h2tap_replica* r, h2tap_apply_stats* completed /* nullable */,
        int* has_completed /* nullable */);

/* The pending set (ops committed after the current snapshot, kept for a later cycle, reading
 * A6) in arrival order with their arrival numbers - the part of a checkpoint the CSR
 * export does not hold (cf. the paper's persistent copy).  Arrays of n_pending
 * entries (h2tap_replica_info), host or device (on_device), any may be NULL.  Restore:
 * h2tap_replica_create_from_csr(create_ts = snapshot_ts) + h2tap_delta_apply of these ops at the
 * same snapshot_ts (they stay pending, in the same relative order). */
h2tap_status h2tap_pending_export(const h2tap_replica* r, uint8_t* kind, uint64_t* src, uint64_t* dst,
        float* w, uint64_t* ts, uint64_t* seq, int on_device);

/* Sizes of the current replica (any pointer may be NULL). */
h2tap_status h2tap_replica_info(const h2tap_replica* r, uint64_t* n_vertices, uint64_t* n_edges,
        uint64_t* snapshot_ts, uint64_t* n_pending, uint64_t* shard_vertex_base,
        uint64_t* shard_edge_base);

/* Copy the replica into caller buffers sized from h2tap_replica_info
 * (offsets V+1, cols E, w E, ext_ids V; any may be NULL).  checksums (nullable)
 * receives the position-keyed 64-bit checksums of {offsets, cols, w, ext_ids}:
 *   cs(a, salt) = sum_i sm64(bits(a_i) ^ sm64(i ^ salt)) mod 2^64, salts 1..4,
 *   sm64 = SplitMix64 finaliser, bits = raw pattern zero-extended to 64 bits. */
h2tap_status h2tap_replica_export(const h2tap_replica* r, int64_t* offsets, uint32_t* cols,
        float* w, uint64_t* ext_ids, int on_device, uint64_t checksums[4]);

/* BFS levels over out-edges from the vertex with external ID source_ext
 * (freshness check, LDBC Graphalytics P:L951-954, reading A18): level int32[V],
 * source 0, unreachable -1.  Unknown source -> E_INVAL. */
h2tap_status h2tap_bfs(const h2tap_replica* r, uint64_t source_ext, int32_t* level_out,
        int on_device);

/* PageRank, fp64 (Graphalytics): PR_0 = 1/V; PR_t(v) = (1-d)/V + d*(sum over
 * in-edges u->v of PR_{t-1}(u)/outdeg(u) + dangling mass / V). rank double[V]. */
/* Liveness of every vertex of the ID map (u8[V], 1 live / 0 tombstoned), in dense-ID
 * order; all 1 for a compacting replica.  live: host (on_device = 0) or device buffer of
 * V bytes, caller-owned.  In tombstone mode BFS / SSSP refuse a dead source (E_INVAL) and
 * PageRank runs on the live subgraph (|V| = live vertices, rank 0 for a tombstone). */
h2tap_status h2tap_replica_liveness(const h2tap_replica* r, uint8_t* live, int on_device);

h2tap_status h2tap_pagerank(const h2tap_replica* r, double damping, int iterations,
        double* rank_out, int on_device);

/* Single-source shortest paths over out-edges from the vertex with external ID
 * source_ext (Table 1's third analytic; reading A21):
 * dist double[V] in dense-ID order, edge length = the f32 weight widened to fp64,
 * path length = fp64 sum along the path, dist[source] = 0, unreachable = +inf.
 * Equal, bit for bit, to Dijkstra's result (the fixpoint is unique for weights >= 0).
 * dist_out: host (on_device = 0) or device (1) buffer of V doubles, caller-owned.
 * Errors: unknown source, a negative or NaN weight, or a sharded replica -> E_INVAL
 * (dist_out unspecified).  Reads the front buffer only. */
h2tap_status h2tap_sssp(const h2tap_replica* r, uint64_t source_ext, double* dist_out,
        int on_device);

/* ---- freshness checks on a sharded replica (SURVEY.md §8(e) "Checks") ----------------
 * Every shard keeps the whole ID map, so dense IDs are global and the per-vertex arrays
 * below are GLOBAL (n_vertices of the whole graph = h2tap_replica_info's shard_vertex_base
 * + ... over all shards; on one replica simply V), device-resident, caller-owned.  Each
 * call does one shard's part of one step on the rows it owns; the caller combines the
 * shards with a collective between steps (sharded.py: MAX of the BFS marks, SUM of the
 * PageRank sums, MIN of the SSSP candidates).  The definitions are those of h2tap_bfs,
 * h2tap_pagerank and h2tap_sssp (readings A18, A21).  Also valid on an unsharded replica. */
/* dense ID of a live vertex (E_INVAL if absent or a tombstone) */
h2tap_status h2tap_replica_lookup(const h2tap_replica* r, uint64_t ext_id, uint64_t* dense_out);
/* BFS: mark[v] = 1 for every v with level[v] < 0 that an owned row u with level[u] == depth
 * points to (mark zeroed by the caller) */
h2tap_status h2tap_shard_bfs_expand(const h2tap_replica* r, const int32_t* level, int32_t depth,
        uint8_t* mark);
/* BFS: level[v] = depth + 1 where mark[v] and level[v] < 0 (mark = the MAX over shards);
 * *n_new (host) = vertices settled */
h2tap_status h2tap_shard_bfs_settle(const h2tap_replica* r, int32_t* level, const uint8_t* mark,
        int32_t depth, uint64_t* n_new);
/* PageRank: acc[v] += pr[u] / outdeg(u) over the owned rows' edges, *dangling (device, one
 * double) += pr[u] of owned rows without out-edges (acc and dangling zeroed by the caller) */
h2tap_status h2tap_shard_pr_push(const h2tap_replica* r, const double* pr, double* acc,
        double* dangling);
/* PageRank: acc (the SUM over shards) becomes the next rank vector in place:
 * (1-d)/V + d * (acc[v] + dangling/V), dangling = the SUM over shards */
h2tap_status h2tap_shard_pr_finish(const h2tap_replica* r, double* acc_to_rank,
        const double* dangling, double damping);
/* SSSP: *bad (host) = 1 if an owned edge weight is negative or NaN */
h2tap_status h2tap_shard_check_weights(const h2tap_replica* r, int* bad);
/* SSSP: nd[v] = min(nd[v], dist[u] + w(u,v)) over owned rows u with frontier[u]
 * (nd starts as a copy of dist) */
h2tap_status h2tap_shard_sssp_relax(const h2tap_replica* r, const uint8_t* frontier,
        const double* dist, double* nd);
/* SSSP: frontier[v] = nd[v] < dist[v], then dist = nd (nd = the MIN over shards);
 * *n_changed (host) = vertices improved */
h2tap_status h2tap_shard_sssp_settle(const h2tap_replica* r, double* dist, const double* nd,
        uint8_t* frontier, uint64_t* n_changed);

/* ---- the dynamic replica ----
 * PAPER.md §5.4 "Dynamic Data Structures" + Algorithm 1: the valid and visible
 * deltas of a cycle are ingested into a hash-table graph.  Storage: one open-addressing table
 * of packed (src_dense, dst_dense) keys with f32 values on the device, vertex ext IDs ascending
 * with a liveness word each; dense ids never move (a deleted node keeps an empty, dead slot).
 * Semantics (readings D1-D5): xid = the largest ext ID held before the cycle;
 * per VALID record: deleted flag -> node deletion queue; node <= xid -> its inserts and
 * deletes; node > xid -> a new node with its inserts.  New nodes are appended ascending
 * (unless the same cycle deletes them), then ALL the cycle's edge inserts are applied
 * (upsert; a repeated (src, dst) keeps its last item in record/slice order; accepted iff both
 * endpoints are live), then all edge deletes, then the node deletions with their edges.
 * Record timestamps are not consulted: the caller passes the deltas the scan found visible.
 * Single GPU; dense ids and edges < 2^32 - 1.  All calls are synchronous on cfg->stream. */
typedef struct h2tap_dyn h2tap_dyn;
/* vertex_ids: n_vertices strictly increasing ext IDs (NULL = 0..n-1); edges (src, dst, w)
 * between them, a repeated pair keeps its last weight (w NULL -> 1.0); host or device
 * (on_device).  cfg: device / stream / allocator only (world and id_mode must be 0).
 * Unknown endpoint or unsorted ids -> E_INVAL; *out = NULL on any error. */
h2tap_status h2tap_dyn_create(const h2tap_config* cfg, size_t n_vertices, const uint64_t* vertex_ids,
        size_t n_edges, const uint64_t* src, const uint64_t* dst, const float* w, int on_device,
        h2tap_dyn** out);
/* One cycle of Algorithm 1 over `batch` (the h2tap_record_batch layout above).  Flag other
 * than 0/1 or a slice outside its array -> E_INVAL before anything is applied.  stats
 * (nullable): n_new / n_upd / n_del / n_casc / n_gated / n_vertex_*, ms_total (device time),
 * ms_merge / bytes_merge = the cascade pass's event-timed duration and table bytes (cycles in
 * which a node died; else 0),
 * n_launches, h2d_bytes; n_visible = expanded items (inserts + deletes + node ops). */
h2tap_status h2tap_dyn_apply_records(h2tap_dyn* d, const h2tap_record_batch* batch,
        h2tap_apply_stats* stats);
/* n_vertices = dense ids (live and dead), n_edges = live edges, table_slots = slots of the
 * per-vertex tables in use (their live keys, tombstones and EMPTY slots; garbage excluded) */
h2tap_status h2tap_dyn_info(const h2tap_dyn* d, uint64_t* n_vertices, uint64_t* n_edges,
        uint64_t* table_slots);
/* Materialise the CSR (rows = dense ids, dead rows empty, columns ascending): offsets
 * [n_vertices + 1], cols / w [n_edges], ext_ids [n_vertices], live u8 [n_vertices]; any
 * pointer may be NULL (skipped); host or device pointers (copied with cudaMemcpyDefault). */
h2tap_status h2tap_dyn_export(h2tap_dyn* d, int64_t* offsets, uint32_t* cols, float* w,
        uint64_t* ext_ids, uint8_t* live);
/* Freshness check on the dynamic replica (Table 1's BFS): materialise the CSR
 * (as h2tap_dyn_export) and run the CSR path's level-synchronous BFS from the live vertex
 * `source_ext`; level_out [n_vertices] (host or device) = hop count or -1 (unreachable or dead).
 * Unknown / dead source -> E_INVAL. */
h2tap_status h2tap_dyn_bfs(h2tap_dyn* d, uint64_t source_ext, int32_t* level_out);
/* PageRank (reading A18: d, fixed iterations, dangling mass spread uniformly, fp64) over the
 * live vertices, reading the per-vertex tables in place; rank_out [n_vertices] (host or
 * device), 0 for a dead vertex. */
h2tap_status h2tap_dyn_pagerank(h2tap_dyn* d, double damping, int iterations, double* rank_out);
/* SSSP (reading A21) from the live vertex source_ext over the tables in place; dist_out
 * [n_vertices] (host or device), +inf unreachable; a negative or NaN weight -> E_INVAL. */
h2tap_status h2tap_dyn_sssp(h2tap_dyn* d, uint64_t source_ext, double* dist_out);
/* Staged host input (as h2tap_batch_stage): start the H2D copy of a host record batch (pinned
 * arrays for an asynchronous copy) into one of two library slots on the copy stream and fill
 * `staged` with the device view; pass `staged` to h2tap_dyn_apply_records, which orders the
 * copy before its kernels.  A slot is reused two stages later. */
h2tap_status h2tap_dyn_stage(h2tap_dyn* d, const h2tap_record_batch* host, h2tap_record_batch* staged);
void h2tap_dyn_destroy(h2tap_dyn* d);

void h2tap_replica_destroy(h2tap_replica* r);
const char* h2tap_status_str(h2tap_status s);
const char* h2tap_last_error(void);
const char* h2tap_version(void);

#ifdef __cplusplus
}
#endif
#endif /* H2TAP_H */
