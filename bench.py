#!/usr/bin/env python
"""Benchmark: delta updates/s merged into the GPU-resident CSR replica.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c1|c2|c3|c4] [--impl h2tap|reference]

A step is one h2tap_delta_apply of one synthetic batch (all SURVEY.md §8(a) steps a1-a7)
into the replica.  Default workload on 1 GPU: BASELINE.json configs[1] (LDBC-SNB-shaped SF10
property graph, 100K-update batches with node inserts and deletes and ID remap); with
--gpus N > 1: configs[3] (RMAT-26, 8M-update batches, the scaling config).  Inputs are
device-resident when the timed region starts (CUDA events on the replica stream, per-step
events for p10/p50/p90); the CSR (GBs read + written per step) exceeds the 126 MB L2, so
no explicit flush is needed (C1 is the L2-resident latency case).  The e2e leg restores
the replica to the state the timed region started from and replays the same batches from
pinned host memory through the public API, every H2D copy inside the timed region.

Prints ONE JSON line (rank 0).  --gpus N > 1 without a launcher re-executes itself under
torch.distributed.run (N ranks, one GPU each, 127.0.0.1); the graph is sharded by 1D
external-ID ranges (bounds from a sample of the edge sources, each rank generates only its
rows), every global batch is split rank-major, routed to the owners with an all-to-all
(NCCL) and applied per shard with a two-phase commit (strong scaling: the global batch is
the config's).  ``--parallelism replicas`` runs independent replicas instead.
The cpu_baseline (1 GPU only) and ``--impl reference`` time O3 - the paper's Algorithm-2
flat-CSR merge on the host (oracle/, test infrastructure), as it stands - on the FULL
workload at every host thread (and at 1 thread for the cpu_baseline).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

METRIC = "delta updates/sec merged into CSR replica"
PEAKS_FILE = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM = 6650.0  # GB/s, /opt/skills/guides/B200_PROFILING.md fallback


# ------------------------------------------------------------- workload ----
class Workload:
    """Initial graph + batch generator for one config (seeded, synthetic)."""

    def __init__(self, name: str, scale_down: int = 1):
        self.name = name
        self.cfg = synth.CONFIGS[name]
        self.seed = synth.seed_of(name)
        self.scale_down = scale_down
        if self.cfg["kind"] == "ldbc":
            s = self.cfg["shape"]
            if scale_down > 1:
                s = synth.LdbcShape(max(64, s.n_person // scale_down), max(64, s.n_msg // scale_down),
                                    max(64, s.e_person // scale_down))
            self.shape = s
            self.batch_size = max(64, self.cfg["batch"] // scale_down)
        else:
            self.scale = self.cfg["scale"] - (int(np.log2(scale_down)) if scale_down > 1 else 0)
            self.batch_size = max(64, self.cfg["batch"] // scale_down)
            self.m_initial = self.cfg["edge_factor"] << self.scale
        self.ts = 0

    def graph(self):
        if self.cfg["kind"] == "ldbc":
            ids = synth.ldbc_vertices(self.shape)
            src, dst, w = synth.ldbc_edges(self.shape, self.seed)
            return self.shape.n_vertices, ids, src, dst, w
        src, dst, w = synth.rmat_edges(self.scale, self.seed, n=self.cfg["edge_factor"] << self.scale)
        self.m_initial = len(src)
        return 1 << self.scale, None, src, dst, w

    def n_edges(self) -> int:
        if self.cfg["kind"] == "ldbc":
            return self.shape.n_edges
        return self.cfg["edge_factor"] << self.scale

    def _edges(self, first: int, n: int):
        if self.cfg["kind"] == "ldbc":
            return synth.ldbc_edges(self.shape, self.seed, first, n)
        return synth.rmat_edges(self.scale, self.seed, n=n, first=first)

    def source_sample(self, n: int = 1 << 20, windows: int = 512) -> np.ndarray:
        """sources of `n` edges taken from `windows` evenly spaced windows of the edge list
        (the generators are counter-based: any window can be generated alone)"""
        m, per = self.n_edges(), max(1, n // windows)
        return np.concatenate([self._edges(i * m // windows, min(per, m - i * m // windows))[0]
                               for i in range(windows)])

    def graph_owned(self, keep, chunk: int = 1 << 26):
        """the graph with only the edges whose source satisfies keep(src): generated chunk by
        chunk, so a rank never holds the whole edge list"""
        m = self.n_edges()
        self.m_initial = m
        parts = []
        for first in range(0, m, chunk):
            s, d, w = self._edges(first, min(chunk, m - first))
            sel = keep(s)
            parts.append((s[sel], d[sel], w[sel]))
        src, dst, w = (np.concatenate([p[i] for p in parts]) for i in range(3))
        if self.cfg["kind"] == "ldbc":
            return self.shape.n_vertices, synth.ldbc_vertices(self.shape), src, dst, w
        return 1 << self.scale, None, src, dst, w

    def batch(self, k: int) -> synth.Batch:
        if self.cfg["kind"] == "ldbc":
            b = synth.ldbc_batch(self.shape, self.seed, k, self.batch_size, ts_base=self.ts)
        else:
            b = synth.rmat_batch(self.scale, self.seed, k, self.batch_size, self.m_initial,
                                 p_insert=self.cfg["p_insert"], ts_base=self.ts)
        self.ts = int(b.ts.max())
        return b

    def describe(self) -> str:
        if self.cfg["kind"] == "ldbc":
            s = self.shape
            return (f"LDBC-SNB-shaped SF10 ({s.n_vertices} vertices, {s.n_edges} generated edges, "
                    f"{s.n_person} Person hubs), {self.batch_size}-op batches "
                    f"(66/22/11/1 insert-rel/insert-node/delete-rel/delete-node)")
        return (f"RMAT scale-{self.scale} ({1 << self.scale} vertices, "
                f"{self.cfg['edge_factor'] << self.scale} generated edges), {self.batch_size}-op "
                f"batches ({int(self.cfg['p_insert'] * 100)}/{100 - int(self.cfg['p_insert'] * 100)} insert/delete)")


# --------------------------------------------------------------- clocks ----
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(r[0]) for r in self.rows if r and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if len(r) > 1 and r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4)
                          if len(r) > 3 + i and r[3 + i].lower().startswith("active")})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def peaks():
    try:
        p = json.load(open(PEAKS_FILE))
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return FALLBACK_HBM, "fallback (B200_PROFILING.md 6.65 TB/s)"


# ------------------------------------------------------------ dist utils ----
def dist_setup():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def cpu_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count()


# ------------------------------------------------------------- oracle arm ----
def host_info() -> dict:
    model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count(), "affinity_cores": cpu_cores()}


def o3_run(name: str, plan, budget_s: float):
    """O3 (oracle/o3_alg2.cpp: the paper's Algorithm-2 flat-CSR merge, as it stands) on the
    FULL workload of `name`: create from the config's graph (untimed), then per (threads,
    max_batches) of `plan` apply the stream's next batches, each timed alone; stops a leg
    once `budget_s` of timed work is spent.  Returns [(threads, updates/s, batches, ms)]."""
    import oracle
    wl = Workload(name)
    nv, ids, src, dst, w = wl.graph()
    oracle.set_threads(0)
    o = oracle.O3.from_edges(nv, ids, src, dst, w)
    del src, dst, w
    out, k = [], 0
    for threads, max_b in plan:
        used = oracle.set_threads(threads)
        times, ops = [], 0
        while len(times) < max_b and sum(times) < budget_s:
            b = wl.batch(k)
            k += 1
            t0 = time.perf_counter()
            rc, st = o.apply(b, int(b.ts.max()))
            times.append(time.perf_counter() - t0)
            assert rc == 0
            ops += st["n_visible"]
        out.append((used, ops / sum(times), len(times), 1e3 * sum(times) / len(times)))
    oracle.set_threads(0)
    return out, wl


def o3_baseline(name: str) -> dict:
    """cpu_baseline: O3 at every host thread and at 1 thread on the full config."""
    nth = os.cpu_count() or 1
    res, wl = o3_run(name, [(nth, 4), (1, 1)], budget_s=30.0)
    (ta, va, na, ma), (t1, v1, n1, m1) = res
    return {"value": va, "unit": "updates/s", "cores": ta, "kind": "oracle",
            "sample": (f"O3 (Algorithm 2 + merge() on a flat host CSR, OpenMP over rows) on the full "
                       f"workload: {wl.describe()}; batches 0..{na - 1} at {ta} threads ({ma:.0f} ms each), "
                       f"then batch {na} at 1 thread ({m1:.0f} ms); create untimed"),
            "single_thread": {"value": v1, "unit": "updates/s", "cores": 1, "batches": n1, "ms_per_batch": m1},
            "ms_per_batch": ma, "host": host_info(),
            "paper_context": "paper's scan + Algorithm 2 merge of 2,014,347 SF10 deltas: 4660.39 ms "
                             "(~432 K deltas/s, 2x EPYC 7F52, P:L1899, P:L1933-1936)"}


def run_reference(args):
    world, rank, _ = dist_setup()
    if rank != 0:
        return
    nth = os.cpu_count() or 1
    res, wl = o3_run(args.config, [(nth, args.warmup), (nth, args.steps)], budget_s=150.0)
    _, value, n_timed, ms = res[1]
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "updates/s",
        "n_gpus": args.gpus, "steps": n_timed, "warmup": args.warmup, "ms_per_step": ms,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32/f32",
        "data": "synthetic", "config": {"workload": wl.describe(), "name": args.config},
        "cpu_baseline": {"value": value, "unit": "updates/s", "cores": res[1][0], "kind": "oracle",
                         "sample": (f"O3 (Algorithm-2 flat-CSR merge, oracle/o3_alg2.cpp, as it stands) on the "
                                    f"full workload, {n_timed} timed batches after {args.warmup} untimed, "
                                    f"{res[1][0]} OpenMP threads; create untimed"),
                         "host": host_info()},
        "e2e": {"value": value, "unit": "updates/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# --------------------------------------------------------------- GPU arm ----
def pct(xs, q):
    xs = sorted(xs)
    return xs[min(len(xs) - 1, int(round(q * (len(xs) - 1))))] if xs else None


def run_gpu(args):
    import torch
    import torch.distributed as dist

    import paper_conf_edbt_jibrilabs23_b200 as h2
    from paper_conf_edbt_jibrilabs23_b200.sharded import LibEngine, ShardedReplica

    world, rank, local = dist_setup()
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}")
    dev_idx = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(dev_idx)
    if world > 1:
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev_idx))
        else:
            dist.init_process_group("gloo")
    stream = torch.cuda.current_stream()
    sharded = world > 1 and args.parallelism == "shard"

    wl = Workload(args.config)
    t0 = time.time()
    if sharded:
        # 1D external-ID ranges balanced by edge count from a sample of the edge sources; each
        # rank generates the edge list chunk by chunk and keeps the rows it owns
        bounds = h2.balanced_bounds(wl.source_sample(), world)
        nv, ids, src, dst, w = wl.graph_owned(lambda s: np.searchsorted(bounds[1:world], s, side="right") == rank)
        rep = h2.Replica.from_edges(nv, ids, src, dst, w, 0, device=dev_idx,
                                    rank=rank, world=world, shard_bounds=bounds)
        eng = LibEngine(rep, f"cuda:{dev_idx}")
        shr = ShardedReplica(eng, rank, world, f"cuda:{dev_idx}", exchange=args.exchange, time_exchange=True)
    else:
        nv, ids, src, dst, w = wl.graph()
        rep = h2.Replica.from_edges(nv, ids, src, dst, w, 0, device=dev_idx, tombstone=args.tombstone)
    del src, dst, w
    setup_s = time.time() - t0

    n_total = args.warmup + args.steps
    # sharded: every rank draws the same global batches and takes its rank-major slice
    # (the global batch is the config's); replicas: rank-distinct streams
    k0 = 0 if sharded else rank * 1000

    def my_part(b):
        if not sharded:
            return b
        return b.slice(slice(rank * len(b) // world, (rank + 1) * len(b) // world))

    glob = [wl.batch(k0 + k) for k in range(n_total)]
    host = [my_part(b) for b in glob]
    snaps = [int(b.ts.max()) for b in glob]
    glob_n = [len(b) for b in glob]
    del glob

    records = args.input == "records"
    if records and sharded:
        raise SystemExit("--input records is single-replica only")

    def tens(a):
        return torch.from_numpy(a.view(np.uint8) if a.dtype.fields else a.view(np.int64) if a.dtype == np.uint64 else a)

    def to_dev(b):
        if records:
            rb = synth.records_from_ops(b)
            return synth.RecordBatch(*(tens(a).cuda() for a in (rb.records, rb.inserts, rb.weights, rb.deletes)))
        return synth.Batch(*(tens(a).cuda() for a in (b.kind, b.src, b.dst, b.w, b.ts)))

    # single replica, flat ops: h2tap_delta_apply_async (cycles enqueued back to back; the stats of
    # cycle k come back from call k+1 or from the final sync, which is inside the timed region)
    use_async = not sharded and not records and not args.sync_apply

    def apply(r, b, snap, out=None):
        if records:
            st = r.apply_records(b, snap)
        elif use_async:
            st = r.apply_async(b, snap)
        elif not sharded:
            st = r.apply(b, snap)
        else:
            l0 = eng.launches
            st = shr.apply(b, snap)
            st["n_launches"] += eng.launches - l0
        if st is not None and out is not None:
            out.append(st)
        return st

    def drain(r, out):
        if use_async:
            st = r.sync()
            if st is not None:
                out.append(st)

    dev = [to_dev(b) for b in host]
    for k in range(args.warmup):
        apply(rep, dev[k], snaps[k])
    drain(rep, [])
    torch.cuda.synchronize()
    # the e2e leg replays the timed batches on the same graph state: keep the state the timed
    # region starts from (device copy of the CSR + ID map; single replica, compact IDs)
    restore = not sharded and not args.tombstone and not records
    inf0 = rep.info()
    if restore:
        snap0 = rep.export(on_device=True)
        snap_ts0 = inf0["snapshot_ts"]
    if world > 1:
        dist.barrier()
    stats = []
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]
    with ClockSampler(dev_idx) as clk:
        torch.cuda.synchronize()
        evs[0].record(stream)
        for j, k in enumerate(range(args.warmup, n_total)):
            apply(rep, dev[k], snaps[k], stats)
            evs[j + 1].record(stream)
        drain(rep, stats)
        evs[-1].record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ms = evs[0].elapsed_time(evs[-1])
    step_ms = [evs[j].elapsed_time(evs[j + 1]) for j in range(args.steps)]
    inf1 = rep.info()
    e_steps = [inf0["n_edges"]]
    for s_ in stats:  # I6: E' = E + NEW - DEL - CASC
        e_steps.append(e_steps[-1] + s_["n_new"] - s_["n_del"] - s_["n_casc"])
    # updates: the global batches' ops (sharded: node ops reach every shard, count them once)
    updates = (sum(glob_n[args.warmup:]) / world if sharded else sum(s["n_visible"] for s in stats))

    def reduce_max_sum(ms_, upd):
        if world == 1:
            return ms_, float(upd)
        t = torch.tensor([ms_, float(upd)], dtype=torch.float64,
                         device="cpu" if args.dist_backend == "gloo" else "cuda")
        mx = t.clone()
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        return float(mx[0]), float(t[1])

    ms_max, updates_all = reduce_max_sum(ms, updates)
    value = updates_all / (ms_max / 1e3)

    # ---- e2e: pinned host batches through the public API, H2D inside the timed region
    pipelined = not sharded and not records
    if restore:   # same graph state, same batches as the device-resident leg
        rep.close()
        rep = h2.Replica.from_csr(*snap0, create_ts=snap_ts0, device=dev_idx)
        del snap0
        # the restored replica's work buffers are allocated by one prepared-and-aborted cycle
        # (two-phase apply: the state does not change), so no allocation falls in the timed region
        rc, _ = rep.prepare(dev[args.warmup], snaps[args.warmup])
        assert rc == 0
        rep.abort()
        rep.sync()
        e_host, e_snaps, e_glob_n = host[args.warmup:], snaps[args.warmup:], glob_n[args.warmup:]
        e_how_state = "same graph state and batches as the device-resident leg (replica restored from a device copy)"
    else:
        e_glob = [wl.batch(k0 + n_total + k) for k in range(args.steps)]
        e_host = [my_part(b) for b in e_glob]
        e_snaps = [int(b.ts.max()) for b in e_glob]
        e_glob_n = [len(b) for b in e_glob]
        del e_glob
        e_how_state = "the stream's next batches (the graph state continues from the device-resident leg)"

    def pinned(b):
        if records:
            rb = synth.records_from_ops(b)
            return synth.RecordBatch(*(tens(a).pin_memory() for a in (rb.records, rb.inserts, rb.weights, rb.deletes)))
        return synth.Batch(*(tens(a).pin_memory() for a in (b.kind, b.src, b.dst, b.w, b.ts)))

    e_pin = [pinned(b) for b in e_host]
    if pipelined:   # allocate and warm both staging slots (nothing is applied)
        rep.stage(e_pin[0])
        rep.stage(e_pin[min(1, len(e_pin) - 1)])
    drain(rep, [])
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    e_stats = []
    h2d0 = eng.h2d if sharded else 0
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    if pipelined:
        # h2tap_batch_stage: the H2D copy of batch k+1 runs on the copy engine while batch k
        # is applied (the copies stay inside the timed region)
        staged = rep.stage(e_pin[0])
        for k in range(args.steps):
            nxt = rep.stage(e_pin[k + 1]) if k + 1 < args.steps else None
            apply(rep, staged, e_snaps[k], e_stats)
            staged = nxt
    else:
        for k in range(args.steps):
            apply(rep, e_pin[k], e_snaps[k], e_stats)
    drain(rep, e_stats)
    ev1.record(stream)
    torch.cuda.synchronize()
    e_ms = ev0.elapsed_time(ev1)
    if sharded:
        e_stats[0]["h2d_bytes"] += eng.h2d - h2d0  # slice staging (route packing reads device memory)
    e_updates = (sum(e_glob_n) / world if sharded else sum(s["n_visible"] for s in e_stats))
    e_ms, e_updates = reduce_max_sum(e_ms, e_updates)
    e_value = e_updates / (e_ms / 1e3)
    if restore:
        assert rep.info()["n_edges"] == inf1["n_edges"], "e2e replay diverged from the device-resident leg"

    checks = None
    if args.checks and not sharded:  # freshness checks on the final snapshot (not in updates/s)
        checks = {"timing": "host wall clock of one call after one warm call, incl. D2H of the result"}
        off_h, _, _, ext_h = rep.export()
        ext0 = int(ext_h[int(np.argmax(np.diff(off_h)))]) if len(ext_h) else None  # the top hub
        del off_h, ext_h
        checks["source_ext"] = ext0
        for name, fn in (("bfs", lambda: rep.bfs(ext0)), ("sssp", lambda: rep.sssp(ext0)),
                         ("pagerank_20", lambda: rep.pagerank(0.85, 20))):
            if ext0 is None and name != "pagerank_20":
                continue
            fn()  # warm
            torch.cuda.synchronize()
            t = time.perf_counter()
            fn()
            torch.cuda.synchronize()
            checks[name + "_ms"] = (time.perf_counter() - t) * 1e3

    route = None
    if sharded:
        rb = [s.get("route_bytes", 0) for s in stats]
        xms = [s.get("ms_exchange", 0.0) for s in stats]
        route = {"bytes_per_step_this_rank": sum(rb) / len(rb), "ms_per_step_this_rank": sum(xms) / len(xms),
                 "exchange": args.exchange, "backend": args.dist_backend}
        route["achieved_gbs"] = (route["bytes_per_step_this_rank"] / (route["ms_per_step_this_rank"] / 1e3) / 1e9
                                 if route["ms_per_step_this_rank"] > 0 else None)
        route["peak_gbs"] = 900.0
        route["peak_source"] = "NVLink 5 per direction per GPU (nominal, north_star)"
        route["frac"] = route["achieved_gbs"] / 900.0 if route["achieved_gbs"] else None
        route["note"] = ("bytes = 40-byte route records this rank sends to other ranks; time = CUDA events "
                         "around pack + exchange on the replica stream (rank 0)")

    if rank == 0:
        peak, peak_src = peaks()
        mean = lambda key: sum(s[key] for s in stats) / len(stats)  # noqa: E731
        merge_ms = mean("ms_merge")
        merge_bytes = mean("bytes_merge")
        achieved = merge_bytes / (merge_ms / 1e3) / 1e9 if merge_ms > 0 else 0.0
        path_bytes = mean("bytes_alg")
        ms_step = ms / len(stats)
        path_gbs = path_bytes / (ms_step / 1e3) / 1e9
        try:  # DRAM bytes per launch of the same kernel from the committed ncu --set full capture
            traffic = (None if sharded else  # captured for the unsharded merge only
                       json.load(open(os.path.join(ROOT, "profiles", "traffic.json"))).get(args.config))
        except Exception:
            traffic = None
        line = {
            "metric": METRIC, "value": value, "unit": "updates/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_max / args.steps,
            "higher_is_better": True, "scaling": "strong" if sharded else "weak", "vs_baseline": None,
            "dtype": "u32/f32", "data": "synthetic",
            "config": {"workload": wl.describe(), "name": args.config, "parallelism":
                       (f"shard{world} (1D vertex ranges, " + (
                           f"all-to-all routing over {args.dist_backend})" if args.exchange == "alltoall" else
                           "fused pack-and-store into peer CUDA-IPC windows)")
                        if sharded else "replicas" if world > 1 else "single"),
                       "l2": "inputs larger than L2 (CSR ~%.1f GB per step)" % (path_bytes / 1e9)
                       if path_bytes > 2e8 else "L2-resident (C1: latency line, see step_ms)"},
            "replica": {"vertices_start": inf0["n_vertices"], "edges_start": inf0["n_edges"],
                        "vertices_end": inf1["n_vertices"], "edges_end": inf1["n_edges"],
                        "edges_per_step": e_steps,
                        "note": ("node deletes cascade (hub-first, the paper's HiDeg window): the graph shrinks "
                                 "batch to batch" if wl.cfg["kind"] == "ldbc" else "")},
            "step_ms": {"p10": pct(step_ms, 0.1), "p50": pct(step_ms, 0.5), "p90": pct(step_ms, 0.9),
                        "min": min(step_ms), "max": max(step_ms),
                        "how": "CUDA events between consecutive applies on the replica stream (rank 0)"},
            "roofline": {"bound": "hbm", "kernel": "k_merge3", "achieved": achieved, "peak": peak,
                         "unit": "GB/s", "frac": achieved / peak, "traffic": traffic,
                         "traffic_source": "ncu --set full (profiles/traffic.json: dram read+write per launch)",
                         "peak_source": peak_src, "bytes_per_launch": merge_bytes,
                         "ms_per_launch": merge_ms},
            "path": {"bytes_alg_per_step": path_bytes, "achieved_gbs": path_gbs,
                     "frac_of_peak": path_gbs / peak,
                     "phase_ms": {k: mean(k) for k in ("ms_ingest", "ms_nodeops", "ms_sort_reduce",
                                                      "ms_merge", "ms_degree_scan", "ms_total")},
                     "setup_s": setup_s},
            "gpu_launches": int(sum(s["n_launches"] for s in stats)),
            "e2e": {"value": e_value, "unit": "updates/s",
                    "how": ("pinned host batches; h2tap_batch_stage copies batch k+1 while batch k is applied"
                            if pipelined else "pinned host batches copied inside each apply") + "; " + e_how_state,
                    "h2d_bytes_per_step": int(sum(s["h2d_bytes"] for s in e_stats) / len(e_stats)),
                    "d2h_bytes_per_step": int(sum(s["d2h_bytes"] for s in e_stats) / len(e_stats))},
            "clocks": clk.summary(),
            "host": host_info(),
            "paper_context": {"what": "the paper's propagation of 2,014,347 SF10 deltas: scan 2595.95 ms + Algorithm 2 "
                                      "merge into the CPU CSR 2064.44 ms = 4660.39 ms (~432 K deltas/s), then 720.64 ms "
                                      "to copy the CSR to an A100 over PCIe 4.0",
                              "hardware": "2x AMD EPYC 7F52 + 1x A100 40 GB", "source": "PAPER.md P:L1899, "
                              "P:L1913, P:L1933-1936", "note": "context, not a target: other hardware, deltas "
                                                               "not flat ops"},
        }
        if route:
            line["nvlink"] = route
        if records:
            line["config"]["input"] = "delta records (paper §5.1 layout, h2tap_delta_apply_records)"
        if args.tombstone:
            line["config"]["id_mode"] = "tombstone rows (reading A23)"
        if checks:
            line["checks"] = checks
        if not args.no_cpu_baseline and world == 1:
            line["cpu_baseline"] = o3_baseline(args.config)
        print(json.dumps(line), flush=True)
    rep.close()
    if world > 1:
        dist.destroy_process_group()


def cpu_baseline_dyn(args, scale: int = 16, cycles: int = 3):
    """cpu_baseline leg of --replica dyn: OD (oracle/od_dynamic.py: Algorithm 1 on Python dicts,
    as it stands - an oracle-only reference, not a tuned CPU implementation) on a bounded
    sample of the SAME generator as the GPU run (bench_dyn.workload: configs[2]'s update mix as
    delta records, plus the same share of NODE_DELETE records) on an RMAT-16 graph, one thread.
    Updates are counted as the GPU counts n_visible (expanded inserts + deletes + node ops)."""
    import types
    import bench_dyn
    from oracle.od_dynamic import DynamicOracle
    n = 1 << scale
    src, dst, w = synth.rmat_edges(scale, synth.seed_of("c3"), n=16 * n)
    o = DynamicOracle(np.arange(n, dtype=np.uint64), src, dst, w)
    batch = max(1000, args.batch >> (args.scale - scale))
    nd = max(1, args.node_deletes * batch // args.batch) if args.node_deletes else 0
    sub = types.SimpleNamespace(scale=scale, batch=batch, node_deletes=nd)
    items, t = 0, 0.0
    for k in range(cycles):
        rb, _ = bench_dyn.workload(sub, n, k)
        t0 = time.perf_counter()
        o.apply_records(rb.records, rb.inserts, rb.weights, rb.deletes)
        t += time.perf_counter() - t0
        r = rb.records
        items += int(r["ins_cnt"].sum() + r["del_cnt"].sum() + r["inserted"].sum() + r["deleted"].sum())
    return {"value": items / t, "unit": "updates/s", "cores": 1, "kind": "oracle",
            "sample": (f"OD (Python dict oracle, as it stands) on RMAT-{scale} x16, {cycles} cycles of the GPU "
                       f"run's generator at {batch} updates (+ {nd} node deletes) per cycle, apply only")}


def run_store(args):
    """--input store: the paper's append-only delta store (h2tap_ds_*) feeds every cycle.  The
    producer (untimed: the update-storage phase of committing transactions)
    commits batch k+1's deltas before cycle k; a cycle (h2tap_delta_apply_store) copies what
    it has not mirrored yet, scans, expands and applies, and its read-ahead copy of batch
    k+1 overlaps it.  Timed: the sum of the cycles (CUDA events around each call)."""
    import torch
    import paper_conf_edbt_jibrilabs23_b200 as h2
    torch.cuda.set_device(0)
    stream = torch.cuda.current_stream()
    wl = Workload(args.config)
    nv, ids, src, dst, w = wl.graph()
    rep = h2.Replica.from_edges(nv, ids, src, dst, w, 0, device=0)
    del src, dst, w
    store = h2.DeltaStore(0)
    n_total = args.warmup + args.steps
    batches = [wl.batch(k) for k in range(n_total + 1)]
    snaps = [int(b.ts.max()) for b in batches]  # (a max over the batch: outside the timed region)
    rbs = []
    for b in batches:
        rb = synth.records_from_ops(b)
        rbs.append(synth.RecordBatch(rb.records, rb.inserts, rb.weights.astype(np.float64), rb.deletes))
    store.append_records(rbs[0])
    stats, ms = [], []
    with ClockSampler(0) as clk:
        for k in range(n_total):
            store.append_records(rbs[k + 1])        # committed before the cycle (untimed)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record(stream)
            st = rep.apply_store(store, snaps[k])
            store.join(stream)                      # the cycle's read-ahead copy is inside the timing
            e1.record(stream)
            torch.cuda.synchronize()
            if k >= args.warmup:
                stats.append(st)
                ms.append(e0.elapsed_time(e1))
    upd = sum(s["n_visible"] for s in stats)
    value = upd / (sum(ms) / 1e3)
    rec_bytes = sum(r.records.nbytes + r.inserts.nbytes + r.weights.nbytes + r.deletes.nbytes for r in rbs) / len(rbs)
    line = {"metric": METRIC, "value": value, "unit": "updates/s", "n_gpus": 1, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": sum(ms) / len(ms), "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32/f32 (8-byte weights in the store, narrowed RN)", "data": "synthetic",
            "config": {"workload": wl.describe(), "name": args.config,
                       "input": "append-only delta store (h2tap_ds_*, §5.1): 48-byte records + inserts / 8-byte "
                                "weights / deletes in pinned host chunks, mirrored to the GPU by the cycle"},
            "step_ms": {"p10": pct(ms, 0.1), "p50": pct(ms, 0.5), "p90": pct(ms, 0.9)},
            "e2e": {"value": value, "unit": "updates/s",
                    "h2d_bytes_per_step": int(sum(s["h2d_bytes"] for s in stats) / len(stats)),
                    "d2h_bytes_per_step": int(sum(s["d2h_bytes"] for s in stats) / len(stats)),
                    "how": "store on the host; every byte of it crosses to the GPU inside the timed cycles "
                           "(read-ahead of batch k+1 overlaps cycle k; a cycle's timing ends when both "
                           "its replica work and its read-ahead copy are complete)"},
            "store_bytes_per_batch": rec_bytes,
            "gpu_launches": int(sum(s["n_launches"] for s in stats)),
            "phase_ms": {k: sum(s[k] for s in stats) / len(stats) for k in ("ms_ingest", "ms_merge", "ms_total")},
            "clocks": clk.summary()}
    print(json.dumps(line), flush=True)
    store.close()
    rep.close()


def spawn(args) -> int:
    """--gpus N > 1 without a launcher: start N ranks of this script (one per GPU) with
    torch.distributed.run on 127.0.0.1; rank 0 prints the line."""
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default=None, choices=sorted(synth.CONFIGS),
                    help="default: c2 (BASELINE.json configs[1], the metric's config) on 1 GPU; c4 "
                         "(configs[3], RMAT-26, the scaling config) when --gpus > 1")
    ap.add_argument("--impl", default="h2tap", choices=["h2tap", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--input", default="ops", choices=["ops", "records", "store"],
                    help="batch format: flat op SoA (h2tap_delta_apply), the paper's delta records "
                         "(h2tap_delta_apply_records, §5.1 layout), or the append-only delta store "
                         "(h2tap_ds_* + h2tap_delta_apply_store, 1 GPU)")
    ap.add_argument("--exchange", default="alltoall", choices=["alltoall", "p2p"],
                    help="sharded exchange: pack + all-to-all (NCCL), or the fused pack-and-store kernel "
                         "into peers' CUDA-IPC windows (h2tap_route_pack_p2p)")
    ap.add_argument("--sync-apply", action="store_true",
                    help="time h2tap_delta_apply (each call returns after its cycle) instead of "
                         "h2tap_delta_apply_async (cycles enqueued back to back)")
    ap.add_argument("--tombstone", action="store_true",
                    help="tombstone-row replica (deleted nodes keep an empty row; reading A23)")
    ap.add_argument("--checks", action="store_true",
                    help="after the timed region, time the freshness checks (BFS, SSSP, PageRank) once")
    ap.add_argument("--parallelism", default="shard", choices=["shard", "replicas"],
                    help="N > 1: shard one graph (default) or run independent replicas")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo lets several ranks share one GPU (testing)")
    ap.add_argument("--replica", default="csr", choices=["csr", "dyn"],
                    help="dyn: the dynamic hash-table replica (Algorithm 1; bench_dyn.py) on configs[2]'s graph")
    import bench_dyn
    bench_dyn.add_args(ap)
    args = ap.parse_args()
    if args.config is None:
        args.config = "c2" if args.gpus == 1 else "c4"
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        raise SystemExit(spawn(args))
    if int(os.environ.get("WORLD_SIZE", "1")) != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={os.environ.get('WORLD_SIZE')}")
    if args.replica == "dyn":
        if args.impl != "h2tap" or args.gpus != 1:
            raise SystemExit("--replica dyn: single GPU, own implementation only")
        args.warmup = max(args.warmup, 3)
        line = bench_dyn.measure(args)
        if not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_baseline_dyn(args)
        print(json.dumps(line))
        return
    if args.warmup < 3 and args.impl == "h2tap":
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    elif args.input == "store":
        run_store(args)
    else:
        run_gpu(args)


if __name__ == "__main__":
    main()
