"""The dynamic replica on B200 (Algorithm 1, §5.4
P:L775-822) beside the CSR merge on the same graph: the paper's point is that a hash-table
replica ingests a batch in O(batch) where the CSR merge rewrites O(E), at the price of a
materialisation for reads.

Graph: configs[2]'s RMAT-24 (16 edges per vertex), device-resident.  Per cycle: configs[2]'s
update stream (the CSR bench's batches: 80% EDGE_INSERT, 20% EDGE_DELETE of initial edges -
deletes hit) in the delta-record layout, `--node-deletes` adds NODE_DELETE records (each
cycle with one costs a pass over every table); applied with h2tap_dyn_apply_records from
device memory (CUDA events around the call), then an e2e leg from pinned host records staged
by the library.  Reads (BFS / SSSP / PageRank) run on the tables in place and, for
comparison, on the same graph loaded into a CSR replica.  One JSON line; the round's copy
lives in profiles/.

usage: python bench.py --replica dyn [--scale 24] [--batch 1000000] [--cycles 5] [--node-deletes 0]
       (adds the OD cpu_baseline); python bench_dyn.py ... prints the GPU part alone
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def add_args(ap):
    ap.add_argument("--scale", type=int, default=24)
    ap.add_argument("--batch", type=int, default=1_000_000, help="updates per cycle (configs[2]'s mix)")
    ap.add_argument("--cycles", type=int, default=5)
    ap.add_argument("--node-deletes", type=int, default=0,
                    help="NODE_DELETE records added to every cycle (each costs the cascade pass)")


def workload(args, n, k):
    """cycle k: configs[2]'s update stream (80% EDGE_INSERT of fresh RMAT pairs, 20% EDGE_DELETE
    of initial edges, so deletes hit existing edges) in the paper's delta-record layout, plus
    --node-deletes NODE_DELETE records of random vertices"""
    b = synth.rmat_batch(args.scale, synth.seed_of("c3"), 100 + k, args.batch, 16 * n, p_insert=0.8, ts_base=k << 24)
    if args.node_deletes:
        rng = np.random.default_rng([k, 77])
        v = rng.integers(0, n, args.node_deletes).astype(np.uint64)
        t = np.full(args.node_deletes, int(b.ts.max()) + 1, np.uint64)
        b = b.concat(synth.Batch(np.full(args.node_deletes, synth.NODE_DELETE, np.uint8), v,
                                 np.zeros_like(v), np.zeros(args.node_deletes, np.float32), t))
    rb = synth.records_from_ops(b)
    return rb, int((b.kind == synth.EDGE_DELETE).sum())


def measure(args) -> dict:
    """GPU measurement only (no oracle here: `bench.py --replica dyn` adds the OD cpu_baseline)."""
    import torch
    import paper_conf_edbt_jibrilabs23_b200 as h2
    torch.cuda.set_device(0)
    st = torch.cuda.current_stream()
    n = 1 << args.scale
    src, dst, w = synth.rmat_edges(args.scale, synth.seed_of("c3"), n=16 * n)
    d = [torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a).cuda() for a in (src, dst, w)]
    del src, dst, w
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    t0 = time.time()
    g = h2.DynReplica.from_edges(n, None, *d)
    torch.cuda.synchronize()
    create_s = time.time() - t0
    del d
    inf0 = g.info()
    tens = lambda a: torch.from_numpy(a.view(np.uint8) if a.dtype.fields else a.view(np.int64) if a.dtype == np.uint64 else a)  # noqa: E731
    n_dev = args.warmup + args.cycles
    batches, host, dels = [], [], []
    for k in range(n_dev + args.cycles):
        rb, nd = workload(args, n, k)
        t = [tens(a) for a in (rb.records, rb.inserts, rb.weights, rb.deletes)]
        if k < n_dev:
            batches.append(synth.RecordBatch(*(x.cuda() for x in t)))
            dels.append(nd)
        else:   # the e2e leg: pinned host records staged by the library
            host.append(synth.RecordBatch(*(x.pin_memory() for x in t)))
    ms, lib_ms, items, sts, casc, hit = [], [], [], [], [], []
    for k, rb in enumerate(batches):
        torch.cuda.synchronize()
        ev0.record(st)
        s = g.apply_records(rb)
        ev1.record(st)
        torch.cuda.synchronize()
        if k >= args.warmup:
            ms.append(ev0.elapsed_time(ev1))
            lib_ms.append(s["ms_total"])
            items.append(s["n_visible"])
            sts.append(s)
            hit.append(s["n_del"] / max(1, dels[k]))
            if s["bytes_merge"]:
                casc.append((s["bytes_merge"], s["ms_merge"]))
    # e2e leg through the library's staging (h2tap_dyn_stage): batch k+1's records are copied on
    # the copy stream while batch k is applied; all copies inside one timed region
    torch.cuda.synchronize()
    ev0.record(st)
    e2e_items, h2d_b, d2h_b = 0, 0, 0
    staged = g.stage(host[0])
    for k in range(len(host)):
        nxt = g.stage(host[k + 1]) if k + 1 < len(host) else None
        s = g.apply_records(staged)
        e2e_items += s["n_visible"]
        h2d_b += s["h2d_bytes"]
        d2h_b += s["d2h_bytes"]
        staged = nxt
    ev1.record(st)
    torch.cuda.synchronize()
    e2e_ms = ev0.elapsed_time(ev1)
    # reads on the tables in place vs the same graph as a CSR replica (Table 1's analytics)
    off, cols, ww, ext, live = g.export()
    hub = int(ext[int(np.argmax(np.diff(off)))])
    csr = h2.Replica.from_csr(off, cols, ww, ext)
    del off, cols, ww
    reads = {}
    for name, fd, fc in (("bfs", lambda: g.bfs(hub), lambda: csr.bfs(hub)),
                         ("sssp", lambda: g.sssp(hub), lambda: csr.sssp(hub)),
                         ("pagerank_20", lambda: g.pagerank(0.85, 20), lambda: csr.pagerank(0.85, 20))):
        for tag, fn in (("dyn", fd), ("csr", fc)):
            fn()
            torch.cuda.synchronize()
            t = time.perf_counter()
            fn()
            torch.cuda.synchronize()
            reads[f"{name}_{tag}_ms"] = (time.perf_counter() - t) * 1e3
        reads[f"{name}_dyn_over_csr"] = reads[f"{name}_dyn_ms"] / reads[f"{name}_csr_ms"]
    csr.close()
    tot_items, tot_ms = sum(items), sum(ms)
    line = {
        "metric": "delta updates/sec ingested into the dynamic (per-vertex hash-table) replica",
        "value": tot_items / (tot_ms / 1e3), "unit": "updates/s", "ms_per_cycle": tot_ms / len(ms),
        "device_ms_per_cycle": sum(lib_ms) / len(lib_ms), "updates_per_cycle": tot_items / len(items),
        "cycles": len(ms), "warmup": args.warmup,
        "config": {"workload": f"configs[2]: RMAT-{args.scale} x16, {args.batch}-update cycles (80% EDGE_INSERT of "
                               f"fresh RMAT pairs, 20% EDGE_DELETE of initial edges) as delta records"
                               + (f", + {args.node_deletes} NODE_DELETE records per cycle" if args.node_deletes else ""),
                   "inputs": "device-resident records"},
        "delete_hit_rate": sum(hit) / len(hit),
        "graph": {"vertices": inf0["n_vertices"], "edges": inf0["n_edges"], "table_slots": inf0["table_slots"]},
        "e2e": {"value": e2e_items / (e2e_ms / 1e3), "unit": "updates/s",
                "h2d_bytes_per_step": h2d_b / len(host), "d2h_bytes_per_step": d2h_b / len(host),
                "how": "pinned host records staged by the library (h2tap_dyn_stage: batch k+1 copied on the copy "
                       "stream while batch k is applied); one timed region over all cycles"},
        "reads": dict(reads, how="host wall clock of one call after a warm call, incl. D2H of the result; source = "
                                 "the top hub; csr = the same graph in a CSR replica (h2tap_replica_create_from_csr)"),
        "create_s": create_s,
        "last_cycle": {k: sts[-1][k] for k in ("n_new", "n_upd", "n_del", "n_casc", "n_gated",
                                                "n_vertex_inserted", "n_vertex_deleted", "n_launches")},
    }
    if casc:   # node-delete cycles: the cascade pass streams every table once
        pk = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
        peak = float(pk["hbm_gbs"])
        b = sum(x[0] for x in casc) / len(casc)
        t = sum(x[1] for x in casc) / len(casc)
        line["roofline"] = {"bound": "hbm", "kernel": "k_dyn_cascade", "achieved": b / (t * 1e-3) / 1e9,
                            "peak": peak, "unit": "GB/s", "frac": b / (t * 1e-3) / 1e9 / peak,
                            "traffic": None, "bytes_per_launch": b, "ms_per_launch": t,
                            "peak_source": "measured (MEASURED_PEAKS.json hbm_gbs)"}
    return line


def main():
    ap = argparse.ArgumentParser()
    add_args(ap)
    ap.add_argument("--warmup", type=int, default=3)
    print(json.dumps(measure(ap.parse_args())))


if __name__ == "__main__":
    main()
