"""The dynamic replica on B200 (Algorithm 1, §5.4
P:L775-822) beside the CSR merge on the same graph: the paper's point is that a hash-table
replica ingests a batch in O(batch) where the CSR merge rewrites O(E), at the price of a
materialisation for reads.

Graph: configs[2]'s RMAT-24 (16 edges per vertex), device-resident.  Per cycle: a seeded
delta-record batch (synth.dyn_record_batch: ~1/2 inserts, ~1/2 deletes per record, a few
new nodes; `--node-deletes` adds deleted-node records, which cost one pass over the table)
applied with h2tap_dyn_apply_records from device memory; device time from the library's
events (stats.ms_total) and CUDA events around the call.  Also timed: one CSR
materialisation (h2tap_dyn_export to device buffers... here host arrays, reported apart).
One JSON line; the round's copy lives in profiles/.

usage: python bench.py --replica dyn [--scale 24] [--records 500000] [--cycles 5] [--node-deletes 0.0]
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
    ap.add_argument("--records", type=int, default=500_000)
    ap.add_argument("--cycles", type=int, default=5)
    ap.add_argument("--node-deletes", type=float, default=0.0)


def measure(args) -> dict:
    """GPU measurement only (no oracle here: `bench.py --replica dyn` adds the OD cpu_baseline)."""
    import torch
    import paper_conf_edbt_jibrilabs23_b200 as h2
    torch.cuda.set_device(0)
    st = torch.cuda.current_stream()
    n = 1 << args.scale
    src, dst, w = synth.rmat_edges(args.scale, synth.seed_of("c3"), n=16 * n)
    d = [torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a).cuda() for a in (src, dst, w)]
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    t0 = time.time()
    g = h2.DynReplica.from_edges(n, None, *d)
    torch.cuda.synchronize()
    create_s = time.time() - t0
    inf0 = g.info()
    batches, host = [], []
    xid = n - 1
    for k in range(2 * (args.warmup + args.cycles)):
        rb = synth.dyn_record_batch(synth.seed_of("c3"), 1000 + k, xid, args.records, n_new=64, max_slice=2,
                                    p_deleted=args.node_deletes, p_new=0.0005, p_invalid=0.0)
        t = (torch.from_numpy(rb.records.view(np.uint8)), torch.from_numpy(rb.inserts.view(np.int64)),
             torch.from_numpy(rb.weights), torch.from_numpy(rb.deletes.view(np.int64)))
        if k < args.warmup + args.cycles:
            batches.append(synth.RecordBatch(*(x.cuda() for x in t)))
        else:   # the e2e leg: pinned host records, the H2D copy inside the timed call
            host.append(synth.RecordBatch(*(x.pin_memory() for x in t)))
        xid += 64
    ms, lib_ms, items, sts, casc = [], [], [], [], []
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
            if s["bytes_merge"]:
                casc.append((s["bytes_merge"], s["ms_merge"]))
    # e2e leg, pipelined through the public API: batch k+1's records are copied from pinned host
    # memory into one of two device slots on a copy stream while batch k is applied; every copy
    # of the timed cycles is inside the timed region (one region over all of them)
    cs = torch.cuda.Stream()
    slots = [None, None]
    evs = [torch.cuda.Event(), torch.cuda.Event()]

    def stage(k):
        with torch.cuda.stream(cs):
            slots[k % 2] = synth.RecordBatch(*(x.to("cuda", non_blocking=True) for x in
                                               (host[k].records, host[k].inserts, host[k].weights, host[k].deletes)))
            evs[k % 2].record(cs)

    def run(lo, hi):
        items, h2d_b, d2h_b = 0, 0, 0
        stage(lo)
        for k in range(lo, hi):
            st.wait_event(evs[k % 2])
            cur = slots[k % 2]
            if k + 1 < hi:
                cs.wait_stream(st)          # slot (k+1)%2 was last read by apply k-1
                stage(k + 1)
            s = g.apply_records(cur)
            items += s["n_visible"]
            h2d_b += sum(int(x.numel() * x.element_size()) for x in
                         (host[k].records, host[k].inserts, host[k].weights, host[k].deletes))
            d2h_b += s["d2h_bytes"]
        return items, h2d_b, d2h_b

    run(0, args.warmup)
    torch.cuda.synchronize()
    ev0.record(st)
    e2e_items, h2d_b, d2h_b = run(args.warmup, len(host))
    ev1.record(st)
    torch.cuda.synchronize()
    e2e_ms = ev0.elapsed_time(ev1)
    n_e2e = len(host) - args.warmup
    torch.cuda.synchronize()
    t0 = time.time()
    g.bfs(0)    # a read on the dynamic replica: CSR materialisation + BFS (Table 1's check)
    bfs_s = time.time() - t0
    torch.cuda.synchronize()
    t0 = time.time()
    out = g.export()
    export_s = time.time() - t0
    tot_items, tot_ms = sum(items), sum(ms)
    line = {
        "metric": "delta updates/sec ingested into the dynamic (hash-table) replica",
        "value": tot_items / (tot_ms / 1e3), "unit": "updates/s", "ms_per_cycle": tot_ms / len(ms),
        "device_ms_per_cycle": sum(lib_ms) / len(lib_ms), "updates_per_cycle": tot_items / len(items),
        "cycles": len(ms), "warmup": args.warmup,
        "config": {"workload": f"RMAT-{args.scale} x16 (configs[2] graph), {args.records} delta records per "
                               f"cycle (<=2 inserts + <=2 deletes each), node-delete records p={args.node_deletes}",
                   "inputs": "device-resident records"},
        "graph": {"vertices": inf0["n_vertices"], "edges": inf0["n_edges"], "table_slots": inf0["table_slots"]},
        "e2e": {"value": e2e_items / (e2e_ms / 1e3), "unit": "updates/s",
                "h2d_bytes_per_step": h2d_b / n_e2e, "d2h_bytes_per_step": d2h_b / n_e2e,
                "note": "records in pinned host memory; the next cycle's records are copied on a copy "
                        "stream into one of two device slots while the current cycle is applied; one timed "
                        "region over all cycles (copies included)"},
        "create_s": create_s, "bfs_with_materialisation_s": bfs_s, "export_host_s": export_s, "export_edges": int(len(out[1])),
        "last_cycle": {k: sts[-1][k] for k in ("n_new", "n_upd", "n_del", "n_casc", "n_gated",
                                                "n_vertex_inserted", "n_vertex_deleted", "n_launches")},
    }
    if casc:   # node-delete cycles: the cascade pass dominates and is HBM-bound
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
