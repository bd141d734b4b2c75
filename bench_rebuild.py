"""Rebuild-vs-merge cost model on B200 (the paper's §6.4,
P:L1738-1811, proposes choosing between rebuilding the CSR and merging deltas but
leaves the evaluation open).

rebuild(E)   = h2tap_replica_create_from_edges over the graph's E edges, device-resident
               (the GPU analogue of the paper's "rebuild the CSR")
merge(E, B)  = one h2tap_delta_apply of a B-op batch (80/20 insert/delete) into the
               same graph (device-resident batch)
Both timed with CUDA events after a warm call, RMAT (configs[2] shape by default).  The
crossover batch size B* solves merge(E, B*) = rebuild(E) on a least-squares line
merge = a + b*B fitted over the measured batch sizes.  One JSON line; the round's copy
lives in profiles/.

usage: python bench_rebuild.py [--scale 24] [--sizes 10000,100000,1000000,4000000,16000000]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
import synth  # noqa: E402


def main():
    import torch
    import paper_conf_edbt_jibrilabs23_b200 as h2
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=24)
    ap.add_argument("--sizes", default="10000,100000,1000000,4000000,16000000")
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    torch.cuda.set_device(0)
    st = torch.cuda.current_stream()
    seed = synth.seed_of("c3")
    n = 1 << args.scale
    src, dst, w = synth.rmat_edges(args.scale, seed, n=16 * n)
    m = len(src)
    d_src, d_dst, d_w = (torch.from_numpy(src.view(np.int64)).cuda(), torch.from_numpy(dst.view(np.int64)).cuda(),
                         torch.from_numpy(w).cuda())
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)

    def timed(fn):
        torch.cuda.synchronize()
        ev0.record(st)
        out = fn()
        ev1.record(st)
        torch.cuda.synchronize()
        return ev0.elapsed_time(ev1), out

    rb = []
    for r in range(args.reps + 1):
        ms, rep = timed(lambda: h2.Replica.from_edges(n, None, d_src, d_dst, d_w, 0))
        if r:
            rb.append(ms)
        E = rep.info()["n_edges"]
        if r < args.reps:
            rep.close()
    rebuild = float(np.median(rb))
    del d_src, d_dst, d_w
    sizes = [int(x) for x in args.sizes.split(",")]
    merge = {}
    k = 0
    ts = 0
    for B in sizes:
        t = []
        for r in range(args.reps + 1):
            b = synth.rmat_batch(args.scale, seed, 1000 + k, B, m, p_insert=0.8, ts_base=ts)
            k += 1
            ts = int(b.ts.max())
            db = synth.Batch(*(torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a).cuda()
                               for a in (b.kind, b.src, b.dst, b.w, b.ts)))
            ms, _ = timed(lambda: rep.apply(db, ts))
            if r:
                t.append(ms)
        merge[B] = float(np.median(t))
    x = np.array(sizes, float)
    y = np.array([merge[B] for B in sizes])
    b_, a_ = np.polyfit(x, y, 1)
    cross = (rebuild - a_) / b_ if b_ > 0 else float("inf")
    print(json.dumps({
        "what": "rebuild-vs-merge cost model (RMAT scale-%d, %d generated edges, %d unique)" % (args.scale, m, E),
        "rebuild_ms": rebuild, "merge_ms": {str(B): merge[B] for B in sizes},
        "fit_merge_ms": {"a_ms": a_, "b_ms_per_op": b_},
        "crossover_batch_ops": cross, "crossover_over_E": cross / E,
        "timing": "CUDA events around the call, median of %d after a warm call; device-resident inputs" % args.reps,
    }))


if __name__ == "__main__":
    main()
