import sys, time, os
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import numpy as np, torch
import paper_conf_edbt_jibrilabs23_b200 as h2
from bench import Workload
import synth
wl = Workload("c3"); nv, ids, src, dst, w = wl.graph()
rep = h2.Replica.from_edges(nv, ids, src, dst, w)
bs = [wl.batch(k) for k in range(16)]
snaps = [int(b.ts.max()) for b in bs]
def pin(b): return synth.Batch(*(torch.from_numpy(a.view(np.int64) if a.dtype == np.uint64 else a).pin_memory() for a in (b.kind, b.src, b.dst, b.w, b.ts)))
P = [pin(b) for b in bs]
for k in range(3): rep.apply(P[k], snaps[k])
torch.cuda.synchronize()
def run(name, f):
    t = time.perf_counter(); f(); torch.cuda.synchronize(); dt = (time.perf_counter() - t) * 1e3
    print(name, "%.3f ms/step" % (dt / 4), flush=True)
it = iter(range(3, 16))
def plain():
    for _ in range(4):
        k = next(it); rep.apply(P[k], snaps[k])
def staged_pipe():
    ks = [next(it) for _ in range(4)]
    s = rep.stage(P[ks[0]])
    for i, k in enumerate(ks):
        n = rep.stage(P[ks[i + 1]]) if i + 1 < 4 else None
        st = rep.apply(s, snaps[k]); s = n
        print({x: round(st[x], 3) for x in ("ms_ingest", "ms_sort_reduce", "ms_merge", "ms_degree_scan", "ms_total")})
def stage_times():
    k = next(it)
    t = time.perf_counter(); s = rep.stage(P[k]); t1 = time.perf_counter(); torch.cuda.synchronize(); t2 = time.perf_counter()
    rep.apply(s, snaps[k]); t3 = time.perf_counter()
    print("stage call %.3f ms, sync %.3f ms, apply %.3f ms" % ((t1 - t) * 1e3, (t2 - t1) * 1e3, (t3 - t2) * 1e3))
run("plain pinned", plain)
run("staged pipeline", staged_pipe)
stage_times(); stage_times()
