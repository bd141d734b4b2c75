"""Create RMAT replicas of growing scale on cuda:0 (robustness at large sizes)."""
import sys, os, time
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import numpy as np, torch
import paper_conf_edbt_jibrilabs23_b200 as h2, synth
for scale, ef in [(int(a.split(":")[0]), int(a.split(":")[1])) for a in sys.argv[1:]]:
    src, dst, w = synth.rmat_edges(scale, 7, n=ef << scale)
    t = time.time()
    try:
        rep = h2.Replica.from_edges(1 << scale, None, src, dst, w)
        print(scale, ef, "ok", rep.info()["n_edges"], "%.1fs" % (time.time() - t), flush=True)
        rep.close()
    except Exception as e:
        print(scale, ef, "FAIL", e, flush=True)
        break
    del src, dst, w
    torch.cuda.empty_cache()
