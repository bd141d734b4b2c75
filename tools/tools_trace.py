import sys, os
sys.path.insert(0, '/root/repo')
import numpy as np
import paper_conf_edbt_jibrilabs23_b200 as h2
from bench import Workload
cfg = sys.argv[1]
wl = Workload(cfg); nv, ids, src, dst, w = wl.graph()
rep = h2.Replica.from_edges(nv, ids, src, dst, w)
for k in range(8):
    b = wl.batch(k)
    st = rep.apply(b, int(b.ts.max()))
print("total", st["ms_total"], file=sys.stderr)
