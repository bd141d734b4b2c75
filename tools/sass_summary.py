"""SASS evidence for the hot kernels of libh2tap.so (no GPU needed): per kernel, the
instruction count, registers / shared memory from the cubin, and the mnemonics that show
the data-movement design - UBLKCP (cp.async.bulk = TMA bulk copy), SYNCS (mbarrier),
LDGSTS (cp.async), MATCH (warp match_any), LDG.E.128 / STG.E.128 (16-byte accesses),
ATOMG / REDG / ATOMS (global / shared atomics), BAR (CTA barriers).
usage: python tools/sass_summary.py [kernel-substring ...] > profiles/<round>/sass_summary.txt"""
import collections
import re
import subprocess
import sys

LIB = "paper_conf_edbt_jibrilabs23_b200/libh2tap.so"
want = sys.argv[1:] or ["k_merge3", "rs_coop", "rs_onesweep", "k_reduce_classify", "k_edge_prep", "k_partition",
                        "k_rows_fused", "k_casc_cols", "k_dyn_cascade", "k_dyn_upsert", "k_dyn_bfs_expand",
                        "k_rec_expand"]
sass = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True).stdout
res = subprocess.run(["cuobjdump", "-res-usage", LIB], capture_output=True, text=True).stdout
usage = {}
for m in re.finditer(r"Function (\S+):\s*\n\s*REG:(\d+) STACK:(\d+) SHARED:(\d+)", res):
    usage[m.group(1)] = (int(m.group(2)), int(m.group(3)), int(m.group(4)))
funcs = re.split(r"\n\s*Function : ", sass)[1:]
keys = ["UBLKCP", "SYNCS", "LDGSTS", "MATCH", "LDG.E.128", "STG.E.128", "LDG.E.64", "LDS", "STS", "ATOMG", "REDG",
        "ATOMS", "BAR", "SHFL", "VOTE", "POPC"]
print(f"# SASS summary of {LIB} (cuobjdump -sass, sm_100a)\n")
for f in funcs:
    name = f.split("\n", 1)[0].strip()
    demangled = subprocess.run(["c++filt", name], capture_output=True, text=True).stdout.strip()
    if not any(w in demangled for w in want):
        continue
    ins = re.findall(r"/\*[0-9a-f]{4}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)", f)
    cnt = collections.Counter()
    for i in ins:
        for k in keys:
            if i == k or i.startswith(k + ".") or (k.endswith("128") and i.startswith(k[:-4]) and ".128" in i) or \
               (k == "LDG.E.64" and i.startswith("LDG.E.64")):
                cnt[k] += 1
    reg, stack, shm = usage.get(name, (None, None, None))
    print(f"{demangled[:110]}")
    print(f"   instructions {len(ins)}, registers {reg}, stack {stack} B, static smem {shm} B")
    print("   " + ", ".join(f"{k} {cnt[k]}" for k in keys if cnt[k]))
