"""Attribute ncu SASS-level instruction/stall counts to CUDA source lines via nvdisasm line info.
usage: python tools_sass_lines.py <report.ncu-rep> <mangled-function-prefix> [top]"""
import collections, csv, os, re, subprocess, sys, tempfile
rep, fn = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath("paper_conf_edbt_jibrilabs23_b200/libh2tap.so")], cwd=d, capture_output=True)
cub = [f for f in os.listdir(d) if f.endswith(".cubin")][0]
sass = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(d, cub)], capture_output=True, text=True).stdout.split("\n")
start = next(i for i, l in enumerate(sass) if l.startswith(".text." + fn))
cur = None; a2l = {}
for l in sass[start + 1:]:
    if l.startswith(".text."): break
    m = re.search(r'//## File "(.*?)", line (\d+)', l)
    if m: cur = (os.path.basename(m.group(1)), int(m.group(2))); continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", l)
    if m: a2l[int(m.group(1), 16)] = cur
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = rows[1]; ia = hdr.index("Address"); ie = hdr.index("Instructions Executed"); iw = hdr.index("Warp Stall Sampling (All Samples)")
data = rows[2:]; base = int(data[0][ia], 16)
agg = collections.Counter(); st = collections.Counter()
for r in data:
    k = a2l.get(int(r[ia], 16) - base)
    agg[k] += float(r[ie] or 0); st[k] += float(r[iw] or 0)
tot = sum(agg.values()) or 1; tst = sum(st.values()) or 1
srcs = {}
def line(k):
    if not k: return "?"
    f, n = k
    if f not in srcs:
        p = os.path.join("paper_conf_edbt_jibrilabs23_b200/csrc", f)
        srcs[f] = open(p).read().split("\n") if os.path.exists(p) else []
    return srcs[f][n - 1].strip()[:90] if n <= len(srcs[f]) else "?"
keys = sorted(set(agg) | set(st), key=lambda k: -(st[k] / tst + agg[k] / tot))
for k in keys[:top]:
    print("%-22s %5.1f%% inst %5.1f%% stall | %s" % (("%s:%d" % k) if k else "?", 100 * agg[k] / tot, 100 * st[k] / tst, line(k)))
