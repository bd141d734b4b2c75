"""Per-kernel table of the LAST apply in an ncu launch list (tools/prof.sh output):
duration, DRAM bytes and share of the step.  usage: launch_table.py <launches.csv>"""
import csv
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ki, mi, vi, ui, ii = (h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"),
                      h.index("Metric Unit"), h.index("ID"))
sc = {"ns": 1e-3, "us": 1.0, "ms": 1e3, "nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3, "second": 1e6, "byte": 1, "Kbyte": 1e3, "Mbyte": 1e6,
      "Gbyte": 1e9}
k = {}
order = []
for r in rows[1:]:
    i = int(r[ii])
    if i not in k:
        k[i] = {"name": r[ki].split("(")[0].replace("void ", "")[:48]}
        order.append(i)
    k[i][r[mi]] = float(r[vi].replace(",", "")) * sc.get(r[ui], 1)
starts = [i for i in order if "k_partition" in k[i]["name"] or "k_rec_count" in k[i]["name"]]
last = [i for i in order if i >= starts[-1]]
tot = sum(k[i]["gpu__time_duration.sum"] for i in last)
print(f"{'kernel':50s} {'us':>8s} {'share':>6s} {'DRAM MB':>9s} {'GB/s':>7s}")
for i in last:
    d = k[i]
    t = d["gpu__time_duration.sum"]
    b = d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
    print(f"{d['name']:50s} {t:8.1f} {100 * t / tot:5.1f}% {b / 1e6:9.1f} {b / t / 1e3 if t else 0:7.0f}")
print(f"{'total (serialised, cold-cache)':50s} {tot:8.1f}")
