"""Summarise an ncu launch list (gpu__time_duration.sum per launch) per kernel for the last N launches."""
import collections, csv, sys
path = sys.argv[1]; last = int(sys.argv[2]) if len(sys.argv) > 2 else 200
rows = [r for r in csv.reader(open(path)) if len(r) > 10]
hdr = rows[0]; ki = hdr.index("Kernel Name"); vi = hdr.index("Metric Value"); ui = hdr.index("Metric Unit")
scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "second": 1e6, "s": 1e6}
agg = collections.OrderedDict(); tot = 0.0
for r in rows[1:][-last:]:
    v = float(r[vi].replace(",", "")) * scale[r[ui]]
    agg.setdefault(r[ki].split("(")[0], []).append(v); tot += v
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
    print("%-45s n=%3d mean=%9.1f us  share=%5.1f%%" % (k[:45], len(v), sum(v) / len(v), 100 * sum(v) / tot))
print("total %.1f us over %d launches" % (tot, sum(len(v) for v in agg.values())))
