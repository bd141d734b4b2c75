"""Per-kernel durations of the last apply in an ncu launch list (gpurun_out/launches_<cfg>.csv)."""
import csv, sys
for c in sys.argv[1:] or ("c2", "c3"):
    rows = [r for r in csv.reader(open(f"gpurun_out/launches_{c}.csv")) if len(r) > 10]
    h = rows[0]; ki = h.index("Kernel Name"); vi = h.index("Metric Value"); ui = h.index("Metric Unit")
    data = rows[1:]
    idx = [i for i, r in enumerate(data) if "k_partition" in r[ki]]
    tot = 0
    print(c)
    for r in data[idx[-1]:]:
        v = float(r[vi].replace(",", "")) * (1e-3 if r[ui].startswith("n") else 1e3 if r[ui].startswith("m") else 1)
        tot += v
        print("  %8.1f  %s" % (v, r[ki].split("(")[0][:60]))
    print("  total", round(tot, 1))
