"""Summarise gpurun_out/ captures into profiles/<round>/ (tracked)."""
import collections, csv, json, os, subprocess, sys
rnd = sys.argv[1] if len(sys.argv) > 1 else "r1"
out = os.path.join("profiles", rnd); os.makedirs(out, exist_ok=True)
scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}
summary = {}
for c in ("c2", "c3"):
    p = f"gpurun_out/launches_{c}.csv"
    if os.path.exists(p):
        rows = [r for r in csv.reader(open(p)) if len(r) > 10]
        hdr = rows[0]; ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
        data = rows[1:]
        subprocess.run(["cp", p, os.path.join(out, f"launches_{c}.csv")])
        # the last 3 applies = the timed steps of the command
        per = collections.OrderedDict(); tot = 0.0
        n = len(data)
        for r in data:
            v = float(r[vi].replace(",", "")) * scale[r[ui]]
            per.setdefault(r[ki].split("(")[0], []).append(v)
        steps = {}
        for k, v in per.items():
            steps[k] = {"launches": len(v), "mean_us": sum(v) / len(v), "total_us": sum(v)}
        summary[f"launches_{c}"] = steps
    rep = f"gpurun_out/ncu_merge_{c}.ncu-rep"
    if os.path.exists(rep):
        raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rr = list(csv.reader(raw.splitlines()))
        h, u = rr[0], rr[1]
        want = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
                "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
                "launch__registers_per_thread", "launch__grid_size", "sm__warps_active.avg.pct_of_peak_sustained_active"]
        d = {}
        for w in want:
            if w in h: d[w] = (rr[2][h.index(w)], u[h.index(w)])
        rb = float(d["dram__bytes_read.sum"][0]) * (1e9 if d["dram__bytes_read.sum"][1] == "Gbyte" else 1e6 if d["dram__bytes_read.sum"][1] == "Mbyte" else 1)
        wb = float(d["dram__bytes_write.sum"][0]) * (1e9 if d["dram__bytes_write.sum"][1] == "Gbyte" else 1e6 if d["dram__bytes_write.sum"][1] == "Mbyte" else 1)
        d["traffic_bytes_per_launch"] = rb + wb
        summary[f"ncu_merge_{c}"] = d
        det = subprocess.run(["ncu", "-i", rep, "--page", "details"], capture_output=True, text=True).stdout
        open(os.path.join(out, f"ncu_merge_{c}_details.txt"), "w").write(det)
json.dump(summary, open(os.path.join(out, "summary.json"), "w"), indent=1)
tr = {c: summary.get(f"ncu_merge_{c}", {}).get("traffic_bytes_per_launch") for c in ("c2", "c3")}
json.dump(tr, open(os.path.join("profiles", "traffic.json"), "w"), indent=1)
print(json.dumps(tr))
