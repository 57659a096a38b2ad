"""Summarise an ncu report: key raw metrics + top SASS stall hotspots (source page)."""
import csv, io, subprocess, sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
h, v = r[0], r[2] if len(r) > 2 else r[1]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "launch__grid_size", "launch__block_size",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread"]
for i, k in enumerate(h):
    if k in want or k.startswith("dram__bytes_read.sum.per_second"):
        print(f"{k:60s} {v[i]}")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hh = rows[1]; data = rows[2:]
ai, si, wi = hh.index("Address"), hh.index("Source"), hh.index("Warp Stall Sampling (All Samples)")
tot = sum(float(x[wi] or 0) for x in data) or 1
print("stall samples", tot)
for x in sorted(data, key=lambda x: -float(x[wi] or 0))[:n]:
    print(x[ai][-5:], f"{float(x[wi]) / tot * 100:5.1f}%", x[si][:90])
