"""Per-launch table of an ncu report (--page raw): kernel, duration, DRAM bytes, grid, SM /
tensor-pipe / DRAM utilisation.  python scripts/ncu_report_table.py REPORT.ncu-rep"""
import csv, io, re, subprocess, sys

raw = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h = rows[0]
units = rows[1]
want = [("gpu__time_duration.sum", "us"), ("dram__bytes_read.sum", "MB rd"), ("dram__bytes_write.sum", "MB wr"),
        ("launch__grid_size", "grid"), ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM %"),
        ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM %"),
        ("sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active", "TC pipe %"),
        ("sm__cycles_active.avg", "SM active cyc")]
idx = {k: h.index(k) for k, _ in want if k in h}
ki = h.index("Kernel Name")
print("| kernel | " + " | ".join(n for k, n in want if k in idx) + " |")
print("|---|" + "---|" * len(idx))
for r in rows[2:]:
    name = re.sub(r"\(.*", "", r[ki]).replace("sfk::", "").replace("<unnamed>::", "").replace("void ", "")
    vals = []
    for k, n in want:
        if k not in idx:
            continue
        v = r[idx[k]].replace(",", "")
        u = units[idx[k]]
        try:
            x = float(v)
            if k == "gpu__time_duration.sum" and u == "nsecond":
                x /= 1e3
            if k.startswith("dram__bytes") and u == "Mbyte":
                pass
            elif k.startswith("dram__bytes") and u == "Kbyte":
                x /= 1e3
            elif k.startswith("dram__bytes") and u == "Gbyte":
                x *= 1e3
            vals.append(f"{x:.1f}")
        except ValueError:
            vals.append(v)
    print(f"| {name} | " + " | ".join(vals) + " |")
