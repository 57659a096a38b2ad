import csv, sys
for m in sys.argv[1:] or ["1", "0"]:
    rows = [r for r in csv.reader(open(f"gpurun_out/infer_{m}.csv")) if len(r) > 10]
    h = rows[0]; ki, mi, vi, ii = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
    by = {}
    for r in rows[1:]:
        by.setdefault(r[ii], {"k": r[ki]})[r[mi]] = r[vi]
    seq = list(by.values())[-10:]
    tot = 0
    print("mode", m)
    for d in seq:
        t = float(d.get("gpu__time_duration.sum", 0)); tot += t
        print(f"   {d['k'][:58]:58s} {t/1e3:7.2f} us  {float(d.get('dram__bytes_read.sum', 0))/1e6:8.2f} MB")
    print("   sum", tot / 1e3)
