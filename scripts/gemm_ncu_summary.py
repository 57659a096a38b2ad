import csv, collections, sys
for mode in sys.argv[1:]:
    rows = list(csv.reader(open(f'gpurun_out/gemm_{mode}.csv')))
    hi = next(i for i, r in enumerate(rows) if 'Kernel Name' in r)
    h = rows[hi]; data = rows[hi+1:]
    ki, mi, vi, gi, ids = h.index('Kernel Name'), h.index('Metric Name'), h.index('Metric Value'), h.index('Grid Size'), h.index('ID')
    by = collections.defaultdict(dict)
    for r in data:
        by[r[ids]][r[mi]] = float(r[vi].replace(',', '')); by[r[ids]]['grid'] = r[gi]; by[r[ids]]['name'] = r[ki][:40]
    tot = sum(v['gpu__time_duration.sum'] for v in by.values())
    print(mode, "kernels", len(by), "total ms", tot/1e6)
    seen = []
    for k, v in by.items():
        key = (v['grid'], v['name'])
        if key not in [s[0] for s in seen]:
            seen.append((key, v['gpu__time_duration.sum']/1e3, v.get('sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed', 0)))
    for s in seen[:12]:
        print("   ", s[0][1][:38], s[0][0], f"{s[1]:.1f}us tensor {s[2]:.1f}%")
