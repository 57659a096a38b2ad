"""Kernel time shares from an ncu launch list (--metrics gpu__time_duration.sum --csv)."""
import collections, csv, re, sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h = rows[0]
ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
agg = collections.defaultdict(lambda: [0, 0.0])
for r in rows[1:]:
    if r[mi] != "gpu__time_duration.sum":
        continue
    name = re.sub(r"\(.*", "", r[ki]).replace("sfk::", "").replace("<unnamed>::", "")
    name = re.sub(r"^void ", "", name)
    a = agg[name]
    a[0] += 1
    a[1] += float(r[vi].replace(",", ""))
tot = sum(a[1] for a in agg.values())
print(f"launches {sum(a[0] for a in agg.values())}, total {tot / 1e3:.1f} us")
print("| kernel | launches | mean us | share |\n|---|---|---|---|")
for name, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1])[:14]:
    print(f"| {name} | {n} | {t / n / 1e3:.1f} | {100 * t / tot:.1f}% |")
