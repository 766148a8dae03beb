"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list:
per kernel launches, total / average ms and share of the listed GPU time."""
import csv, sys, collections

rows = list(csv.reader(l for l in open(sys.argv[1]) if not l.startswith("==")))
hdr = rows[0]
ki, mi, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
agg = collections.defaultdict(lambda: [0, 0.0])
for r in rows[1:]:
    if len(r) <= vi or r[mi] != "gpu__time_duration.sum":
        continue
    v = float(r[vi].replace(",", ""))
    v = v / 1e6 if r[ui] == "ns" else v / 1e3 if r[ui] == "us" else v * 1e3 if r[ui] == "s" else v
    agg[r[ki]][0] += 1
    agg[r[ki]][1] += v
tot = sum(t for _, t in agg.values())
print("kernel, launches, total_ms, avg_ms, share")
for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{k}, {n}, {t:.2f}, {t / n:.3f}, {t / tot:.4f}")
