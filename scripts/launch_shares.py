"""Per-kernel launch counts, total time and share from an ncu launch-list CSV
(ncu --metrics gpu__time_duration.sum --csv).  python scripts/launch_shares.py csv"""
import collections, csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
h = rows[hdr]
ki, mi, vi, ui = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
scale = {"nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "second": 1e3, "ns": 1e-6, "us": 1e-3, "ms": 1.0}
tot, cnt = collections.OrderedDict(), collections.Counter()
for r in rows[hdr + 1:]:
    if len(r) <= vi or r[mi] != "gpu__time_duration.sum":
        continue
    name = r[ki].split("(")[0]
    tot[name] = tot.get(name, 0.0) + float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0)
    cnt[name] += 1
T = sum(tot.values())
for k, v in tot.items():
    print(f"{k:60s} launches {cnt[k]:4d}  total {v:10.2f} ms  share {100 * v / T:5.1f}%")
