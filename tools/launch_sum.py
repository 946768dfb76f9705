"""Sum an ncu launch list (--metrics gpu__time_duration.sum --csv) by kernel name.

    python tools/launch_sum.py launches.csv
"""
import collections
import csv
import sys

tot = collections.defaultdict(float)
cnt = collections.Counter()
rows = [r for r in csv.reader(open(sys.argv[1])) if r]
hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hdr]
ik, iv, iu = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
scale = {"nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "second": 1e3}
for r in rows[hdr + 1:]:
    name = r[ik].split("(")[0].split("<")[0].replace("void ", "").strip()
    tot[name] += float(r[iv].replace(",", "")) * scale.get(r[iu], 1e-6)
    cnt[name] += 1
all_ms = sum(tot.values())
print(f"{'kernel':40s} {'launches':>9s} {'total ms':>10s} {'mean us':>9s} {'share':>6s}")
for k, v in sorted(tot.items(), key=lambda x: -x[1]):
    print(f"{k[:40]:40s} {cnt[k]:9d} {v:10.3f} {1e3 * v / cnt[k]:9.2f} {100 * v / all_ms:5.1f}%")
print(f"{'total':40s} {sum(cnt.values()):9d} {all_ms:10.3f}")
