"""Summarise an ncu --page source --print-source sass CSV: stall reasons and hottest SASS."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
data = rows[2:]
cols = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
tot = {c: sum(float(r[h.index(c)] or 0) for r in data) for c in cols}
T = sum(tot.values())
print("stall reasons (% of samples):")
for c, v in sorted(tot.items(), key=lambda x: -x[1])[:10]:
    print(f"  {c:28s} {100 * v / T:5.1f}%")
wi = h.index("Warp Stall Sampling (All Samples)")
si = h.index("Source")
n = int(sys.argv[2]) if len(sys.argv) > 2 else 15
print("hottest instructions:")
for r in sorted(data, key=lambda r: -float(r[wi] or 0))[:n]:
    print(f"  {100 * float(r[wi]) / T:5.1f}%  {r[si][:100]}")
