"""Per-CUDA-source-line warp-stall samples of an ncu report (source page, cuda+sass view).

    python tools/ncu_lines.py report.ncu-rep [top_n]
"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
fname, rows = "", []
for r in csv.reader(io.StringIO(txt)):
    if len(r) >= 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if len(r) > 5 and r[0] and r[0] != "Line No":
        try:
            rows.append((int(r[4] or 0), int(r[5] or 0), fname, r[0], r[1].strip()[:100]))
        except ValueError:
            pass
tot = sum(x[0] for x in rows) or 1
print(f"total samples {tot}")
for s, ni, f, ln, src in sorted(rows, reverse=True)[:top]:
    print(f"{s:7d} {100 * s / tot:5.1f}% (not-issued {ni:6d}) {f}:{ln:>4}  {src}")
