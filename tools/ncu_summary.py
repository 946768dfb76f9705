"""Summaries of ncu output for profiles/: per-kernel launch-time shares from a
`--metrics gpu__time_duration.sum --csv` launch list, and key metrics of `--set full` reports.

    python tools/ncu_summary.py launches <launches.csv>
    python tools/ncu_summary.py report <a.ncu-rep> [...]
"""
import collections
import csv
import io
import subprocess
import sys

UNIT = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0, "s": 1e3, "second": 1e3}
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "sm__cycles_elapsed.avg.per_second"]


def launches(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h, data = rows[hi], rows[hi + 1:]
    ki, mi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    tot, cnt = collections.defaultdict(float), collections.Counter()
    for r in data:
        if len(r) <= mi:
            continue
        v = float(r[mi].replace(",", "")) * UNIT.get(r[ui], 1.0)
        name = r[ki].split("(")[0].replace("void ", "").replace("gmpsvm::", "")
        tot[name] += v
        cnt[name] += 1
    T = sum(tot.values())
    print("| kernel | launches | total ms | share |\n|---|---|---|---|")
    for n, v in sorted(tot.items(), key=lambda x: -x[1]):
        print(f"| {n} | {cnt[n]} | {v:.3f} | {100 * v / T:.1f}% |")
    print(f"| **all** | {sum(cnt.values())} | {T:.3f} | 100% |")


def report(paths):
    for p in paths:
        out = subprocess.run(["ncu", "-i", p, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(io.StringIO(out)))
        h, u = rows[0], rows[1]
        for v in rows[2:]:
            name = v[h.index("Kernel Name")].split("(")[0] if "Kernel Name" in h else p
            print(f"### {name}  ({p.split('/')[-1]})")
            for k in KEYS:
                if k in h:
                    i = h.index(k)
                    print(f"- {k}: {v[i]} {u[i]}")


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        launches(sys.argv[2])
    else:
        report(sys.argv[2:])
