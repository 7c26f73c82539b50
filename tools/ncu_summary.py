"""Summarise ncu CSV outputs for profiles/ (launch lists and --set full raw pages).

    python tools/ncu_summary.py launches <launches.csv>      # per-kernel count/time/share
    python tools/ncu_summary.py raw <report.ncu-rep>          # key metrics per captured launch
"""
import collections
import csv
import io
import subprocess
import sys

UNIT = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "second": 1e6}


def _rows(text):
    lines = text.splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"') or l.startswith('"Process ID"') or '"Kernel Name"' in l)
    return list(csv.reader(io.StringIO("\n".join(lines[start:]))))


def launches(path):
    rows = _rows(open(path).read())
    h = rows[0]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.OrderedDict()
    for r in rows[1:]:
        if len(r) <= vi or not r[vi]:
            continue
        name = r[ki].split("(")[0].replace("void ", "")
        us = float(r[vi].replace(",", "")) * UNIT.get(r[ui], 1.0)
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += us
    tot = sum(v[1] for v in agg.values())
    print(f"{'kernel':55s} {'launches':>8s} {'total_us':>12s} {'avg_us':>9s} {'share':>6s}")
    for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"{k[:55]:55s} {n:8d} {t:12.1f} {t / n:9.2f} {t / tot:6.3f}")
    print(f"{'TOTAL':55s} {sum(v[0] for v in agg.values()):8d} {tot:12.1f}")


KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum",
        "smsp__inst_executed.sum", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"]


def raw(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    for r in rows[2:]:
        print(r[h.index("Kernel Name")][:90])
        for k in KEYS:
            if k in h:
                i = h.index(k)
                print(f"    {k:60s} {r[i]:>16s} {units[i]}")


if __name__ == "__main__":
    {"launches": launches, "raw": raw}[sys.argv[1]](sys.argv[2])
