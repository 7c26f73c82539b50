"""Per-kernel table from an ncu CSV launch list captured with
--metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum:
launches, mean duration, mean DRAM bytes read / written, DRAM GB/s, share of the total.

    python tools/launch_table.py launches.csv [top]
"""
import collections
import csv
import io
import sys


def table(path, top=20):
    txt = open(path).read().splitlines()
    st = next(i for i, l in enumerate(txt) if l.startswith('"ID"'))
    rows = list(csv.reader(io.StringIO("\n".join(txt[st:]))))
    h = rows[0]
    ki, mi, vi, ii = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
    ui = h.index("Metric Unit")
    scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1.0,
             "Gbyte": 1e3}
    per = collections.defaultdict(dict)
    for r in rows[1:]:
        per[(int(r[ii]), r[ki].split("(")[0].replace("void ", ""))][r[mi]] = \
            float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0)
    agg = collections.defaultdict(lambda: [0, 0.0, 0.0, 0.0])
    for (_, k), d in per.items():
        a = agg[k]
        a[0] += 1
        a[1] += d.get("gpu__time_duration.sum", 0.0)
        a[2] += d.get("dram__bytes_read.sum", 0.0)
        a[3] += d.get("dram__bytes_write.sum", 0.0)
    tot = sum(a[1] for a in agg.values())
    out = [f"{'kernel':58s} {'n':>5s} {'avg_us':>8s} {'rd_MB':>8s} {'wr_MB':>8s} {'GB/s':>7s} {'share':>6s}"]
    for k, (n, t, r, w) in sorted(agg.items(), key=lambda x: -x[1][1])[:top]:
        out.append(f"{k[:58]:58s} {n:5d} {t / n:8.1f} {r / n:8.1f} {w / n:8.1f} {1e3 * (r + w) / t if t else 0:7.0f} {t / tot:6.3f}")
    out.append(f"{'TOTAL':58s} {sum(a[0] for a in agg.values()):5d} {tot:8.0f} us")
    return "\n".join(out)


if __name__ == "__main__":
    print(table(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 20))
