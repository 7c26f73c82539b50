"""Launch sequence from an ncu CSV launch list (same metrics as launch_table.py): one line per
launch in issue order — id, kernel, duration, DRAM MB read / written — for a window of launches,
e.g. to compare alternate sweep directions under --cache-control none (serpentine order).

    python tools/launch_seq.py launches.csv [first] [count]
"""
import sys

from launch_table import table  # noqa: F401  (same CSV dialect)
import collections
import csv
import io


def seq(path):
    txt = open(path).read().splitlines()
    st = next(i for i, l in enumerate(txt) if l.startswith('"ID"'))
    rows = list(csv.reader(io.StringIO("\n".join(txt[st:]))))
    h = rows[0]
    ki, mi, vi, ii, ui = (h.index(x) for x in ("Kernel Name", "Metric Name", "Metric Value", "ID", "Metric Unit"))
    scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "byte": 1e-6, "Kbyte": 1e-3,
             "Mbyte": 1.0, "Gbyte": 1e3}
    per = collections.OrderedDict()
    for r in rows[1:]:
        key = int(r[ii])
        d = per.setdefault(key, {"k": r[ki].split("(")[0].replace("void ", "")})
        d[r[mi]] = float(r[vi].replace(",", "")) * scale.get(r[ui], 1.0)
    return per


if __name__ == "__main__":
    per = seq(sys.argv[1])
    first = int(sys.argv[2]) if len(sys.argv) > 2 else 0
    cnt = int(sys.argv[3]) if len(sys.argv) > 3 else 200
    for i, (key, d) in enumerate(per.items()):
        if first <= i < first + cnt:
            print(f"{key:6d} {d['k'][:52]:52s} {d.get('gpu__time_duration.sum', 0):8.1f} us "
                  f"{d.get('dram__bytes_read.sum', 0):8.1f} {d.get('dram__bytes_write.sum', 0):8.1f} MB")
