"""Parse an ncu launch log of tools/panel_scaling.py: panel-kernel durations per n."""
import sys

seq, cur = [], None
for line in open(sys.argv[1]):
    if "Context" in line and "Stream" in line:
        cur = line.strip().replace("void ", "").replace("kern::", "").replace("<unnamed>::", "").split("(")[0]
    elif "gpu__time_duration" in line and cur:
        seq.append((cur, float(line.split()[-1])))
        cur = None
keep = [(a, b) for a, b in seq if not any(k in a for k in ("spmv", "elementwise", "Fill", "fill", "distribution", "normal"))]
ns = [65536, 262144, 1048576, 2097152]
per = len(keep) // len(ns)
for i, n in enumerate(ns):
    print(n, [(a[:24], b) for a, b in keep[i * per:(i + 1) * per]][-4:])
