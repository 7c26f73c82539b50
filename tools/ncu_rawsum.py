"""Key metrics + top stall reasons of an ncu --set full raw page (ncu -i X.ncu-rep --page raw --csv > X.csv).

    python tools/ncu_rawsum.py X.csv
"""
import csv,sys
rows=list(csv.reader(open(sys.argv[1])))
h=rows[0]; u=rows[1]; v=rows[2]
want=['gpu__time_duration.sum','dram__bytes_read.sum','dram__bytes_write.sum','gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed','sm__cycles_active.avg','sm__cycles_elapsed.avg','sm__warps_active.avg.pct_of_peak_sustained_active','smsp__inst_executed.sum','launch__registers_per_thread','launch__grid_size','launch__block_size','lts__t_bytes.sum','sm__throughput.avg.pct_of_peak_sustained_elapsed','l1tex__throughput.avg.pct_of_peak_sustained_active','lts__throughput.avg.pct_of_peak_sustained_elapsed']
print(v[h.index('Kernel Name')][:70] if 'Kernel Name' in h else '')
for w in want:
    if w in h: i=h.index(w); print(f"  {w:60s} {v[i]:>16s} {u[i]}")
st=[(h[i],v[i]) for i in range(len(h)) if h[i].startswith('smsp__average_warp_latency_issue_stalled') or h[i].startswith('smsp__average_warps_issue_stalled')]
st=[(a,float(b.replace(',',''))) for a,b in st if b not in ('','n/a')]
st.sort(key=lambda x:-x[1])
print('  stalls:', ', '.join(f"{a.split('stalled_')[-1].replace('_per_issue_active.ratio','')} {b:.2f}" for a,b in st[:7]))
