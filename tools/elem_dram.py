"""Summarise an ncu --csv metrics capture (dram bytes + duration per kernel)
into per-kernel GB/s vs the HBM peak.  usage: python tools/elem_dram.py capture.csv [peak_GBps]"""
import csv
import sys
from collections import defaultdict

rows = [r for r in csv.reader(open(sys.argv[1])) if r]
hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r and "Metric Name" in r)
H = rows[hdr]
ki, mi, vi, ii = H.index("Kernel Name"), H.index("Metric Name"), H.index("Metric Value"), H.index("ID")
peak = float(sys.argv[2]) if len(sys.argv) > 2 else 6553.0
per = defaultdict(dict)
names = {}
for r in rows[hdr + 1:]:
    try:
        v = float(r[vi].replace(",", ""))
    except ValueError:
        continue
    per[r[ii]][r[mi]] = v
    names[r[ii]] = r[ki]
print("kernel,launch,time_us,dram_read_MB,dram_write_MB,GBps,frac_of_peak")
for i in sorted(per, key=int):
    m = per[i]
    t = m.get("gpu__time_duration.sum", 0.0) / 1e3  # ns -> us
    rd = m.get("dram__bytes_read.sum", 0.0)
    wr = m.get("dram__bytes_write.sum", 0.0)
    gbps = (rd + wr) / (t * 1e-6) / 1e9 if t else 0.0
    nm = names[i].split("(")[0][:60]
    print(f"{nm},{i},{t:.1f},{rd / 1e6:.1f},{wr / 1e6:.1f},{gbps:.0f},{gbps / peak:.3f}")
