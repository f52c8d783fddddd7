"""Summarise an `ncu --set full --page raw --csv` export of tools/gemm_prof.py
(one launch per 1.5B GEMM shape, in its SHAPES order) into per-shape
duration, TF/s, DRAM traffic vs the algorithmic bytes (operands + outputs
read/written once) and tensor-pipe activity.
usage: python tools/gemm_traffic.py raw.csv out.json"""
import csv
import json
import sys

sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.abspath(__file__)))
from gemm_prof import SHAPES  # noqa: E402

rows = list(csv.reader(open(sys.argv[1])))
hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hdr_i]
data = [r for r in rows[hdr_i + 1:] if len(r) == len(h) and "gemm" in r[h.index("Kernel Name")]]


units = rows[hdr_i + 1]
SCALE = {"ns": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6, "nsecond": 1, "byte": 1, "Kbyte": 1e3,
         "Mbyte": 1e6, "Gbyte": 1e9, "%": 1}


def col(r, name):
    v = r[h.index(name)].replace(",", "")
    if v in ("", "n/a"):
        return None
    return float(v) * SCALE.get(units[h.index(name)], 1)


tcol = "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed" if "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed" in h else None
out = []
for (name, M, N, K, amn, bmn, epi, cf), r in zip(SHAPES, data):
    dur_ns = col(r, "gpu__time_duration.sum")
    dram = col(r, "dram__bytes_read.sum") + col(r, "dram__bytes_write.sum")
    e_out = 4 if cf else 2
    alg = 2 * (M * K + N * K) + e_out * M * N * (2 if epi == 5 else 1)  # operands + C (read+write for accumulate)
    if epi in (2,):
        alg += 2 * M * N          # AUX output
    if epi in (3, 4):
        alg += 2 * M * N          # R read
    out.append({"gemm": name, "M": M, "N": N, "K": K, "duration_us_ncu": dur_ns / 1e3,
                "tflops_ncu": 2.0 * M * N * K / dur_ns / 1e3, "dram_bytes": dram, "algorithmic_bytes": alg,
                "traffic_over_algorithmic": dram / alg,
                "tensor_active_pct": col(r, tcol) if tcol else None})
json.dump(out, open(sys.argv[2], "w"), indent=1)
print(json.dumps(out, indent=1))
