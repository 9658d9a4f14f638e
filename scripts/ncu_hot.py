"""Summarise an .ncu-rep: key metrics + hottest SASS lines by stall samples.
usage: python scripts/ncu_hot.py rep.ncu-rep [n_lines]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
KEYS = ("Duration", "Memory Throughput", "DRAM Throughput", "L1/TEX Hit Rate", "L2 Hit Rate",
        "Compute (SM) Throughput", "Achieved Occupancy", "Registers Per Thread", "Warp Cycles Per Issued Instruction",
        "Issued Warp Per Scheduler", "No Eligible", "Theoretical Occupancy", "Block Limit Registers",
        "L1/TEX Cache Throughput", "L2 Cache Throughput", "Mem Busy", "Max Bandwidth", "Elapsed Cycles",
        "SM Frequency", "DRAM Frequency")
d = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
for r in csv.reader(io.StringIO(d)):
    if len(r) > 14 and r[12] in KEYS:
        print(f"{r[12]:40s} {r[14]:>14s} {r[13]}")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
if len(rows) > 2:
    hdr, units, vals = rows[0], rows[1], rows[2]
    for k in ("dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum", "l1tex__t_bytes.sum",
              "smsp__inst_executed.sum", "launch__grid_size", "launch__registers_per_thread",
              "smsp__inst_executed_op_global_red.sum", "sm__warps_active.avg.pct_of_peak_sustained_active"):
        if k in hdr:
            i = hdr.index(k)
            print(f"{k:40s} {vals[i]:>14s} {units[i]}")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hdr = None
lines = []
for r in rows:
    if "Address" in r and "Source" in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        dd = dict(zip(hdr, r))
        try:
            lines.append((int(dd["Warp Stall Sampling (All Samples)"]), dd["Address"][-5:], dd["Source"].strip()))
        except ValueError:
            pass
tot = sum(x[0] for x in lines) or 1
print(f"--- top {n} SASS by stall samples (total {tot})")
for s, a, t in sorted(lines, reverse=True)[:n]:
    print(f"{100*s/tot:5.1f}% {a} {t}")
