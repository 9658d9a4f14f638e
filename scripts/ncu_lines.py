"""Per-CUDA-source-line totals of an ncu report's SASS metrics (stall samples,
instructions executed), mapped through nvdisasm line info of the object file.
usage: python scripts/ncu_lines.py REP.ncu-rep OBJ.o KERNEL_SUBSTR [n]"""
import csv
import io
import os
import re
import subprocess
import sys
import tempfile

rep, obj, kname = sys.argv[1], sys.argv[2], sys.argv[3]
n = int(sys.argv[4]) if len(sys.argv) > 4 else 40
tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=tmp, capture_output=True)
cubin = [f for f in os.listdir(tmp) if f.endswith(".cubin")][0]
dis = subprocess.run(["nvdisasm", "--print-line-info", os.path.join(tmp, cubin)], capture_output=True, text=True).stdout
# offset -> (file, line) inside the kernel's function
line_of, in_fn, cur = {}, False, None
for ln in dis.splitlines():
    if ln.startswith("\t.text.") or ln.startswith(".text."):
        in_fn = kname in ln
    if ".text." in ln and ":" in ln and not ln.strip().startswith("//"):
        in_fn = kname in ln
    if not in_fn:
        continue
    m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
    if m:
        cur = (os.path.basename(m.group(1)), int(m.group(2)))
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", ln)
    if m and cur:
        line_of[int(m.group(1), 16)] = cur
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hdr = rows[1]
data = [dict(zip(hdr, r)) for r in rows[2:] if len(r) == len(hdr)]
base = int(data[0]["Address"], 16)
agg = {}
for d in data:
    off = int(d["Address"], 16) - base
    key = line_of.get(off, ("?", 0))
    a = agg.setdefault(key, [0, 0, {}])
    a[0] += int(d["Warp Stall Sampling (All Samples)"] or 0)
    a[1] += int(d["Instructions Executed"] or 0)
    for k, v in d.items():
        if k.startswith("stall_") and "Not Issued" not in k:
            try:
                a[2][k[6:]] = a[2].get(k[6:], 0) + int(v or 0)
            except ValueError:
                pass
tot_s = sum(v[0] for v in agg.values()) or 1
tot_i = sum(v[1] for v in agg.values()) or 1
print(f"{len(line_of)} mapped SASS offsets; {tot_s} stall samples; {tot_i} warp instructions")
srcfiles = {}
for (f, l), (s, i, st) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:n]:
    text = ""
    for root, _, files in os.walk(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))):
        if f in files and "build" not in root:
            p = os.path.join(root, f)
            srcfiles.setdefault(p, open(p).read().splitlines())
            text = srcfiles[p][l - 1].strip() if 0 < l <= len(srcfiles[p]) else ""
            break
    top = sorted(st.items(), key=lambda kv: -kv[1])[:3]
    why = " ".join(f"{k}:{100 * v / max(s, 1):.0f}%" for k, v in top if v)
    print(f"{100 * s / tot_s:5.1f}% stall {100 * i / tot_i:5.1f}% inst  {f}:{l}  {text[:70]}  [{why}]")
