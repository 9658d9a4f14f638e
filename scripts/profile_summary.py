"""Write a markdown summary of an ncu launch list (+ optional --set full
report) into profiles/.  usage:
  python scripts/profile_summary.py OUT.md LAUNCHES.csv [FULL.ncu-rep ...]"""
import collections
import csv
import subprocess
import sys

out, launches, reps = sys.argv[1], sys.argv[2], sys.argv[3:]
rows = list(csv.reader(open(launches)))
hdr, ks = None, []
for r in rows:
    if "Kernel Name" in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        ks.append((d["Kernel Name"].split("(")[0].replace("lf::<unnamed>::", "").replace("void ", ""),
                   float(d["Metric Value"]) / 1000))
agg = collections.OrderedDict()
for k, v in ks:
    agg.setdefault(k, []).append(v)
tot = sum(v for _, v in ks)
lines = [f"# {out.split('/')[-1]}", "", f"Launch list `{launches.split('/')[-1]}`: {len(ks)} launches, "
         f"{tot:.1f} us total (ncu `gpu__time_duration.sum`, `--clock-control none`, cold-cache and "
         "serialised: compare shares, not absolutes).", "",
         "| kernel | launches | mean us | share |", "|---|---|---|---|"]
for k, v in agg.items():
    lines.append(f"| `{k}` | {len(v)} | {sum(v)/len(v):.1f} | {100*sum(v)/tot:.1f}% |")
for rep in reps:
    lines += ["", f"## `{rep.split('/')[-1]}` (ncu --set full)", "", "```"]
    lines += subprocess.run([sys.executable, "scripts/ncu_hot.py", rep, "12"], capture_output=True,
                            text=True).stdout.splitlines()
    lines.append("```")
open(out, "w").write("\n".join(lines) + "\n")
print("\n".join(lines))
