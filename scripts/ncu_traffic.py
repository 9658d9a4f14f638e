"""DRAM traffic per lf_spmm launch, measured with ncu on the current sources.

For every workload (config:J) this runs scripts/spmm_once.py under
  ncu --kernel-name regex:<SpMM kernels> --launch-skip K --launch-count K
      --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum
capturing the LAST lf_spmm call (its zero_rows_kernel and SpMM kernel; K =
kernels per call) and writes profiles/traffic.json = {src_hash, when,
entries: {config:J: {kernels, dram_read, dram_write, dram_bytes, ncu_us}}}.
bench.py reports `roofline.traffic` from it only when src_hash matches the
sources it runs (bench.src_hash), so the number is never stale.

    python scripts/ncu_traffic.py [c2_rmat20:128 c3b_banded2M:128 ...]
"""
import csv
import io
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402

DEFAULT = ["c2_rmat20:128", "c2p_rmat20_perm:128", "c3b_banded2M:64", "c3b_banded2M:128", "c3_stencil126:64", "c3_stencil126:128",
           "c4_reddit:256"]
KREGEX = "regex:cell_spmm|csr_spmm|zero_rows"


def measure(cfg, J):
    n_calls = 3
    base = [sys.executable, os.path.join(ROOT, "scripts", "spmm_once.py"), cfg, str(J), str(n_calls)]
    # how many matching kernels does one call launch?  (1 = CSR path, 2 = zero_rows + SpMM)
    out = subprocess.run(["ncu", "--kernel-name", KREGEX, "--metrics", "gpu__time_duration.sum", "--csv",
                          "--clock-control", "none", *base], capture_output=True, text=True, cwd=ROOT)
    rows = [r for r in csv.reader(io.StringIO(out.stdout[out.stdout.find('"ID"'):])) if r]
    n_k = (len(rows) - 1) // n_calls
    out = subprocess.run(["ncu", "--kernel-name", KREGEX, "--launch-skip", str(n_k * (n_calls - 1)),
                          "--launch-count", str(n_k), "--clock-control", "none", "--csv", "--metrics",
                          "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum", *base],
                         capture_output=True, text=True, cwd=ROOT)
    rows = list(csv.DictReader(io.StringIO(out.stdout[out.stdout.find('"ID"'):])))
    tot = {"dram__bytes_read.sum": 0.0, "dram__bytes_write.sum": 0.0, "gpu__time_duration.sum": 0.0}
    names = set()
    for r in rows:
        if r.get("Metric Name") in tot:
            v = float(r["Metric Value"].replace(",", ""))
            u = r.get("Metric Unit", "")
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-3, "ns": 1e-3,
                     "usecond": 1, "us": 1, "msecond": 1e3, "ms": 1e3}.get(u, 1)
            tot[r["Metric Name"]] += v * scale
            names.add(r["Kernel Name"].split("(")[0].split("<")[0])
    return {"kernels": sorted(names), "dram_read": int(tot["dram__bytes_read.sum"]),
            "dram_write": int(tot["dram__bytes_write.sum"]),
            "dram_bytes": int(tot["dram__bytes_read.sum"] + tot["dram__bytes_write.sum"]),
            "ncu_us": tot["gpu__time_duration.sum"], "kernels_per_call": n_k}


def main():
    items = sys.argv[1:] or DEFAULT
    res = {"src_hash": bench.src_hash(), "when": time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime()),
           "how": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum "
                  "--clock-control none on the last of 3 lf_spmm calls (scripts/spmm_once.py)", "entries": {}}
    for it in items:
        cfg, J = it.split(":")
        res["entries"][f"{cfg}:J{J}"] = measure(cfg, int(J))
        print(it, res["entries"][f"{cfg}:J{J}"], flush=True)
    path = os.path.join(ROOT, "profiles", "traffic.json")
    with open(path, "w") as f:
        json.dump(res, f, indent=1)
    print("wrote", path)


if __name__ == "__main__":
    main()
