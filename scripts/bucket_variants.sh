#!/bin/bash
# bucket_kernel variants: builder bit-exact parity subset + warm bucket_kernel time per config; then bench repeats.
# usage: gpurun -- 'bash scripts/slotfill_variants.sh TAG lib1.so lib2.so ...'
TAG=$1; shift
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for lib in "$@"; do
  export LF_LIB=$PWD/paper_conf_hpdc_pengtpk25_b200/$lib
  timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "bit_exact or full_config or edge or long_rows" \
     > gpurun_out/${TAG}_${lib}_pytest.txt 2>&1
  echo "$lib $(tail -1 gpurun_out/${TAG}_${lib}_pytest.txt)" >> gpurun_out/${TAG}_summary.txt
  for c in c2_rmat20 c3_stencil126 c4_reddit; do
    timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv -k regex:bucket_kernel \
      --log-file gpurun_out/${TAG}_${lib}_${c}.csv python scripts/prof.py $c 5 > /dev/null 2>&1
    python - "$lib" "$c" gpurun_out/${TAG}_${lib}_${c}.csv >> gpurun_out/${TAG}_summary.txt <<'PY'
import csv, sys
rows = [r for r in csv.reader(open(sys.argv[3])) if len(r) > 10]
h = rows[0]; ki = h.index("Kernel Name"); vi = h.index("Metric Value"); ui = h.index("Metric Unit")
v = [float(r[vi].replace(",", "")) for r in rows[1:] if "bucket_kernel" in r[ki]]
v = v[2:] or v
u = rows[1][ui] if len(rows) > 1 else "?"
print(sys.argv[1], sys.argv[2], "bucket_kernel", round(sum(v) / max(len(v), 1), 1), u, "n", len(v))
PY
  done
done
cat gpurun_out/${TAG}_summary.txt
