#!/bin/bash
# slot_fill variants: builder bit-exact parity subset + warm slot_fill time per config; then bench repeats.
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
    timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv -k regex:slot_fill \
      --log-file gpurun_out/${TAG}_${lib}_${c}.csv python scripts/prof.py $c 5 > /dev/null 2>&1
    python - "$lib" "$c" gpurun_out/${TAG}_${lib}_${c}.csv >> gpurun_out/${TAG}_summary.txt <<'PY'
import csv, sys
rows = [r for r in csv.reader(open(sys.argv[3])) if len(r) > 10]
h = rows[0]; ki = h.index("Kernel Name"); vi = h.index("Metric Value"); ui = h.index("Metric Unit")
v = [float(r[vi].replace(",", "")) for r in rows[1:] if "slot_fill" in r[ki]]
v = v[2:] or v
u = rows[1][ui] if len(rows) > 1 else "?"
print(sys.argv[1], sys.argv[2], "slot_fill", round(sum(v) / max(len(v), 1), 1), u, "n", len(v))
PY
  done
done
unset LF_LIB
for i in 1 2 3; do
  for s in 2 1; do
    timeout 600 python bench.py --streams $s --no-cpu-baseline > gpurun_out/${TAG}_b${s}_$i.json 2>/dev/null
    python -c "
import json; d=json.load(open('gpurun_out/${TAG}_b${s}_$i.json'))
print('bench streams $s rep $i', round(d['value']), round(d['ms_per_step'], 4), round(d['ms_per_step_serial'], 4))" >> gpurun_out/${TAG}_summary.txt
  done
done
cat gpurun_out/${TAG}_summary.txt
