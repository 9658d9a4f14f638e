#!/bin/bash
# SpMM grid capped below full occupancy (LF_SPMM_GRID_BPS) x steps in flight: bench step time.
# usage: gpurun -- 'bash scripts/grid_share.sh TAG lib1.so lib2.so ...'
TAG=$1; shift
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for lib in "$@"; do
  LF_LIB=$PWD/paper_conf_hpdc_pengtpk25_b200/$lib timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x \
     -k "integer_exact or full_config or in_flight or repeated" > gpurun_out/${TAG}_${lib}_pytest.txt 2>&1
  echo "$lib $(tail -1 gpurun_out/${TAG}_${lib}_pytest.txt)" >> gpurun_out/${TAG}_summary.txt
done
for rep in 1 2; do
  for lib in "$@"; do
    for s in 1 2 3; do
      LF_LIB=$PWD/paper_conf_hpdc_pengtpk25_b200/$lib timeout 600 python bench.py --streams $s --no-cpu-baseline --no-e2e \
        > gpurun_out/${TAG}_${lib}_s${s}_$rep.json 2>/dev/null
      python -c "
import json; d=json.load(open('gpurun_out/${TAG}_${lib}_s${s}_$rep.json'))
print('$lib streams $s rep $rep', round(d['value']), round(d['ms_per_step'], 4), 'serial', round(d['ms_per_step_serial'], 4), 'spmm_only', round(d['spmm_only']['ms'], 4))" >> gpurun_out/${TAG}_summary.txt
    done
  done
done
cat gpurun_out/${TAG}_summary.txt
