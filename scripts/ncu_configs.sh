#!/bin/bash
# ncu --set full of the CELL SpMM kernel on each named config (one launch each, after 2 warm launches).
# usage: gpurun -- 'bash scripts/ncu_configs.sh TAG c2_rmat20 c3_stencil126 ...'
TAG=$1; shift
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
for cfg in "$@"; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-cell_spmm} -s 2 -c 1 \
     -f -o gpurun_out/${TAG}_${cfg} python scripts/prof.py $cfg 3 > gpurun_out/${TAG}_${cfg}.log 2>&1
  python scripts/spmm_time.py $cfg >> gpurun_out/${TAG}_times.txt 2>&1
done
