#!/bin/bash
# per-kernel durations of configure + build + spmm (ncu launch list), one config per argument
mkdir -p gpurun_out
for cfg in "$@"; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv -s 0 \
      python scripts/prof.py $cfg 2 > gpurun_out/ll_$cfg.csv 2> gpurun_out/ll_$cfg.err
done
