#!/bin/bash
# One gpurun call: smoke, GPU parity tests, bench (N=1), ncu launch list, ncu --set full of the SpMM.
# usage: gpurun -- 'bash scripts/gpu_round.sh TAG'
TAG=${1:-run}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/${TAG}_smoke.txt 2>&1
if [ -z "$SKIP_TESTS" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 > gpurun_out/${TAG}_pytest_gpu.txt 2>&1
fi
timeout 600 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${TAG}_bench_ref.json 2>> gpurun_out/${TAG}_bench.err
if [ -z "$SKIP_NCU" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
     --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:cell_spmm -s 2 -c 1 \
     -f -o gpurun_out/${TAG}_spmm_full python scripts/prof.py c2_rmat20 4 > gpurun_out/${TAG}_ncu.log 2>&1
fi
tail -3 gpurun_out/${TAG}_smoke.txt; tail -3 gpurun_out/${TAG}_pytest_gpu.txt 2>/dev/null; cat gpurun_out/${TAG}_bench.json
# per-config SpMM timing (configure / build / spmm phases; grouped path where chosen)
for c in c1_uniform1024 c3_stencil126 c3b_banded2M c4_reddit; do
  echo "$c $(timeout 300 python scripts/spmm_time.py $c iters=10 | tail -1)" >> gpurun_out/${TAG}_configs.txt
done
