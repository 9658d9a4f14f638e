#!/bin/bash
# Quick gpurun iteration: GPU tests (optional), bench, warm per-kernel launch list.
# usage: gpurun -- 'bash scripts/quick_round.sh TAG [notests]'
TAG=${1:-q}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/${TAG}_smoke.txt 2>&1
if [ "$2" != "notests" ]; then
  timeout 1200 python -m pytest tests -m gpu -q -x --timeout 900 > gpurun_out/${TAG}_pytest_gpu.txt 2>&1
  tail -3 gpurun_out/${TAG}_pytest_gpu.txt
fi
timeout 600 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv \
  --log-file gpurun_out/${TAG}_warm.csv python scripts/prof.py c2_rmat20 5 > /dev/null 2>&1
tail -2 gpurun_out/${TAG}_smoke.txt
python -c "
import json; d=json.load(open('gpurun_out/${TAG}_bench.json'))
print('value', d['value'], 'ms/step', d['ms_per_step'], 'phases', d['phases_ms'], 'frac', d['roofline']['frac'], 'e2e', d['e2e']['value'])"
