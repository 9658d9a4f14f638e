bash scripts/rows_variants.sh sr liblf.so lib_sr4.so lib_sr16.so lib_sr64.so > /dev/null 2>&1
for c in c3_stencil126 c3b_banded2M; do timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/r1m_bench_$c.json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/r1m_bench_$c.json')); print('$c', round(d['value']), d['ms_per_step'], d['ms_per_step_serial'])" >> gpurun_out/sr_summary.txt; done
cat gpurun_out/sr_summary.txt
