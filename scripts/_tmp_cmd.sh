bash scripts/gpu_round.sh r2i
timeout 1500 python scripts/ncu_traffic.py > gpurun_out/r2i_traffic.log 2>&1
cp profiles/traffic.json gpurun_out/r2i_traffic.json
timeout 600 python bench.py > gpurun_out/r2i_bench2.json 2> gpurun_out/r2i_bench2.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv python scripts/prof.py c2_rmat20 4 2>/dev/null | grep '^"' > gpurun_out/r2i_c2_step_warm.csv
python -c "
import json; d=json.load(open('gpurun_out/r2i_bench2.json')); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['roofline']['traffic'], d['gpu_launches'], d['e2e']['value'])"
