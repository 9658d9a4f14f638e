mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for s in 2 1 3; do timeout 600 python bench.py --streams $s --no-cpu-baseline > gpurun_out/st${s}.json 2> gpurun_out/st${s}.err; done
for s in 2 1 3; do python -c "
import json; d=json.load(open('gpurun_out/st$s.json'))
print('streams $s value', round(d['value']), 'ms', round(d['ms_per_step'],4), 'serial', round(d['ms_per_step_serial'],4), d['phases_ms'], d['clocks'])"; done
tail -3 gpurun_out/st2.err
