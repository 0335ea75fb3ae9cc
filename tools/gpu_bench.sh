set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python bench.py > gpurun_out/bench_final.log 2>&1; echo bench=$?
tail -1 gpurun_out/bench_final.log | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print(round(d['value']), d['ms_per_step'], d['roofline']['kernel'], round(d['roofline']['frac'],3), d['clocks'], round(d['e2e']['value'],1))
for k,v in d['config']['per_op'].items(): print(k, v['kernel'], round(v['GB_s']), round(v['frac_of_measured_peak'],3), round(v['frac_of_8TBs'],3), v['steady'] and round(v['steady']['GB_s']), v['steady'] and round(v['steady']['frac_of_measured_peak'],3))
"
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.log 2>&1; echo ref=$?
tail -1 gpurun_out/bench_ref.log | cut -c1-300
