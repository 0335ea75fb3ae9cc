set -x
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 1800 python -m pytest tests/test_full_size_gpu.py tests/test_parity_gpu.py -q -x -m gpu -k "cfg3 or nhwc or tma" > gpurun_out/pytest_tr_zc.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_tr_zc.log
timeout 600 python tools/tr_variety.py > gpurun_out/tr_variety_zc.log 2>&1; echo tr=$?
python -c "
import json
for l in open('gpurun_out/tr_variety_zc.log'):
    if l.startswith('{'):
        d=json.loads(l); print(d['case'][:40].ljust(40), d['selected'][0], d['selected'][1:], round(d['GB_s']), round(d['frac_of_copy'],3))
"
for i in 1 2; do
timeout 900 python bench.py --no-cpu > gpurun_out/bench_zc$i.log 2>&1; echo bench=$?
tail -1 gpurun_out/bench_zc$i.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),d['clocks'],{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"
done
