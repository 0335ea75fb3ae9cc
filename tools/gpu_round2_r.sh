set -x
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 900 compute-sanitizer --tool initcheck --print-limit 20 --error-exitcode 99 python -m pytest tests/test_int_gpu.py tests/test_odd_gpu.py -m gpu -q -x -k "not full_size" -p no:cacheprovider > gpurun_out/san_initcheck2.log 2>&1; echo initcheck=$?
grep -E "ERROR SUMMARY|passed|failed" gpurun_out/san_initcheck2.log | tail -2
b() { timeout 600 python bench.py --no-cpu --steps 50 "$@" 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),{k:round(v['GB_s']) for k,v in d['config']['per_op'].items()}, d['clocks']['sm_mhz'])"; }
echo default; b --no-steady
echo store_stream; FOP_STORE_POLICY=stream b --no-steady
echo default2; b --no-steady
