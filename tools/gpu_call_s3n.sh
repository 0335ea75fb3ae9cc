timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_fuzz.py tests/test_repeat_runs.py tests/test_edge_cases.py -x -q > gpurun_out/pytest_smem.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_smem.log
SAN_TOOLS="memcheck racecheck" SAN_TIMEOUT=600 bash tools/gpu_sanitize.sh 2>&1 | grep -E '=|SUMMARY|passed|failed' | grep -v '^+' | head
timeout 900 python tools/tr_variety.py > gpurun_out/tr_variety3.log 2>&1; echo rc=$?
timeout 600 python tools/sweep.py cfg3 "" > /dev/null 2>&1
python - <<'PY'
import json
for l in open('gpurun_out/tr_variety3.log'):
    if l.startswith('{'):
        d=json.loads(l)
        if 'error' in d: print(d); continue
        print(f"{d['case']:40s} {d['class']:10s} v={d['vec_loop']}/{d['width']} r={d['read_loop']}/{d['read_width']} {d['selected'][0]:22s} {d['us']:8.1f}us {d['GB_s']:7.0f} GB/s copy {d['copy_GB_s']:6.0f} frac {d['frac_of_copy']:.3f}")
PY
