timeout 900 python tools/red_variety.py > gpurun_out/red_variety6.log 2>&1; echo rc=$?
python - <<'PY'
import json
for l in open('gpurun_out/red_variety6.log'):
    if l.startswith('{'):
        d=json.loads(l)
        if 'error' in d: print(d); continue
        print(f"{d['case']:34s} {d['selected'][0]:26s} grid {d['selected'][1]:5d} {d['us']:8.1f}us {d['GB_s']:7.0f} GB/s")
PY
timeout 900 python -m pytest tests/test_n4_ops.py tests/test_parity_gpu.py -x -q -k "vocab or wide or bn_stats or row or cfg4a" > gpurun_out/pytest_rowq.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_rowq.log
