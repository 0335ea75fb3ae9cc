timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_n4_ops.py tests/test_fuzz.py tests/test_edge_cases.py -x -q > gpurun_out/pytest_rtkk.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_rtkk.log
timeout 900 python tools/row_long_probe.py > gpurun_out/row_long2.log 2>&1; echo rc=$?
python -c "
import json
for l in open('gpurun_out/row_long2.log'):
    if l.startswith('{'):
        d=json.loads(l); print(d['shape'], f\"{d['variant']:32s}\", d.get('grid'), d.get('block'), round(d.get('us',0),1), round(d.get('GB_s',0)), d.get('error',''))
"
timeout 900 python tools/red_variety.py > gpurun_out/red_variety5.log 2>&1
python - <<'PY'
import json
for l in open('gpurun_out/red_variety5.log'):
    if l.startswith('{'):
        d=json.loads(l)
        if 'error' in d: print(d); continue
        print(f"{d['case']:34s} {d['selected'][0]:26s} grid {d['selected'][1]:5d} {d['us']:8.1f}us {d['GB_s']:7.0f} GB/s")
PY
