timeout 900 python tools/red_variety.py > gpurun_out/red_variety3.log 2>&1; echo rc=$?
python - <<'PY'
import json
for l in open('gpurun_out/red_variety3.log'):
    if l.startswith('{'):
        d=json.loads(l)
        if 'error' in d: print(d); continue
        print(f"{d['case']:34s} {d['selected'][0]:26s} grid {d['selected'][1]:5d} {d['us']:8.1f}us {d['GB_s']:7.0f} GB/s")
PY
