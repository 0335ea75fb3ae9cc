timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_peel.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_peel.log
for s in 15 16; do timeout 900 python tools/fuzz_campaign.py --seed $s --count 300 --repeat > gpurun_out/fuzz_s$s.log 2>&1; echo fuzz_$s=$?; tail -1 gpurun_out/fuzz_s$s.log; done
SAN_TOOLS="memcheck" SAN_TIMEOUT=600 bash tools/gpu_sanitize.sh 2>&1 | grep -E '=|SUMMARY|passed|failed' | grep -v '^+' | head -4
timeout 900 python tools/red_variety.py > gpurun_out/red_variety8.log 2>&1; echo rc=$?
python - <<'PY'
import json
for l in open('gpurun_out/red_variety8.log'):
    if l.startswith('{'):
        d=json.loads(l)
        if 'error' in d: print(d); continue
        print(f"{d['case']:38s} {d['selected'][0]:26s} grid {d['selected'][1]:5d} {d['us']:8.1f}us {d['GB_s']:7.0f} GB/s")
PY
