timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_lnpeel.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_lnpeel.log
timeout 900 python tools/fuzz_campaign.py --seed 21 --count 300 --repeat > gpurun_out/fuzz_s21.log 2>&1; echo fuzz=$?; grep -E '^\{|^[0-9]+ ' gpurun_out/fuzz_s21.log | head -3 | cut -c1-300
SAN_TOOLS="memcheck" SAN_TIMEOUT=900 bash tools/gpu_sanitize.sh 2>&1 | grep -E '=|SUMMARY|passed|failed' | grep -v '^+' | head -3
timeout 900 python tools/red_variety.py > gpurun_out/red_variety9.log 2>&1
grep -E 'layernorm|vocab' gpurun_out/red_variety9.log | python -c "
import sys, json
for l in sys.stdin:
    d = json.loads(l); print(f\"{d['case']:38s} {d['selected'][0]:26s} {d['us']:8.1f}us {d['GB_s']:7.0f} GB/s\")
"
