python -X faulthandler tools/fuzz_one.py 21 294 > gpurun_out/f294.log 2>&1; echo one=$?; tail -1 gpurun_out/f294.log
timeout 1500 python -X faulthandler -m pytest tests -m gpu -x -q > gpurun_out/pytest_fast2.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_fast2.log
for s in 21 23; do timeout 900 python -X faulthandler tools/fuzz_campaign.py --seed $s --count 300 --repeat > gpurun_out/fuzz_s$s.log 2>&1; echo fuzz_$s=$?; grep -E '^\{|^[0-9]+ ' gpurun_out/fuzz_s$s.log | head -3 | cut -c1-300; done
SAN_TOOLS="memcheck" SAN_TIMEOUT=900 bash tools/gpu_sanitize.sh 2>&1 | grep -E '=|SUMMARY|passed|failed' | grep -v '^+' | head -3
