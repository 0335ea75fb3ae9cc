python -X faulthandler tools/fuzz_one.py 21 294 > gpurun_out/f294.log 2>&1; echo one=$?; tail -1 gpurun_out/f294.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_fast.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_fast.log
for s in 21 22; do timeout 900 python tools/fuzz_campaign.py --seed $s --count 300 --repeat > gpurun_out/fuzz_s$s.log 2>&1; echo fuzz_$s=$?; grep -E '^\{|^[0-9]+ ' gpurun_out/fuzz_s$s.log | head -3 | cut -c1-300; done
python bench.py > gpurun_out/bench_final2.log 2>&1; echo bench=$?
python - <<'PY'
import json
d=json.loads(open("gpurun_out/bench_final2.log").read().strip().splitlines()[-1])
print(d["value"], d["ms_per_step"], d["e2e"]["value"], d["roofline"]["frac"], d["clocks"])
for k,v in d["config"]["per_op"].items(): print(k, v["kernel"], round(v["GB_s"]), v["steady"] and round(v["steady"]["GB_s"]))
PY
