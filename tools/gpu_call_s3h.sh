for op in bert_layernorm cfg4a bert_softmax cfg4b cfg2 cfg3; do
timeout 600 python tools/sweep.py $op "opt:autotune=0" "opt:autotune=1" "opt:autotune=1,FOP_TUNE_HOT=1" >> gpurun_out/sweep_tune3.log 2>&1
done
python - <<'PY'
import json
for l in open("gpurun_out/sweep_tune3.log"):
    if l.startswith("{"):
        d=json.loads(l); print(d["op"], d["variant"], round(d.get("us_median",0),2), round(d.get("GBs_median",0)), d.get("selected", ""), d.get("error",""))
    else: print(l.rstrip()[:200])
PY
timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_repeat_runs.py -x -q > gpurun_out/pytest_tune3.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_tune3.log
python bench.py > gpurun_out/bench_s3i.log 2>&1; echo bench=$?
python - <<'PY'
import json
d=json.loads(open("gpurun_out/bench_s3i.log").read().strip().splitlines()[-1])
print(d["value"], d["ms_per_step"])
for k,v in d["config"]["per_op"].items(): print(k, v["kernel"], v["grid"], v["block"], round(v["GB_s"]), v["steady"] and round(v["steady"]["GB_s"]))
PY
