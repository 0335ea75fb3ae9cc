timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_n4_ops.py tests/test_fuzz.py -x -q > gpurun_out/pytest_rowp2.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_rowp2.log
timeout 900 python tools/red_variety.py > gpurun_out/red_variety4.log 2>&1; echo rc=$?
python - <<'PY'
import json
for l in open('gpurun_out/red_variety4.log'):
    if l.startswith('{'):
        d=json.loads(l)
        if 'error' in d: print(d); continue
        print(f"{d['case']:34s} {d['selected'][0]:26s} grid {d['selected'][1]:5d} {d['us']:8.1f}us {d['GB_s']:7.0f} GB/s")
PY
python bench.py > gpurun_out/bench_s3r.log 2>&1; echo bench=$?
python - <<'PY'
import json
d=json.loads(open("gpurun_out/bench_s3r.log").read().strip().splitlines()[-1])
print(d["value"], d["ms_per_step"], d["e2e"]["value"])
for k,v in d["config"]["per_op"].items(): print(k, v["kernel"], v["grid"], v["block"], round(v["GB_s"]), v["steady"] and round(v["steady"]["GB_s"]))
PY
