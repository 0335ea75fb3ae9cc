timeout 600 python tools/sweep.py cfg4a "opt:autotune=0" "opt:autotune=0,FOP_GELU_PAIR=1" "opt:autotune=0" "opt:autotune=0,FOP_GELU_PAIR=1" > gpurun_out/sweep_gpair.log 2>&1
python - <<'PY'
import json
for l in open("gpurun_out/sweep_gpair.log"):
    if l.startswith("{"):
        d=json.loads(l); print(d["op"], d["variant"], round(d.get("us_median",0),2), round(d.get("GBs_median",0)), d.get("error",""))
PY
FOP_GELU_PAIR=1 timeout 600 python -m pytest tests/test_parity_gpu.py tests/test_fuzz.py -x -q -k "cfg4a or gelu or fuzz" > gpurun_out/pytest_gpair.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpair.log
