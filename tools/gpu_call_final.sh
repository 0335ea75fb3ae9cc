python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.log 2>&1; echo smoke=$?
SAN_TOOLS="memcheck racecheck" SAN_TIMEOUT=900 bash tools/gpu_sanitize.sh 2>&1 | grep -E '=|SUMMARY|passed|failed' | grep -v '^+' | head -6
FOP_BENCH_ONE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29541 bench.py --gpus 2 --steps 5 --warmup 3 --no-cpu > gpurun_out/bench_onegpu2_final.log 2>&1; echo bench2=$?
tail -1 gpurun_out/bench_onegpu2_final.log | cut -c1-200
python bench.py > gpurun_out/bench_final.log 2>&1; echo bench=$?
python - <<'PY'
import json
d=json.loads(open("gpurun_out/bench_final.log").read().strip().splitlines()[-1])
print(d["value"], d["ms_per_step"], d["e2e"]["value"], d["roofline"]["frac"], d["clocks"], d["gpu_launches"])
for k,v in d["config"]["per_op"].items(): print(k, v["kernel"], round(v["GB_s"]), v["steady"] and round(v["steady"]["GB_s"]))
PY
