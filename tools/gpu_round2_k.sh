# full GPU suite, sanitizers (memcheck + racecheck), one-GPU multi-rank strong-scaling bench
set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
SAN_TOOLS="memcheck racecheck" SAN_TIMEOUT=1500 bash tools/gpu_sanitize.sh
for n in 2 4; do
FOP_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 2957$n bench.py --gpus $n --steps 5 --warmup 3 --scaling strong --no-cpu --no-steady > gpurun_out/bench_onegpu${n}_strong.log 2>&1; echo strong$n=$?
tail -1 gpurun_out/bench_onegpu${n}_strong.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(d['value'],d['scaling'],d['config']['global_batch_scale'],d['config']['exchange_check'])"
done
timeout 900 python bench.py --steps 5 --warmup 3 --scaling strong --no-cpu --no-steady > gpurun_out/bench_strong1.log 2>&1; echo strong1=$?
tail -1 gpurun_out/bench_strong1.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(d['value'],d['scaling'],d['config']['global_batch_scale'],d['ms_per_step'])"
