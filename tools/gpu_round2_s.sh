set -x
for n in 2; do
FOP_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 2958$n bench.py --gpus $n --steps 5 --warmup 3 --no-cpu --no-steady > gpurun_out/bench_onegpu${n}_weak.log 2>&1; echo weak$n=$?
tail -1 gpurun_out/bench_onegpu${n}_weak.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),d['scaling'],d['config']['parallelism'],d['config']['exchange_check'],d['config']['exchange_note'])"
done
