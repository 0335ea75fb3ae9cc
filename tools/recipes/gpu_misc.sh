for ex in peer nccl; do
FOP_BENCH_ONE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --exchange $ex --no-cpu > gpurun_out/bench_onegpu2_$ex.log 2>&1; echo bench_$ex=$?
tail -1 gpurun_out/bench_onegpu2_$ex.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(d['value'],d['config']['launch'],d['config']['parallelism'])"
done
for s in 7 8; do timeout 1000 python tools/fuzz_campaign.py --seed $s --count 400 --repeat 2>&1 | tail -4; done
