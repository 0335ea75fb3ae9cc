# N > 1 bench path on one GPU (every rank on cuda:0, gloo host plumbing, CUDA IPC exchange buffers)
for n in 2 4; do
FOP_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 2953$n bench.py --gpus $n --steps 10 --warmup 3 --exchange peer > gpurun_out/bench_onegpu${n}_peer.log 2>&1; echo bench_$n=$?
tail -1 gpurun_out/bench_onegpu${n}_peer.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(d['n_gpus'],d['value'],d['config']['launch'],{k:(v['steady'] or {}).get('GB_s') for k,v in d['config']['per_op'].items()})"
done
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_s3c.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_gpu_s3c.log
