# GPU checks of the in-kernel cross-GPU combine on a 1-GPU box
set -x
timeout 900 python -m pytest tests/test_peer.py -m gpu -x -q > gpurun_out/pytest_peer.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_peer.log
for ex in peer nccl; do
FOP_BENCH_ONE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --exchange $ex > gpurun_out/bench_onegpu2_$ex.log 2>&1; echo bench_$ex=$?
tail -c 1500 gpurun_out/bench_onegpu2_$ex.log
done
