python bench.py > gpurun_out/bench_s3b.log 2>&1; echo bench=$?
tail -c 2500 gpurun_out/bench_s3b.log
bash tools/gpu_sanitize.sh
