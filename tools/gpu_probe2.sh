# round-2 probes: streaming strategies (tools/probes/bw_probe2.cu) then the GPU tests
set -x
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/bw_probe2 tools/probes/bw_probe2.cu
timeout 600 /tmp/bw_probe2 > gpurun_out/bw_probe2.log 2>&1; echo probe=$?
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -30 gpurun_out/pytest_gpu.log
