nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/bw_probe3 tools/probes/bw_probe3.cu
timeout 600 /tmp/bw_probe3 > gpurun_out/bw_probe3.log 2>&1; echo probe=$?
