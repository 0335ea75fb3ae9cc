nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tr_probe tools/probes/tr_probe.cu && timeout 300 /tmp/tr_probe > gpurun_out/tr_probe2.log 2>&1; echo probe=$?
cat gpurun_out/tr_probe2.log
