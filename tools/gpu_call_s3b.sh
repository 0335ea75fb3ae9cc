# transpose probe (full-row smem staging vs the register skeleton) + GV sweep + race/sync check
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tr_probe tools/probes/tr_probe.cu && timeout 300 /tmp/tr_probe > gpurun_out/tr_probe.log 2>&1; echo probe=$?
cat gpurun_out/tr_probe.log
timeout 600 python tools/sweep.py cfg3 "" "FOP_TR_GV=32" "FOP_TR_GV=32,FOP_TR_U=4" "FOP_TR_GV=16" "FOP_TR_GV=16,FOP_TR_U=4" "FOP_TR_GV=4" "FOP_TR_GV=4,FOP_TR_U=1" > gpurun_out/sweep_gv.log 2>&1; echo sweep=$?
cut -c1-200 gpurun_out/sweep_gv.log
SAN_TOOLS="racecheck synccheck" bash tools/gpu_sanitize.sh
