# ncu evidence for profiles/ (one GPU): launch list of the bench command + --set full of the tuned kernels
# usage: bash tools/gpu_profile.sh <tag>   (outputs gpurun_out/launches_<tag>.csv, gpurun_out/prof_<tag>.ncu-rep)
set -x
TAG=${1:-r01}
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-cpu --no-steady > gpurun_out/launches_bench_$TAG.log 2>&1; echo ll=$?
ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:fop_ -c 4 -o gpurun_out/prof_$TAG python tools/profile_ops.py --reps 1 > gpurun_out/prof_$TAG.log 2>&1; echo full=$?
ls -la gpurun_out
