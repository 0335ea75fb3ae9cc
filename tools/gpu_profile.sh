# ncu evidence for profiles/ (one GPU): launch list of the bench command + --set full of the tuned kernels
set -x
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches_r01_s2.csv python bench.py --steps 3 --warmup 3 --no-cpu > gpurun_out/launches_bench.log 2>&1; echo ll=$?
ncu --set full --clock-control none --import-source on --profile-from-start off -k regex:fop_ -c 4 -o gpurun_out/prof_r01_s2 python tools/profile_ops.py --reps 1 > gpurun_out/prof.log 2>&1; echo full=$?
ls -la gpurun_out
