python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
export FOP_TUNE_LOG=1
for c in 1 0 1 0 1 0; do
FOP_TUNE_COLD=$c timeout 900 python bench.py --no-cpu --no-steady > gpurun_out/bench_ze.log 2> gpurun_out/bench_ze.err; echo cold=$c bench=$?
grep "fop tune" gpurun_out/bench_ze.err
tail -1 gpurun_out/bench_ze.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),{k:(v['kernel'],round(v['GB_s'])) for k,v in d['config']['per_op'].items()})"
done
