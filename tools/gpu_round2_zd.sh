python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
export FOP_TUNE_LOG=1
for i in 1 2 3; do
timeout 900 python bench.py --no-cpu --no-steady > gpurun_out/bench_zd$i.log 2> gpurun_out/bench_zd$i.err; echo bench=$?
grep "fop tune" gpurun_out/bench_zd$i.err | grep transpose
tail -1 gpurun_out/bench_zd$i.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),{k:(v['kernel'],round(v['GB_s'])) for k,v in d['config']['per_op'].items()})"
done
