python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
export FOP_TUNE_LOG=1 FOP_TUNE_COLD=1
for v in "" "FOP_COL_U=2 FOP_COL_MINB=8" "" "FOP_COL_U=2 FOP_COL_MINB=8" "FOP_COL_U=2 FOP_COL_MINB=6" "FOP_COL_U=4 FOP_COL_MINB=8" "FOP_COL_U=1 FOP_COL_MINB=8"; do
env $v timeout 900 python bench.py --no-cpu > gpurun_out/bench_zf.log 2> gpurun_out/bench_zf.err; echo "[$v] bench=$?"
grep "fop tune" gpurun_out/bench_zf.err | grep col
tail -1 gpurun_out/bench_zf.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),round(d['roofline']['frac'],3),{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"
done
