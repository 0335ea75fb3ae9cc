python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 900 python -m pytest tests/test_odd_gpu.py tests/test_int_gpu.py -q -x -k "column or reduction" > gpurun_out/pytest_colodd.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_colodd.log
S="timeout 600 python tools/sweep.py"
A="opt:autotune=0"
$S colsum_1001 "$A,FOP_COL_SHFL=0" "$A" "$A,FOP_COL_MINB=4" "$A,FOP_COL_U=8,FOP_COL_MINB=4" "$A,FOP_COL_U=2,FOP_COL_MINB=8" "$A,FOP_COL_U=2,FOP_COL_MINB=6" "$A,FOP_COL_MINB=5" > gpurun_out/sweep_y.log 2>&1
grep "^{" gpurun_out/sweep_y.log | python -c "
import sys, json
for l in sys.stdin:
    j=json.loads(l)
    print(j['op'], j['variant'][:80].ljust(80), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
"
