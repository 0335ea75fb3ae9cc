python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
S="timeout 600 python tools/sweep.py"
A="opt:autotune=0"
$S cfg4a "$A" "$A,FOP_BLOCK=64,FOP_ROW_MINB=12" "$A,FOP_BLOCK=128,FOP_ROW_MINB=6" "$A,FOP_BLOCK=64,FOP_ROW_MINB=16" "$A,FOP_BLOCK=32,FOP_ROW_MINB=24" > gpurun_out/sweep_v.log 2>&1
$S cfg4b "$A" "$A,FOP_BLOCK=128,FOP_COL_MINB=12" "$A,FOP_BLOCK=64,FOP_COL_MINB=24" "$A,FOP_BLOCK=128,FOP_COL_MINB=8" >> gpurun_out/sweep_v.log 2>&1
$S cfg2 "$A,FOP_VEC_BYTES=32,FOP_EW_U=4,FOP_EW_MINB=1" "$A,FOP_VEC_BYTES=32,FOP_EW_U=4,FOP_EW_MINB=4,FOP_BLOCK=64" "$A,FOP_VEC_BYTES=32,FOP_EW_U=4,FOP_EW_MINB=8,FOP_BLOCK=32" >> gpurun_out/sweep_v.log 2>&1
grep "^{" gpurun_out/sweep_v.log | python -c "
import sys, json
for l in sys.stdin:
    j=json.loads(l)
    print(j['op'], j['variant'][:90].ljust(90), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
"
