python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
S="timeout 600 python tools/sweep.py"
A="opt:autotune=0"
$S cfg3 "$A" "$A,FOP_BLOCK=128,FOP_TR_MINB=2" "$A,FOP_BLOCK=128,FOP_TR_MINB=3" "$A,FOP_BLOCK=64,FOP_TR_MINB=4" "$A,FOP_BLOCK=64,FOP_TR_MINB=5" "$A,FOP_BLOCK=64,FOP_TR_MINB=6" "$A,FOP_BLOCK=32,FOP_TR_MINB=8" "$A,FOP_BLOCK=96,FOP_TR_MINB=3" "$A,FOP_BLOCK=128,FOP_TR_MINB=2,FOP_VEC_BYTES=32,FOP_TR_WR_BYTES=16,FOP_TR_U=1" "$A,FOP_BLOCK=64,FOP_TR_MINB=4,FOP_VEC_BYTES=32,FOP_TR_WR_BYTES=16,FOP_TR_U=1" "$A,FOP_BLOCK=128,FOP_TR_MINB=2,FOP_TR_PIPE=1" > gpurun_out/sweep_t.log 2>&1
$S nhwc_nchw_7x7 "$A" > /dev/null 2>&1
grep "^{" gpurun_out/sweep_t.log | python -c "
import sys, json
for l in sys.stdin:
    j=json.loads(l)
    print(j['op'], j['variant'][:90].ljust(90), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
"
