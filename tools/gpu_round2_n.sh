python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
S="timeout 600 python tools/sweep.py"
A="opt:autotune=0"
O="$A,FOP_TR_SMEM_OUT=1"
$S cfg3 "$A" "$O" "$O,FOP_TR_SMEM_MINB=2" "$O,FOP_TR_SMEM_MINB=3" "$O,FOP_TR_SMEM_MINB=6" "$O,FOP_TR_SMEM_BYTES=16384,FOP_TR_SMEM_MINB=8" "$O,FOP_TR_SMEM_BYTES=49152,FOP_TR_SMEM_MINB=3" "$O,FOP_TR_WR_BYTES=16" > gpurun_out/sweep_n.log 2>&1
$S nhwc_nchw_7x7 "$A" "$A,FOP_TR_SMEM_MINB=2" "$A,FOP_TR_SMEM_MINB=6" "$A,FOP_TR_SMEM_BYTES=16384,FOP_TR_SMEM_MINB=8" >> gpurun_out/sweep_n.log 2>&1
grep "^{" gpurun_out/sweep_n.log | python -c "
import sys, json
for l in sys.stdin:
    j=json.loads(l)
    print(j['op'], j['variant'][:80].ljust(80), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
"
