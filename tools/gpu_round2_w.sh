python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
S="timeout 300 python tools/sweep.py"
A="opt:autotune=0"
$S cfg4b "$A" "$A,FOP_COL_FIN=3,FOP_COL_SPIN=1" "$A,FOP_COL_FIN=1,FOP_COL_SPIN=1" "$A,FOP_COL_FIN=2,FOP_COL_SPIN=1" "$A,FOP_COL_FIN=3" > gpurun_out/sweep_w.log 2>&1
grep "^{" gpurun_out/sweep_w.log | python -c "
import sys, json
for l in sys.stdin:
    j=json.loads(l)
    print(j['op'], j['variant'][:90].ljust(90), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
"
