python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 900 python -m pytest tests/test_odd_gpu.py -q -x -k "pipelined" > gpurun_out/pytest_pipe.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_pipe.log
S="timeout 600 python tools/sweep.py"
A="opt:autotune=0"
P="$A,FOP_TR_PIPE=1"
$S cfg3 "$A" "$P" "$P,FOP_TR_U=1" "$P,FOP_TR_U=1,FOP_TR_MINB=1" "$P,FOP_TR_U=1,FOP_TR_MINB=2,FOP_BLOCK=128" "$P,FOP_TR_U=2,FOP_BLOCK=128,FOP_TR_MINB=2" "$P,FOP_VEC_BYTES=32,FOP_TR_WR_BYTES=16,FOP_TR_U=1,FOP_TR_MINB=1" > gpurun_out/sweep_pipe.log 2>&1
grep "^{" gpurun_out/sweep_pipe.log | python -c "
import sys, json
for l in sys.stdin:
    j=json.loads(l)
    print(j['op'], j['variant'][:80].ljust(80), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
"
