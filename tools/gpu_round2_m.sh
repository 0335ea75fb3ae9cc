python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 1200 python -m pytest tests/test_int_gpu.py tests/test_n4_ops.py -q -x -m gpu > gpurun_out/pytest_int.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_int.log
S="timeout 600 python tools/sweep.py"
T="opt:autotune=0,FOP_TR_TMA=1,FOP_TR_TMA_STAGES=2"
$S cfg3 "opt:autotune=0" "$T" "$T,FOP_TMA_L2PROMO=0" "$T,FOP_TMA_L2PROMO=1" "$T,FOP_TMA_L2PROMO=2" "$T,FOP_TR_TMA_WARPS=2" "$T,FOP_TR_TMA_WARPS=6" "$T,FOP_TR_TMA_WARPS=2,FOP_TR_TMA_MINB=2" "$T,FOP_TR_TMA_WARPS=4,FOP_TR_TMA_MINB=2,FOP_TMA_L2PROMO=2" > gpurun_out/sweep_tma2_r02.log 2>&1
grep "^{" gpurun_out/sweep_tma2_r02.log | python -c "
import sys, json
for l in sys.stdin:
    j=json.loads(l)
    print(j['op'], j['variant'][:80].ljust(80), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
"
