python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 400 python tools/sweep.py cfg3 "" "FOP_TMA_L2PROMO=0" "FOP_TMA_L2PROMO=2" "FOP_TR_TMA_WARPS=8" "FOP_TR_TMA_WARPS=2,FOP_TR_TMA_STAGES=4,FOP_TR_TMA_MINB=2" "FOP_TR_TMA_WARPS=1,FOP_TR_TMA_STAGES=6,FOP_TR_TMA_MINB=4" > gpurun_out/sweep_tma2.log 2>&1; echo "sweep rc=$?"
grep "^{" gpurun_out/sweep_tma2.log | python -c "
import sys, json
for l in sys.stdin:
    j=json.loads(l)
    print(j[\"op\"], j[\"variant\"][:60].ljust(60), \"%.0f\" % j.get(\"GBs_median\",0), \"%.0f\" % j.get(\"GBs_best\",0), \"%.1f\" % j.get(\"us_median\",0), j.get(\"grid\"), j.get(\"error\",\"\")[:200])
"
timeout 300 ncu --set full --clock-control none -k regex:fop_transpose -s 1 -c 1 -o gpurun_out/prof_tma python tools/profile_ops.py --reps 2 --ops cfg3 > /dev/null 2>&1; echo ncu1=$?
FOP_TR_TMA=0 timeout 300 ncu --set full --clock-control none -k regex:fop_transpose -s 1 -c 1 -o gpurun_out/prof_trreg python tools/profile_ops.py --reps 2 --ops cfg3 > /dev/null 2>&1; echo ncu2=$?
