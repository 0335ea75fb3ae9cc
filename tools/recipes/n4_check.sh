python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
rm -f gpurun_out/sweep_n4c.log
timeout 300 python tools/sweep.py cfg2 "" "FOP_SMEM_TABLES=0" >> gpurun_out/sweep_n4c.log 2>&1
timeout 300 python tools/sweep.py mobilenet_bn_relu6 "" "FOP_SMEM_TABLES=0" >> gpurun_out/sweep_n4c.log 2>&1
timeout 300 python tools/sweep.py resnext_bn_add_relu "" "FOP_EW_U=2,FOP_EW_MINB=3" "FOP_EW_U=8,FOP_EW_MINB=1" "FOP_EW_U=2,FOP_EW_MINB=4" "FOP_EW_U=4,FOP_EW_MINB=3" >> gpurun_out/sweep_n4c.log 2>&1
grep "^{" gpurun_out/sweep_n4c.log | python -c "
import sys, json
for l in sys.stdin:
    j=json.loads(l)
    print(j[\"op\"].ljust(22), j[\"variant\"].ljust(36), \"%.0f\" % j.get(\"GBs_median\",0), \"%.1f us\" % j.get(\"us_median\",0), j.get(\"grid\"), j.get(\"error\",\"\")[:200])
"
