python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
rm -f gpurun_out/sweep_ewgrid.log
V='"" "FOP_EW_U=2,FOP_EW_MINB=4" "FOP_EW_U=4,FOP_EW_MINB=2" "FOP_EW_U=2,FOP_EW_MINB=3" "FOP_EW_U=4,FOP_EW_MINB=3" "FOP_EW_U=1,FOP_EW_MINB=8" "FOP_EW_U=2,FOP_EW_MINB=4,FOP_SMEM_TABLES=0" "FOP_EW_U=4,FOP_EW_MINB=2,FOP_SMEM_TABLES=0"'
for op in cfg2 mobilenet_bn_relu6 resnext_bn_add_relu vgg_bias_relu; do eval timeout 300 python tools/sweep.py $op $V >> gpurun_out/sweep_ewgrid.log 2>&1; done
grep "^{" gpurun_out/sweep_ewgrid.log | python -c "
import sys, json
for l in sys.stdin:
    j=json.loads(l)
    print(j[\"op\"].ljust(22), j[\"variant\"].ljust(44), \"%.0f\" % j.get(\"GBs_median\",0), \"%.1f us\" % j.get(\"us_median\",0), j.get(\"grid\"), j.get(\"error\",\"\")[:200])
"
