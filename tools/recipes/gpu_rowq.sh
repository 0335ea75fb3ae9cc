rm -f gpurun_out/sweep_rowq4.log
timeout 400 python tools/sweep.py bn_stats_nchw "" "FOP_ROW_Q=8,FOP_ROW_CLUSTERS=16" "FOP_ROW_Q=8,FOP_ROW_CLUSTERS=24" "FOP_ROW_Q=8,FOP_ROW_CLUSTERS=32" "FOP_ROW_Q=8,FOP_ROW_G=16,FOP_ROW_CLUSTERS=16" "FOP_ROW_Q=8,FOP_ROW_G=16,FOP_ROW_CLUSTERS=24" "FOP_ROW_Q=4,FOP_ROW_CLUSTERS=32" "FOP_ROW_Q=4,FOP_ROW_G=16,FOP_ROW_CLUSTERS=32" >> gpurun_out/sweep_rowq4.log 2>&1
grep "^{" gpurun_out/sweep_rowq4.log | python -c "
import sys, json
for l in sys.stdin:
    j=json.loads(l)
    print(j['op'].ljust(22), j['variant'].ljust(44), '%.0f' % j.get('GBs_median',0), '%.1f us' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
"
