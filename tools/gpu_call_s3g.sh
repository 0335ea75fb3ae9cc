for op in bert_layernorm cfg4a bert_softmax; do
timeout 600 python tools/sweep.py $op "opt:autotune=0" "opt:autotune=0,FOP_ROW_MINB=2" "opt:autotune=0,FOP_BLOCK=160,FOP_ROW_MINB=5" "opt:autotune=0,FOP_BLOCK=160,FOP_ROW_MINB=2" "opt:autotune=0,FOP_BLOCK=128,FOP_ROW_MINB=6" "opt:autotune=0,FOP_ROW_MINB=4" "opt:autotune=1" >> gpurun_out/sweep_rowexp.log 2>&1
done
python - <<'PY'
import json
for l in open("gpurun_out/sweep_rowexp.log"):
    if l.startswith("{"):
        d=json.loads(l); print(d["op"], d["variant"], round(d.get("us_median",0),2), round(d.get("GBs_median",0)), d.get("selected", ""), d.get("error",""))
    else: print(l.rstrip()[:200])
PY
