# ROW_REDUCE: warps per SM vs rows-per-warp rounds (cfg4a: 32768 rows; 24 warps/SM -> 9.22 rows per warp, 25 -> 8.86)
timeout 900 python tools/sweep.py cfg4a "" "FOP_BLOCK=160,FOP_ROW_MINB=5" "FOP_BLOCK=800,FOP_ROW_MINB=1" "FOP_BLOCK=96,FOP_ROW_MINB=8" "FOP_BLOCK=416,FOP_ROW_MINB=2" "FOP_BLOCK=64,FOP_ROW_MINB=13" "FOP_BLOCK=128,FOP_ROW_MINB=7" "" > gpurun_out/sweep_rowbal.log 2>&1; echo sweep=$?
timeout 900 python tools/sweep.py bert_layernorm "" "FOP_BLOCK=160,FOP_ROW_MINB=5" "FOP_BLOCK=800,FOP_ROW_MINB=1" >> gpurun_out/sweep_rowbal.log 2>&1; echo sweep2=$?
cut -c1-230 gpurun_out/sweep_rowbal.log
