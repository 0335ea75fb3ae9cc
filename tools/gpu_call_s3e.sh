timeout 600 python -m pytest tests/test_parity_gpu.py -x -q -k "row_block_geometries or cfg4a" > gpurun_out/pytest_rowgeo.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_rowgeo.log
timeout 900 python tools/sweep.py bert_layernorm "" "opt:autotune=1" > gpurun_out/sweep_rowtune.log 2>&1
timeout 900 python tools/sweep.py bert_softmax "" "opt:autotune=1" "FOP_BLOCK=160,FOP_ROW_MINB=5" >> gpurun_out/sweep_rowtune.log 2>&1
timeout 900 python tools/sweep.py cfg4a "" "opt:autotune=1" >> gpurun_out/sweep_rowtune.log 2>&1; echo sweep=$?
cut -c1-260 gpurun_out/sweep_rowtune.log
