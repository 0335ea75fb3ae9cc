python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu4.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu4.log
FOP_GELU_NR=1 timeout 900 python -m pytest tests -m gpu -x -q -k "cfg4a or smoke or row" > gpurun_out/pytest_gpu4nr.log 2>&1; echo "pytest-nr rc=$?"; tail -2 gpurun_out/pytest_gpu4nr.log
S="python tools/sweep.py"
$S cfg4a "" "FOP_GELU_NR=1" "FOP_GELU_NR=1,FOP_ROW_MINB=4" "FOP_GELU_NR=1,FOP_ROW_MINB=2" "FOP_ROW_MINB=4"
$S cfg4b "" "FOP_COL_PIPE=0" "FOP_COL_U=4,FOP_COL_MINB=3" "FOP_COL_U=4,FOP_COL_MINB=4" "FOP_COL_U=8,FOP_COL_MINB=2" "FOP_COL_U=2,FOP_COL_MINB=4" "FOP_COL_U=4,FOP_COL_MINB=2,FOP_BLOCK=512" "FOP_COL_U=4,FOP_COL_MINB=1,FOP_BLOCK=1024"
