python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu3.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu3.log
S="python tools/sweep.py"
$S cfg2 "" "FOP_PACKED=0"
$S cfg3 "" "FOP_PACKED=0" "FOP_TR_U=1,FOP_TR_MINB=2"
$S cfg4a "" "FOP_PACKED=0" "FOP_ROW_MINB=2" "FOP_ROW_MINB=4" "FOP_ROW_PREFETCH=0"
$S cfg4b "" "FOP_PACKED=0" "FOP_COL_U=4,FOP_COL_MINB=3" "FOP_COL_U=8,FOP_COL_MINB=3"
python bench.py --steps 100 > gpurun_out/bench3.log 2>&1; tail -c 600 gpurun_out/bench3.log
