python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu2.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu2.log
S="python tools/sweep.py"
$S cfg2 "" "FOP_EW_U=4,FOP_EW_MINB=2" "FOP_EW_U=2,FOP_EW_MINB=3" "FOP_EW_U=2,FOP_EW_MINB=2" "FOP_EW_U=8,FOP_EW_MINB=1" "FOP_BLOCK=512,FOP_EW_MINB=2" "FOP_BLOCK=128,FOP_EW_MINB=8" "FOP_BLOCK=1024,FOP_EW_MINB=1" "opt:max_vec_bytes=32,FOP_EW_U=4,FOP_EW_MINB=2"
$S cfg3 "" "FOP_TR_MINB=1" "FOP_TR_U=2,FOP_TR_MINB=2" "FOP_TR_U=2,FOP_TR_MINB=1" "FOP_TR_U=4,FOP_TR_MINB=1" "FOP_BLOCK=128,FOP_TR_MINB=4" "FOP_BLOCK=512,FOP_TR_MINB=1" "FOP_TR_U=2,FOP_BLOCK=128,FOP_TR_MINB=3"
