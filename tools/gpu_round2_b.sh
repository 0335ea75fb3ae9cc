python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
S="timeout 300 python tools/sweep.py"
A="opt:autotune=0"
$S cfg4a "$A" "$A,FOP_ROW_ONEPASS=1" "$A,FOP_ROW_ONEPASS=1,FOP_ROW_MINB=4" "$A,FOP_ROW_ONEPASS=1,FOP_ROW_MINB=2" "$A,FOP_ROW_ONEPASS=1,FOP_BLOCK=128,FOP_ROW_MINB=8" "$A,FOP_ROW_ONEPASS=1,FOP_BLOCK=512,FOP_ROW_MINB=2" "$A,FOP_ROW_MINB=4" > gpurun_out/sweep_row1.log 2>&1
timeout 900 python -m pytest tests/test_transcendental_gpu.py -q -x > gpurun_out/pytest_tr.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_tr.log
