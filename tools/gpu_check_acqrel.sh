# COL finalize: acq_rel arrival atomic vs membar.gl + relaxed atomic (cfg4b, odd fold), parity under it
set -x
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
S="timeout 300 python tools/sweep.py"
A="opt:autotune=0"
for i in 1 2; do
$S cfg4b "$A" "$A,FOP_COL_ACQREL=1" "$A,FOP_COL_U=2,FOP_COL_MINB=8" "$A,FOP_COL_U=2,FOP_COL_MINB=8,FOP_COL_ACQREL=1" 2>&1 | cut -c1-160
$S colsum_1001 "$A" "$A,FOP_COL_ACQREL=1" "$A,FOP_COL_FOLD=0" 2>&1 | cut -c1-160
done
FOP_COL_ACQREL=1 timeout 1200 python -m pytest tests/test_parity_gpu.py tests/test_repeat_runs.py tests/test_odd_gpu.py tests/test_full_size_gpu.py -q -x -k "col or colsum or cfg4b or repeat or reduce or odd" > gpurun_out/pytest_acqrel.log 2>&1; echo pytest=$?
tail -1 gpurun_out/pytest_acqrel.log
