# COL_REDUCE finalize ablation (FOP_COL_FIN 0/1/2) + COL parity tests under each
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
S="timeout 300 python tools/sweep.py"
A="opt:autotune=0"
$S cfg4b "$A" "$A,FOP_COL_FIN=1" "$A,FOP_COL_FIN=2" "$A,FOP_COL_FIN=2,FOP_COL_U=8,FOP_COL_MINB=4" "$A,FOP_COL_U=8,FOP_COL_MINB=4" > gpurun_out/sweep_f.log 2>&1
for fin in 1 2; do
FOP_COL_FIN=$fin timeout 1200 python -m pytest tests/test_parity_gpu.py tests/test_repeat_runs.py tests/test_peer.py -q -x -k "col or colsum or cfg4b or repeat or peer or reduce" > gpurun_out/pytest_col$fin.log 2>&1; echo pytest$fin=$?
tail -1 gpurun_out/pytest_col$fin.log
done
