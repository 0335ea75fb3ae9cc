# COL over odd rows: parity of the fold/shift/shfl modes + integer reductions, then the odd-extent sweep
set -x
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 1500 python -m pytest tests/test_odd_gpu.py tests/test_int_gpu.py -q -x -m gpu > gpurun_out/pytest_col.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_col.log
timeout 600 python tools/odd_variety.py > gpurun_out/odd_variety_fold.log 2>&1; echo odd=$?
cut -c1-200 gpurun_out/odd_variety_fold.log
