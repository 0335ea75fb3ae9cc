set -x
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 1200 python -m pytest tests/test_int_gpu.py tests/test_n4_ops.py -q -x -m gpu > gpurun_out/pytest_int.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_int.log
bash tools/gpu_round2_tma.sh
