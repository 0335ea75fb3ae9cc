bash tools/gpu_sweep_vec32.sh > gpurun_out/sweep_vec32.log 2>&1; echo sweep=$?
timeout 900 python -m pytest tests/test_transcendental_gpu.py -q -x > gpurun_out/pytest_tr.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_tr.log
