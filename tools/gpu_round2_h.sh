python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 900 python -m pytest tests/test_odd_gpu.py tests/test_parity_gpu.py -q -x -k "odd or transpose or nhwc or smem or bias" > gpurun_out/pytest_odd.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_odd.log
timeout 600 python tools/odd_variety.py > gpurun_out/odd_variety_r02.log 2>&1; echo odd=$?
cat gpurun_out/odd_variety_r02.log
timeout 600 python tools/tr_variety.py > gpurun_out/tr_variety_r02.log 2>&1; echo tr=$?
cat gpurun_out/tr_variety_r02.log
