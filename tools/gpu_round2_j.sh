python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 900 python -m pytest tests/test_odd_gpu.py -q -x -k "column" > gpurun_out/pytest_colodd.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_colodd.log
timeout 600 python tools/odd_variety.py > gpurun_out/odd_variety_r02.log 2>&1; echo odd=$?
head -3 gpurun_out/odd_variety_r02.log
