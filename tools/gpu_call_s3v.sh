timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_tblv3.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_tblv3.log
