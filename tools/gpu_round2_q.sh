set -x
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
timeout 900 python -m pytest tests/test_fuzz.py tests/test_odd_gpu.py -q -x -m gpu -k "regression or pipelined or bias or nhwc" > gpurun_out/pytest_q.log 2>&1; echo pytest=$?
tail -2 gpurun_out/pytest_q.log
SEEDS="35 37" COUNT=300 bash tools/gpu_fuzz.sh
bash tools/gpu_round2_p.sh
SAN_TOOLS="initcheck" SAN_TIMEOUT=1500 bash tools/gpu_sanitize.sh
