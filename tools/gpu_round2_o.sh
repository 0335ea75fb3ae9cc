set -x
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
SEEDS="34 35 36 37" COUNT=300 bash tools/gpu_fuzz.sh
SAN_TOOLS="synccheck initcheck" SAN_TIMEOUT=1500 bash tools/gpu_sanitize.sh
