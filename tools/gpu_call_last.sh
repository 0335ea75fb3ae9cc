bash tools/gpu_check.sh
SAN_TOOLS="memcheck" SAN_TIMEOUT=900 bash tools/gpu_sanitize.sh 2>&1 | grep -E '=|SUMMARY|passed|failed' | grep -v '^+' | head -3
