# Evidence refresh on HEAD (one GPU): ncu launch list + --set full of the tuned kernels,
# then the odd-extent and transpose variety sweeps.
# usage: bash tools/gpu_evidence.sh <tag>
set -x
TAG=${1:-r02}
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
bash tools/gpu_profile.sh $TAG
timeout 900 python tools/odd_variety.py > gpurun_out/odd_variety_$TAG.log 2>&1; echo odd=$?
timeout 900 python tools/tr_variety.py > gpurun_out/tr_variety_$TAG.log 2>&1; echo tr=$?
