# fuzz campaign seeds (tests/fuzz_gen.py operators vs the oracle, re-runs incl. misaligned)
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
for s in ${SEEDS:-31 32 33}; do timeout 900 python tools/fuzz_campaign.py --seed $s --count ${COUNT:-300} --repeat ${VARIANTS_EVERY:+--variants-every $VARIANTS_EVERY} > gpurun_out/fuzz_r02_s$s.log 2>&1; echo seed$s=$?; tail -2 gpurun_out/fuzz_r02_s$s.log; done
