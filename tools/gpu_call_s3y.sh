timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_peel2.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_peel2.log
for s in 17 18; do timeout 900 python tools/fuzz_campaign.py --seed $s --count 300 --repeat > gpurun_out/fuzz_s$s.log 2>&1; echo fuzz_$s=$?; tail -1 gpurun_out/fuzz_s$s.log | cut -c1-300; done
