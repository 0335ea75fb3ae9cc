timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_final1.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_final1.log
for s in 18 19 20; do timeout 900 python tools/fuzz_campaign.py --seed $s --count 300 --repeat > gpurun_out/fuzz_s$s.log 2>&1; echo fuzz_$s=$?; grep -E '^\{|^[0-9]+ ' gpurun_out/fuzz_s$s.log | head -3 | cut -c1-300; done
