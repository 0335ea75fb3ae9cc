timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_tbl2.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_tbl2.log
timeout 900 python tools/fuzz_campaign.py --seed 24 --count 200 --repeat > gpurun_out/fuzz_s24.log 2>&1; echo fuzz=$?; grep -E '^\{|^[0-9]+ ' gpurun_out/fuzz_s24.log | head -2 | cut -c1-300
timeout 900 python tools/ew_variety.py > gpurun_out/ew_variety4.log 2>&1
grep NHWC gpurun_out/ew_variety4.log | cut -c1-300
