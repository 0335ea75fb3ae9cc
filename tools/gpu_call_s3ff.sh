python -X faulthandler tools/fuzz_one.py 21 294 > gpurun_out/f294b.log 2>&1; echo one=$?; tail -1 gpurun_out/f294b.log
timeout 1500 python -X faulthandler -m pytest tests -m gpu -x -q > gpurun_out/pytest_div.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_div.log
for s in 21 24; do timeout 700 python -X faulthandler tools/fuzz_campaign.py --seed $s --count 300 --repeat > gpurun_out/fuzz_d$s.log 2>&1; echo fuzz_$s=$?; grep -E '^\{|^[0-9]+ ' gpurun_out/fuzz_d$s.log | head -3 | cut -c1-300; done
timeout 900 python tools/red_variety.py > gpurun_out/red_variety10.log 2>&1
grep -E 'layernorm|vocab' gpurun_out/red_variety10.log | cut -c1-200
