timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_tblv2.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_tblv.log
timeout 900 python tools/fuzz_campaign.py --seed 14 --count 200 --repeat > gpurun_out/fuzz_s14.log 2>&1; echo fuzz=$?; tail -1 gpurun_out/fuzz_s14.log
timeout 900 python tools/ew_variety.py > gpurun_out/ew_variety3.log 2>&1; echo rc=$?
python - <<'PY'
import json
for l in open('gpurun_out/ew_variety3.log'):
    if l.startswith('{'):
        d=json.loads(l)
        if 'error' in d: print(d); continue
        print(f"{d['case']:42s} v={d['vec_loop']}/{d['width']} {d['selected'][0]:16s} {d['us']:8.1f}us {d['GB_s']:7.0f} GB/s copy {d['copy_GB_s']:6.0f} frac {d['frac_of_copy']:.3f}")
PY
