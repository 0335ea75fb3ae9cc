timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
b() { python bench.py --no-cpu --steps 100 "$@" 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['clocks']['sm_mhz'],d['clocks']['reasons'],d['config']['launch'])"; }
echo graph; b
echo eager_many; b --no-graph
echo nopdl; b --no-pdl
echo graph; b
python tools/pdl_time.py 2>&1 | tail -1
