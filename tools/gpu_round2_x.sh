# op order of the (independent) suite ops: suite total and per-op attribution
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
b() { timeout 600 python bench.py --no-cpu --no-steady --steps 100 "$@" 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),{k:round(v['GB_s']) for k,v in d['config']['per_op'].items()})"; }
for o in cfg2,cfg3,cfg4a,cfg4b cfg2,cfg3,cfg4b,cfg4a cfg3,cfg4b,cfg2,cfg4a cfg4a,cfg2,cfg3,cfg4b cfg3,cfg2,cfg4b,cfg4a cfg4a,cfg4b,cfg2,cfg3 cfg2,cfg4a,cfg3,cfg4b cfg2,cfg3,cfg4a,cfg4b; do echo $o; b --op-order $o; done
