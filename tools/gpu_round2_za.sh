python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
b() { timeout 600 python bench.py --no-cpu --no-steady --steps 100 "$@" 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),{k:(round(v['GB_s'])) for k,v in d['config']['per_op'].items()})"; }
echo default; b
for c in "FOP_TR_TMA_STAGES=2" "FOP_TR_TMA_STAGES=3" "FOP_TR_TMA_STAGES=2 FOP_TR_TMA_WARPS=2 FOP_TR_TMA_MINB=2" "FOP_TR_TMA_STAGES=3 FOP_TR_TMA_WARPS=2 FOP_TR_TMA_MINB=2" "FOP_TR_TMA_STAGES=2 FOP_TMA_L2PROMO=0" "FOP_TR_TMA_STAGES=2 FOP_TR_TMA_WARPS=6" "FOP_TR_TMA_STAGES=2 FOP_TR_TMA_WARPS=3" "FOP_TR_TMA_STAGES=4"; do echo "$c"; env FOP_TR_TMA=1 $c bash -c "$(declare -f b); b"; done
echo default_again; b
