python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
S="timeout 300 python tools/sweep.py"
A="opt:autotune=0"
V="$A,FOP_VEC_BYTES=32,FOP_ROW_PFORCE=2"
$S cfg4a "$A" "$V,FOP_ROW_MINB=2" "$V,FOP_ROW_MINB=3" "$V,FOP_ROW_MINB=2,FOP_ROW_PREFETCH=0" "$V,FOP_ROW_MINB=2,FOP_ROW_HOIST=0" "$V,FOP_ROW_MINB=2,FOP_BLOCK=128" "$V,FOP_ROW_MINB=1,FOP_BLOCK=512" "$A,FOP_ROW_PFORCE=2,FOP_ROW_MINB=2" "$A,FOP_ROW_PFORCE=2,FOP_ROW_MINB=3" > gpurun_out/sweep_e.log 2>&1
