# round 2: separate load/store vector widths (FOP_LD_BYTES, FOP_TR_WR_BYTES) on cfg2/cfg3
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
S="timeout 300 python tools/sweep.py"
A="opt:autotune=0"
$S cfg3 "$A" "$A,FOP_TR_WR_BYTES=32" "$A,FOP_TR_WR_BYTES=32,FOP_TR_U=1" "$A,FOP_TR_WR_BYTES=32,FOP_TR_U=1,FOP_TR_MINB=1" "$A,FOP_VEC_BYTES=32,FOP_TR_WR_BYTES=32,FOP_TR_U=1,FOP_TR_MINB=1" "$A,FOP_VEC_BYTES=32,FOP_TR_WR_BYTES=16,FOP_TR_U=1,FOP_TR_MINB=1" > gpurun_out/sweep_c.log 2>&1
$S cfg2 "$A" "$A,FOP_LD_BYTES=32" "$A,FOP_LD_BYTES=32,FOP_EW_U=2,FOP_EW_MINB=2" "$A,FOP_LD_BYTES=32,FOP_EW_U=2,FOP_EW_MINB=3" "$A,FOP_LD_BYTES=32,FOP_EW_U=4,FOP_EW_MINB=2" "$A,FOP_LD_BYTES=32,FOP_EW_U=1,FOP_EW_MINB=4" "$A,FOP_VEC_BYTES=32,FOP_EW_U=2,FOP_EW_MINB=2" "$A,FOP_VEC_BYTES=32,FOP_EW_U=1,FOP_EW_MINB=2" "$A,FOP_VEC_BYTES=32,FOP_EW_U=4,FOP_EW_MINB=1" >> gpurun_out/sweep_c.log 2>&1
