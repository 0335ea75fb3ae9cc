python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
S="timeout 300 python tools/sweep.py"
A="opt:autotune=0"
$S nchw_nhwc_c255 "$A" "$A,FOP_TR_WR_BYTES=32" "$A,FOP_TR_SMEM_MINB=2" "$A,FOP_TR_SMEM_MINB=6" "$A,FOP_TR_WR_BYTES=32,FOP_TR_SMEM_MINB=2" "$A,FOP_TR_SMEM_BYTES=16384,FOP_TR_SMEM_MINB=8" "$A,FOP_TR_SMEM_BYTES=65536,FOP_TR_SMEM_MINB=2" "$A,FOP_TR_WR_BYTES=32,FOP_TR_SMEM_BYTES=65536,FOP_TR_SMEM_MINB=2" > gpurun_out/sweep_i.log 2>&1
$S nhwc_nchw_7x7 "$A" "$A,FOP_TR_SMEM_OM=0" "$A,FOP_TR_WR_BYTES=32" "$A,FOP_TR_SMEM_MINB=2" "$A,FOP_TR_SMEM_MINB=6" >> gpurun_out/sweep_i.log 2>&1
