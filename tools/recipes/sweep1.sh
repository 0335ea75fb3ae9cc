set -x
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
S="python tools/sweep.py"
$S cfg2 "" "FOP_EW_U=2,FOP_EW_MINB=4" "FOP_EW_U=4,FOP_EW_MINB=3" "FOP_EW_U=4,FOP_EW_MINB=2" "FOP_EW_U=1,FOP_EW_MINB=8" "FOP_EW_U=2,FOP_EW_MINB=6" "FOP_EW_U=2,FOP_EW_MINB=8" "opt:coalesce_order=1" "opt:max_vec_bytes=32" "opt:coalesce_order=1,opt:max_vec_bytes=32" "FOP_STORE_POLICY=stream" "FOP_EW_U=4,FOP_EW_MINB=4"
$S cfg3 "" "FOP_TR_MINB=2" "FOP_TR_MINB=3" "FOP_TR_MINB=6" "FOP_TR_MINB=8" "opt:coalesce_order=1" "FOP_STORE_POLICY=stream" "opt:max_vec_bytes=32"
$S cfg4a "" "FOP_ROW_PREFETCH=0" "FOP_ROW_MINB=2" "FOP_ROW_MINB=4" "FOP_ROW_PREFETCH=0,FOP_ROW_MINB=4" "opt:max_vec_bytes=32"
$S cfg4b "" "FOP_COL_U=4,FOP_COL_MINB=4" "FOP_COL_U=8,FOP_COL_MINB=2" "FOP_COL_U=4,FOP_COL_MINB=2" "FOP_COL_U=16,FOP_COL_MINB=1" "FOP_COL_U=6,FOP_COL_MINB=3" "opt:max_vec_bytes=32"
