#!/bin/bash
# Round-2 sweep recipes: the exact command lists that produced the profiles/r02/ logs.
# usage (on a B200, from the repo root): bash tools/recipes/round2.sh <name>
#   e.g. gpurun --timeout 1800 -- 'bash tools/recipes/round2.sh tma'
# names: a b c d e f g h i j k l m n o p q r s t tma u v w x y z za zb zc zd ze zf col_fold acqrel final rowpf tune2 rowhoist suite_fuzz tma_misalign closing rowtma final2 tiebreak rowcs multirank carveout carveout_tma final3 order2 final4 final5
case "$1" in
a)
  bash tools/gpu_sweep_vec32.sh > gpurun_out/sweep_vec32.log 2>&1; echo sweep=$?
  timeout 900 python -m pytest tests/test_transcendental_gpu.py -q -x > gpurun_out/pytest_tr.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_tr.log
  ;;
b)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 300 python tools/sweep.py"
  A="opt:autotune=0"
  $S cfg4a "$A" "$A,FOP_ROW_ONEPASS=1" "$A,FOP_ROW_ONEPASS=1,FOP_ROW_MINB=4" "$A,FOP_ROW_ONEPASS=1,FOP_ROW_MINB=2" "$A,FOP_ROW_ONEPASS=1,FOP_BLOCK=128,FOP_ROW_MINB=8" "$A,FOP_ROW_ONEPASS=1,FOP_BLOCK=512,FOP_ROW_MINB=2" "$A,FOP_ROW_MINB=4" > gpurun_out/sweep_row1.log 2>&1
  timeout 900 python -m pytest tests/test_transcendental_gpu.py -q -x > gpurun_out/pytest_tr.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_tr.log
  ;;
c)
  # round 2: separate load/store vector widths (FOP_LD_BYTES, FOP_TR_WR_BYTES) on cfg2/cfg3
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 300 python tools/sweep.py"
  A="opt:autotune=0"
  $S cfg3 "$A" "$A,FOP_TR_WR_BYTES=32" "$A,FOP_TR_WR_BYTES=32,FOP_TR_U=1" "$A,FOP_TR_WR_BYTES=32,FOP_TR_U=1,FOP_TR_MINB=1" "$A,FOP_VEC_BYTES=32,FOP_TR_WR_BYTES=32,FOP_TR_U=1,FOP_TR_MINB=1" "$A,FOP_VEC_BYTES=32,FOP_TR_WR_BYTES=16,FOP_TR_U=1,FOP_TR_MINB=1" > gpurun_out/sweep_c.log 2>&1
  $S cfg2 "$A" "$A,FOP_LD_BYTES=32" "$A,FOP_LD_BYTES=32,FOP_EW_U=2,FOP_EW_MINB=2" "$A,FOP_LD_BYTES=32,FOP_EW_U=2,FOP_EW_MINB=3" "$A,FOP_LD_BYTES=32,FOP_EW_U=4,FOP_EW_MINB=2" "$A,FOP_LD_BYTES=32,FOP_EW_U=1,FOP_EW_MINB=4" "$A,FOP_VEC_BYTES=32,FOP_EW_U=2,FOP_EW_MINB=2" "$A,FOP_VEC_BYTES=32,FOP_EW_U=1,FOP_EW_MINB=2" "$A,FOP_VEC_BYTES=32,FOP_EW_U=4,FOP_EW_MINB=1" >> gpurun_out/sweep_c.log 2>&1
  ;;
d)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 300 python tools/sweep.py"
  A="opt:autotune=0"
  V="$A,FOP_VEC_BYTES=32"
  $S cfg2 "$V,FOP_EW_U=4,FOP_EW_MINB=1" "$V,FOP_EW_U=8,FOP_EW_MINB=1" "$V,FOP_EW_U=2,FOP_EW_MINB=1" "$V,FOP_EW_U=4,FOP_EW_MINB=1,FOP_BLOCK=512" "$V,FOP_EW_U=2,FOP_EW_MINB=1,FOP_BLOCK=512" "$V,FOP_EW_U=4,FOP_EW_MINB=2,FOP_BLOCK=128" "$V,FOP_EW_U=4,FOP_EW_MINB=1,FOP_SMEM_TABLES=0" "$A,FOP_LD_BYTES=32,FOP_EW_U=4,FOP_EW_MINB=1" "$A,FOP_LD_BYTES=32,FOP_EW_U=2,FOP_EW_MINB=1,FOP_BLOCK=512" > gpurun_out/sweep_d.log 2>&1
  T="$A,FOP_VEC_BYTES=32,FOP_TR_WR_BYTES=16"
  $S cfg3 "$A" "$T,FOP_TR_U=1,FOP_TR_MINB=1" "$T,FOP_TR_U=1,FOP_TR_MINB=2" "$T,FOP_TR_U=1,FOP_TR_MINB=1,FOP_BLOCK=512" "$T,FOP_TR_U=1,FOP_TR_MINB=3,FOP_BLOCK=128" "$T,FOP_TR_U=1,FOP_TR_MINB=1,FOP_TR_GV=4" "$T,FOP_TR_U=1,FOP_TR_MINB=1,FOP_TR_GV=16" "$T,FOP_TR_U=2,FOP_TR_MINB=1,FOP_BLOCK=128" >> gpurun_out/sweep_d.log 2>&1
  ;;
e)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 300 python tools/sweep.py"
  A="opt:autotune=0"
  V="$A,FOP_VEC_BYTES=32,FOP_ROW_PFORCE=2"
  $S cfg4a "$A" "$V,FOP_ROW_MINB=2" "$V,FOP_ROW_MINB=3" "$V,FOP_ROW_MINB=2,FOP_ROW_PREFETCH=0" "$V,FOP_ROW_MINB=2,FOP_ROW_HOIST=0" "$V,FOP_ROW_MINB=2,FOP_BLOCK=128" "$V,FOP_ROW_MINB=1,FOP_BLOCK=512" "$A,FOP_ROW_PFORCE=2,FOP_ROW_MINB=2" "$A,FOP_ROW_PFORCE=2,FOP_ROW_MINB=3" > gpurun_out/sweep_e.log 2>&1
  ;;
f)
  # COL_REDUCE finalize ablation (FOP_COL_FIN 0/1/2) + COL parity tests under each
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 300 python tools/sweep.py"
  A="opt:autotune=0"
  $S cfg4b "$A" "$A,FOP_COL_FIN=1" "$A,FOP_COL_FIN=2" "$A,FOP_COL_FIN=2,FOP_COL_U=8,FOP_COL_MINB=4" "$A,FOP_COL_U=8,FOP_COL_MINB=4" > gpurun_out/sweep_f.log 2>&1
  for fin in 1 2; do
  FOP_COL_FIN=$fin timeout 1200 python -m pytest tests/test_parity_gpu.py tests/test_repeat_runs.py tests/test_peer.py -q -x -k "col or colsum or cfg4b or repeat or peer or reduce" > gpurun_out/pytest_col$fin.log 2>&1; echo pytest$fin=$?
  tail -1 gpurun_out/pytest_col$fin.log
  done
  ;;
g)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 900 python -m pytest tests/test_odd_gpu.py -q -x > gpurun_out/pytest_odd.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_odd.log
  timeout 600 python tools/odd_variety.py > gpurun_out/odd_variety_r02.log 2>&1; echo odd=$?
  cat gpurun_out/odd_variety_r02.log
  ;;
h)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 900 python -m pytest tests/test_odd_gpu.py tests/test_parity_gpu.py -q -x -k "odd or transpose or nhwc or smem or bias" > gpurun_out/pytest_odd.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_odd.log
  timeout 600 python tools/odd_variety.py > gpurun_out/odd_variety_r02.log 2>&1; echo odd=$?
  cat gpurun_out/odd_variety_r02.log
  timeout 600 python tools/tr_variety.py > gpurun_out/tr_variety_r02.log 2>&1; echo tr=$?
  cat gpurun_out/tr_variety_r02.log
  ;;
i)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 300 python tools/sweep.py"
  A="opt:autotune=0"
  $S nchw_nhwc_c255 "$A" "$A,FOP_TR_WR_BYTES=32" "$A,FOP_TR_SMEM_MINB=2" "$A,FOP_TR_SMEM_MINB=6" "$A,FOP_TR_WR_BYTES=32,FOP_TR_SMEM_MINB=2" "$A,FOP_TR_SMEM_BYTES=16384,FOP_TR_SMEM_MINB=8" "$A,FOP_TR_SMEM_BYTES=65536,FOP_TR_SMEM_MINB=2" "$A,FOP_TR_WR_BYTES=32,FOP_TR_SMEM_BYTES=65536,FOP_TR_SMEM_MINB=2" > gpurun_out/sweep_i.log 2>&1
  $S nhwc_nchw_7x7 "$A" "$A,FOP_TR_SMEM_OM=0" "$A,FOP_TR_WR_BYTES=32" "$A,FOP_TR_SMEM_MINB=2" "$A,FOP_TR_SMEM_MINB=6" >> gpurun_out/sweep_i.log 2>&1
  ;;
j)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 900 python -m pytest tests/test_odd_gpu.py tests/test_int_gpu.py -q -x -k "column or reduction" > gpurun_out/pytest_colodd.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_colodd.log
  S="timeout 600 python tools/sweep.py"
  A="opt:autotune=0"
  for op in colsum_1001; do $S $op "$A" "$A,FOP_COL_XCHG=0" "$A,FOP_COL_U=8,FOP_COL_MINB=4" "$A,FOP_COL_U=2,FOP_COL_MINB=8" "$A,FOP_COL_U=4,FOP_COL_MINB=4"; done > gpurun_out/sweep_colx.log 2>&1
  grep "^{" gpurun_out/sweep_colx.log | python -c "
  import sys, json
  for l in sys.stdin:
      j=json.loads(l)
      print(j['op'], j['variant'][:80].ljust(80), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
  "
  ;;
k)
  # full GPU suite, sanitizers (memcheck + racecheck), one-GPU multi-rank strong-scaling bench
  set -x
  python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
  timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_gpu.log
  SAN_TOOLS="memcheck racecheck" SAN_TIMEOUT=1500 bash tools/gpu_sanitize.sh
  for n in 2 4; do
  FOP_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 2957$n bench.py --gpus $n --steps 5 --warmup 3 --scaling strong --no-cpu --no-steady > gpurun_out/bench_onegpu${n}_strong.log 2>&1; echo strong$n=$?
  tail -1 gpurun_out/bench_onegpu${n}_strong.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(d['value'],d['scaling'],d['config']['global_batch_scale'],d['config']['exchange_check'])"
  done
  timeout 900 python bench.py --steps 5 --warmup 3 --scaling strong --no-cpu --no-steady > gpurun_out/bench_strong1.log 2>&1; echo strong1=$?
  tail -1 gpurun_out/bench_strong1.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(d['value'],d['scaling'],d['config']['global_batch_scale'],d['ms_per_step'])"
  ;;
l)
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 1200 python -m pytest tests/test_int_gpu.py tests/test_n4_ops.py -q -x -m gpu > gpurun_out/pytest_int.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_int.log
  bash tools/gpu_round2_tma.sh
  ;;
m)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 1200 python -m pytest tests/test_int_gpu.py tests/test_n4_ops.py -q -x -m gpu > gpurun_out/pytest_int.log 2>&1; echo pytest=$?
  tail -2 gpurun_out/pytest_int.log
  S="timeout 600 python tools/sweep.py"
  T="opt:autotune=0,FOP_TR_TMA=1,FOP_TR_TMA_STAGES=2"
  $S cfg3 "opt:autotune=0" "$T" "$T,FOP_TMA_L2PROMO=0" "$T,FOP_TMA_L2PROMO=1" "$T,FOP_TMA_L2PROMO=2" "$T,FOP_TR_TMA_WARPS=2" "$T,FOP_TR_TMA_WARPS=6" "$T,FOP_TR_TMA_WARPS=2,FOP_TR_TMA_MINB=2" "$T,FOP_TR_TMA_WARPS=4,FOP_TR_TMA_MINB=2,FOP_TMA_L2PROMO=2" > gpurun_out/sweep_tma2_r02.log 2>&1
  grep "^{" gpurun_out/sweep_tma2_r02.log | python -c "
  import sys, json
  for l in sys.stdin:
      j=json.loads(l)
      print(j['op'], j['variant'][:80].ljust(80), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
  "
  ;;
n)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 600 python tools/sweep.py"
  A="opt:autotune=0"
  O="$A,FOP_TR_SMEM_OUT=1"
  $S cfg3 "$A" "$O" "$O,FOP_TR_SMEM_MINB=2" "$O,FOP_TR_SMEM_MINB=3" "$O,FOP_TR_SMEM_MINB=6" "$O,FOP_TR_SMEM_BYTES=16384,FOP_TR_SMEM_MINB=8" "$O,FOP_TR_SMEM_BYTES=49152,FOP_TR_SMEM_MINB=3" "$O,FOP_TR_WR_BYTES=16" > gpurun_out/sweep_n.log 2>&1
  $S nhwc_nchw_7x7 "$A" "$A,FOP_TR_SMEM_MINB=2" "$A,FOP_TR_SMEM_MINB=6" "$A,FOP_TR_SMEM_BYTES=16384,FOP_TR_SMEM_MINB=8" >> gpurun_out/sweep_n.log 2>&1
  grep "^{" gpurun_out/sweep_n.log | python -c "
  import sys, json
  for l in sys.stdin:
      j=json.loads(l)
      print(j['op'], j['variant'][:80].ljust(80), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
  "
  ;;
o)
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  SEEDS="34 35 36 37" COUNT=300 bash tools/gpu_fuzz.sh
  SAN_TOOLS="synccheck initcheck" SAN_TIMEOUT=1500 bash tools/gpu_sanitize.sh
  ;;
p)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 900 python -m pytest tests/test_odd_gpu.py -q -x -k "pipelined" > gpurun_out/pytest_pipe.log 2>&1; echo pytest=$?
  tail -2 gpurun_out/pytest_pipe.log
  S="timeout 600 python tools/sweep.py"
  A="opt:autotune=0"
  P="$A,FOP_TR_PIPE=1"
  $S cfg3 "$A" "$P" "$P,FOP_TR_U=1" "$P,FOP_TR_U=1,FOP_TR_MINB=1" "$P,FOP_TR_U=1,FOP_TR_MINB=2,FOP_BLOCK=128" "$P,FOP_TR_U=2,FOP_BLOCK=128,FOP_TR_MINB=2" "$P,FOP_VEC_BYTES=32,FOP_TR_WR_BYTES=16,FOP_TR_U=1,FOP_TR_MINB=1" > gpurun_out/sweep_pipe.log 2>&1
  grep "^{" gpurun_out/sweep_pipe.log | python -c "
  import sys, json
  for l in sys.stdin:
      j=json.loads(l)
      print(j['op'], j['variant'][:80].ljust(80), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
  "
  ;;
q)
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 900 python -m pytest tests/test_fuzz.py tests/test_odd_gpu.py -q -x -m gpu -k "regression or pipelined or bias or nhwc" > gpurun_out/pytest_q.log 2>&1; echo pytest=$?
  tail -2 gpurun_out/pytest_q.log
  SEEDS="35 37" COUNT=300 bash tools/gpu_fuzz.sh
  bash tools/gpu_round2_p.sh
  SAN_TOOLS="initcheck" SAN_TIMEOUT=1500 bash tools/gpu_sanitize.sh
  ;;
r)
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 900 compute-sanitizer --tool initcheck --print-limit 20 --error-exitcode 99 python -m pytest tests/test_int_gpu.py tests/test_odd_gpu.py -m gpu -q -x -k "not full_size" -p no:cacheprovider > gpurun_out/san_initcheck2.log 2>&1; echo initcheck=$?
  grep -E "ERROR SUMMARY|passed|failed" gpurun_out/san_initcheck2.log | tail -2
  b() { timeout 600 python bench.py --no-cpu --steps 50 "$@" 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),{k:round(v['GB_s']) for k,v in d['config']['per_op'].items()}, d['clocks']['sm_mhz'])"; }
  echo default; b --no-steady
  echo store_stream; FOP_STORE_POLICY=stream b --no-steady
  echo default2; b --no-steady
  ;;
s)
  set -x
  for n in 2; do
  FOP_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 2958$n bench.py --gpus $n --steps 5 --warmup 3 --no-cpu --no-steady > gpurun_out/bench_onegpu${n}_weak.log 2>&1; echo weak$n=$?
  tail -1 gpurun_out/bench_onegpu${n}_weak.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),d['scaling'],d['config']['parallelism'],d['config']['exchange_check'],d['config']['exchange_note'])"
  done
  ;;
t)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 600 python tools/sweep.py"
  A="opt:autotune=0"
  $S cfg3 "$A" "$A,FOP_BLOCK=128,FOP_TR_MINB=2" "$A,FOP_BLOCK=128,FOP_TR_MINB=3" "$A,FOP_BLOCK=64,FOP_TR_MINB=4" "$A,FOP_BLOCK=64,FOP_TR_MINB=5" "$A,FOP_BLOCK=64,FOP_TR_MINB=6" "$A,FOP_BLOCK=32,FOP_TR_MINB=8" "$A,FOP_BLOCK=96,FOP_TR_MINB=3" "$A,FOP_BLOCK=128,FOP_TR_MINB=2,FOP_VEC_BYTES=32,FOP_TR_WR_BYTES=16,FOP_TR_U=1" "$A,FOP_BLOCK=64,FOP_TR_MINB=4,FOP_VEC_BYTES=32,FOP_TR_WR_BYTES=16,FOP_TR_U=1" "$A,FOP_BLOCK=128,FOP_TR_MINB=2,FOP_TR_PIPE=1" > gpurun_out/sweep_t.log 2>&1
  $S nhwc_nchw_7x7 "$A" > /dev/null 2>&1
  grep "^{" gpurun_out/sweep_t.log | python -c "
  import sys, json
  for l in sys.stdin:
      j=json.loads(l)
      print(j['op'], j['variant'][:90].ljust(90), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
  "
  ;;
tma)
  # round 2: TMA transpose vs the register transpose on cfg3 (verdict item: tune the TMA path or show why not)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 600 python tools/sweep.py"
  A="opt:autotune=0"
  T="$A,FOP_TR_TMA=1"
  $S cfg3 "$A" "$A,FOP_TR_U=1,FOP_TR_MINB=4" "$A,FOP_TR_U=1,FOP_TR_MINB=3" "$T" "$T,FOP_TR_TMA_STAGES=2" "$T,FOP_TR_TMA_STAGES=6" "$T,FOP_TR_TMA_STAGES=8,FOP_TR_TMA_WARPS=2" "$T,FOP_TR_TMA_WARPS=8,FOP_TR_TMA_STAGES=2" "$T,FOP_TR_TMA_WARPS=2,FOP_TR_TMA_STAGES=4,FOP_TR_TMA_MINB=2" "$T,FOP_TR_TMA_WARPS=1,FOP_TR_TMA_STAGES=6,FOP_TR_TMA_MINB=4" "$T,FOP_TR_TMA_WARPS=4,FOP_TR_TMA_STAGES=3,FOP_TR_TMA_MINB=2" "$T,FOP_TR_TMA_WARPS=2,FOP_TR_TMA_STAGES=3,FOP_TR_TMA_MINB=3" > gpurun_out/sweep_tma_r02.log 2>&1
  grep "^{" gpurun_out/sweep_tma_r02.log | python -c "
  import sys, json
  for l in sys.stdin:
      j=json.loads(l)
      print(j['op'], j['variant'][:80].ljust(80), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
  "
  # ncu of the register default and the best-known TMA geometry (one launch each, after tuning/warm-up)
  M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,launch__grid_size,launch__block_size,launch__shared_mem_per_block_dynamic,smsp__average_warp_latency_issue_stalled_long_scoreboard.ratio,smsp__average_warp_latency_issue_stalled_barrier.ratio,smsp__average_warp_latency_issue_stalled_short_scoreboard.ratio,l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_write.sum
  for v in reg tma; do
    if [ $v = tma ]; then export FOP_TR_TMA=1; else unset FOP_TR_TMA; fi
    timeout 300 ncu --metrics $M --clock-control none --profile-from-start off -k regex:fop_transpose -c 1 --csv --log-file gpurun_out/ncu_tr_$v.csv python tools/profile_ops.py --reps 1 --ops cfg3 > /dev/null 2>&1; echo ncu_$v=$?
  done
  unset FOP_TR_TMA
  ;;
u)
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 1500 python -m pytest tests/test_parity_gpu.py tests/test_full_size_gpu.py tests/test_odd_gpu.py tests/test_int_gpu.py -q -x -m gpu -k "transpose or cfg3 or nhwc or tma or every_tuning" > gpurun_out/pytest_tr.log 2>&1; echo pytest=$?
  tail -2 gpurun_out/pytest_tr.log
  timeout 600 python tools/tr_variety.py > gpurun_out/tr_variety_r02b.log 2>&1; echo tr=$?
  python -c "
  import json
  for l in open('gpurun_out/tr_variety_r02b.log'):
      if l.startswith('{'):
          d=json.loads(l); print(d['case'][:40].ljust(40), d['selected'][0], d['selected'][1:], round(d['GB_s']), round(d['frac_of_copy'],3))
  "
  timeout 900 python bench.py --no-cpu --steps 50 > gpurun_out/bench_u.log 2>&1; echo bench=$?
  tail -1 gpurun_out/bench_u.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"
  ;;
v)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 600 python tools/sweep.py"
  A="opt:autotune=0"
  $S cfg4a "$A" "$A,FOP_BLOCK=64,FOP_ROW_MINB=12" "$A,FOP_BLOCK=128,FOP_ROW_MINB=6" "$A,FOP_BLOCK=64,FOP_ROW_MINB=16" "$A,FOP_BLOCK=32,FOP_ROW_MINB=24" > gpurun_out/sweep_v.log 2>&1
  $S cfg4b "$A" "$A,FOP_BLOCK=128,FOP_COL_MINB=12" "$A,FOP_BLOCK=64,FOP_COL_MINB=24" "$A,FOP_BLOCK=128,FOP_COL_MINB=8" >> gpurun_out/sweep_v.log 2>&1
  $S cfg2 "$A,FOP_VEC_BYTES=32,FOP_EW_U=4,FOP_EW_MINB=1" "$A,FOP_VEC_BYTES=32,FOP_EW_U=4,FOP_EW_MINB=4,FOP_BLOCK=64" "$A,FOP_VEC_BYTES=32,FOP_EW_U=4,FOP_EW_MINB=8,FOP_BLOCK=32" >> gpurun_out/sweep_v.log 2>&1
  grep "^{" gpurun_out/sweep_v.log | python -c "
  import sys, json
  for l in sys.stdin:
      j=json.loads(l)
      print(j['op'], j['variant'][:90].ljust(90), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
  "
  ;;
w)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 300 python tools/sweep.py"
  A="opt:autotune=0"
  $S cfg4b "$A" "$A,FOP_COL_FIN=3,FOP_COL_SPIN=1" "$A,FOP_COL_FIN=1,FOP_COL_SPIN=1" "$A,FOP_COL_FIN=2,FOP_COL_SPIN=1" "$A,FOP_COL_FIN=3" > gpurun_out/sweep_w.log 2>&1
  grep "^{" gpurun_out/sweep_w.log | python -c "
  import sys, json
  for l in sys.stdin:
      j=json.loads(l)
      print(j['op'], j['variant'][:90].ljust(90), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
  "
  ;;
x)
  # op order of the (independent) suite ops: suite total and per-op attribution
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  b() { timeout 600 python bench.py --no-cpu --no-steady --steps 100 "$@" 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),{k:round(v['GB_s']) for k,v in d['config']['per_op'].items()})"; }
  for o in cfg2,cfg3,cfg4a,cfg4b cfg2,cfg3,cfg4b,cfg4a cfg3,cfg4b,cfg2,cfg4a cfg4a,cfg2,cfg3,cfg4b cfg3,cfg2,cfg4b,cfg4a cfg4a,cfg4b,cfg2,cfg3 cfg2,cfg4a,cfg3,cfg4b cfg2,cfg3,cfg4a,cfg4b; do echo $o; b --op-order $o; done
  ;;
y)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 900 python -m pytest tests/test_odd_gpu.py tests/test_int_gpu.py -q -x -k "column or reduction" > gpurun_out/pytest_colodd.log 2>&1; echo pytest=$?
  tail -2 gpurun_out/pytest_colodd.log
  S="timeout 600 python tools/sweep.py"
  A="opt:autotune=0"
  $S colsum_1001 "$A,FOP_COL_SHFL=0" "$A" "$A,FOP_COL_MINB=4" "$A,FOP_COL_U=8,FOP_COL_MINB=4" "$A,FOP_COL_U=2,FOP_COL_MINB=8" "$A,FOP_COL_U=2,FOP_COL_MINB=6" "$A,FOP_COL_MINB=5" > gpurun_out/sweep_y.log 2>&1
  grep "^{" gpurun_out/sweep_y.log | python -c "
  import sys, json
  for l in sys.stdin:
      j=json.loads(l)
      print(j['op'], j['variant'][:80].ljust(80), '%.0f' % j.get('GBs_median',0), '%.1f' % j.get('us_median',0), j.get('grid'), j.get('error','')[:200])
  "
  ;;
z)
  # TMA transpose: DRAM bytes read vs L2 promotion and stages (is the 7 % over-fetch promotion?)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,smsp__inst_executed_op_shared_ld.sum,smsp__inst_executed_op_shared_st.sum,lts__t_sectors_srcunit_tex_op_read.sum
  export FOP_TR_TMA=1
  for cfg in "FOP_TR_TMA_STAGES=2" "FOP_TR_TMA_STAGES=2 FOP_TMA_L2PROMO=0" "FOP_TR_TMA_STAGES=2 FOP_TMA_L2PROMO=2" "FOP_TR_TMA_STAGES=4"; do
    env $cfg timeout 300 ncu --metrics $M --clock-control none --profile-from-start off -k regex:fop_transpose -c 1 --csv python tools/profile_ops.py --reps 1 --ops cfg3 2>/dev/null | grep -E "dram__bytes|time_duration|conflicts|shared_ld|shared_st|lts__t" | awk -F'","' -v c="$cfg" '{print c" | "$(NF-2)" "$NF}'
  done
  ;;
za)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  b() { timeout 600 python bench.py --no-cpu --no-steady --steps 100 "$@" 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),{k:(round(v['GB_s'])) for k,v in d['config']['per_op'].items()})"; }
  echo default; b
  for c in "FOP_TR_TMA_STAGES=2" "FOP_TR_TMA_STAGES=3" "FOP_TR_TMA_STAGES=2 FOP_TR_TMA_WARPS=2 FOP_TR_TMA_MINB=2" "FOP_TR_TMA_STAGES=3 FOP_TR_TMA_WARPS=2 FOP_TR_TMA_MINB=2" "FOP_TR_TMA_STAGES=2 FOP_TMA_L2PROMO=0" "FOP_TR_TMA_STAGES=2 FOP_TR_TMA_WARPS=6" "FOP_TR_TMA_STAGES=2 FOP_TR_TMA_WARPS=3" "FOP_TR_TMA_STAGES=4"; do echo "$c"; env FOP_TR_TMA=1 $c bash -c "$(declare -f b); b"; done
  echo default_again; b
  ;;
zb)
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 1800 python -m pytest tests/test_parity_gpu.py tests/test_full_size_gpu.py tests/test_odd_gpu.py tests/test_int_gpu.py -q -x -m gpu -k "transpose or cfg3 or nhwc or tma or every_tuning" > gpurun_out/pytest_tr_zb.log 2>&1; echo pytest=$?
  tail -2 gpurun_out/pytest_tr_zb.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke_zb.log 2>&1; echo smoke=$?; tail -1 gpurun_out/smoke_zb.log
  timeout 600 python tools/tr_variety.py > gpurun_out/tr_variety_zb.log 2>&1; echo tr=$?
  python -c "
  import json
  for l in open('gpurun_out/tr_variety_zb.log'):
      if l.startswith('{'):
          d=json.loads(l); print(d['case'][:40].ljust(40), d['selected'][0], d['selected'][1:], round(d['GB_s']), round(d['frac_of_copy'],3))
  "
  for i in 1 2; do
  timeout 900 python bench.py > gpurun_out/bench_zb$i.log 2>&1; echo bench=$?
  tail -1 gpurun_out/bench_zb$i.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),d['clocks'],{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"
  done
  bash tools/gpu_profile.sh r02t
  ;;
zc)
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 1800 python -m pytest tests/test_full_size_gpu.py tests/test_parity_gpu.py -q -x -m gpu -k "cfg3 or nhwc or tma" > gpurun_out/pytest_tr_zc.log 2>&1; echo pytest=$?
  tail -2 gpurun_out/pytest_tr_zc.log
  timeout 600 python tools/tr_variety.py > gpurun_out/tr_variety_zc.log 2>&1; echo tr=$?
  python -c "
  import json
  for l in open('gpurun_out/tr_variety_zc.log'):
      if l.startswith('{'):
          d=json.loads(l); print(d['case'][:40].ljust(40), d['selected'][0], d['selected'][1:], round(d['GB_s']), round(d['frac_of_copy'],3))
  "
  for i in 1 2; do
  timeout 900 python bench.py --no-cpu > gpurun_out/bench_zc$i.log 2>&1; echo bench=$?
  tail -1 gpurun_out/bench_zc$i.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),d['clocks'],{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"
  done
  ;;
zd)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  export FOP_TUNE_LOG=1
  for i in 1 2 3; do
  timeout 900 python bench.py --no-cpu --no-steady > gpurun_out/bench_zd$i.log 2> gpurun_out/bench_zd$i.err; echo bench=$?
  grep "fop tune" gpurun_out/bench_zd$i.err | grep transpose
  tail -1 gpurun_out/bench_zd$i.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),{k:(v['kernel'],round(v['GB_s'])) for k,v in d['config']['per_op'].items()})"
  done
  ;;
ze)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  export FOP_TUNE_LOG=1
  for c in 1 0 1 0 1 0; do
  FOP_TUNE_COLD=$c timeout 900 python bench.py --no-cpu --no-steady > gpurun_out/bench_ze.log 2> gpurun_out/bench_ze.err; echo cold=$c bench=$?
  grep "fop tune" gpurun_out/bench_ze.err
  tail -1 gpurun_out/bench_ze.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),{k:(v['kernel'],round(v['GB_s'])) for k,v in d['config']['per_op'].items()})"
  done
  ;;
zf)
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  export FOP_TUNE_LOG=1 FOP_TUNE_COLD=1
  for v in "" "FOP_COL_U=2 FOP_COL_MINB=8" "" "FOP_COL_U=2 FOP_COL_MINB=8" "FOP_COL_U=2 FOP_COL_MINB=6" "FOP_COL_U=4 FOP_COL_MINB=8" "FOP_COL_U=1 FOP_COL_MINB=8"; do
  env $v timeout 900 python bench.py --no-cpu > gpurun_out/bench_zf.log 2> gpurun_out/bench_zf.err; echo "[$v] bench=$?"
  grep "fop tune" gpurun_out/bench_zf.err | grep col
  tail -1 gpurun_out/bench_zf.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),round(d['roofline']['frac'],3),{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"
  done
  ;;
col_fold)
  # COL over odd rows: parity of the fold/shift/shfl modes + integer reductions, then the odd-extent sweep
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 1500 python -m pytest tests/test_odd_gpu.py tests/test_int_gpu.py -q -x -m gpu > gpurun_out/pytest_col.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_col.log
  timeout 600 python tools/odd_variety.py > gpurun_out/odd_variety_fold.log 2>&1; echo odd=$?
  cut -c1-200 gpurun_out/odd_variety_fold.log
  ;;
acqrel)
  # COL finalize: acq_rel arrival atomic vs membar.gl + relaxed atomic (cfg4b, odd fold), parity under it
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 300 python tools/sweep.py"
  A="opt:autotune=0"
  for i in 1 2; do
  $S cfg4b "$A" "$A,FOP_COL_ACQREL=1" "$A,FOP_COL_U=2,FOP_COL_MINB=8" "$A,FOP_COL_U=2,FOP_COL_MINB=8,FOP_COL_ACQREL=1" 2>&1 | cut -c1-160
  $S colsum_1001 "$A" "$A,FOP_COL_ACQREL=1" "$A,FOP_COL_FOLD=0" 2>&1 | cut -c1-160
  done
  FOP_COL_ACQREL=1 timeout 1200 python -m pytest tests/test_parity_gpu.py tests/test_repeat_runs.py tests/test_odd_gpu.py tests/test_full_size_gpu.py -q -x -k "col or colsum or cfg4b or repeat or reduce or odd" > gpurun_out/pytest_acqrel.log 2>&1; echo pytest=$?
  tail -1 gpurun_out/pytest_acqrel.log
  ;;
final)
  # Round-2 closing evidence on HEAD: variety sweeps (graph-timed), bench line, smoke
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 900 python tools/odd_variety.py > gpurun_out/odd_variety_final.log 2>&1; echo odd=$?
  timeout 900 python tools/tr_variety.py > gpurun_out/tr_variety_final.log 2>&1; echo tr=$?
  timeout 900 python tools/red_variety.py > gpurun_out/red_variety_final.log 2>&1; echo red=$?
  timeout 900 python bench.py > gpurun_out/bench_final.log 2>&1; echo bench=$?
  ;;
rowpf)
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 300 python tools/sweep.py"
  A="opt:autotune=0"
  $S cfg4a "$A" "$A,FOP_ROW_PREFETCH=2,FOP_BLOCK=128,FOP_ROW_MINB=5" "$A,FOP_ROW_PREFETCH=2,FOP_BLOCK=256,FOP_ROW_MINB=2" "$A,FOP_ROW_PREFETCH=3,FOP_BLOCK=128,FOP_ROW_MINB=4" "$A,FOP_ROW_PREFETCH=2,FOP_BLOCK=96,FOP_ROW_MINB=7" "$A,FOP_ROW_PREFETCH=2,FOP_BLOCK=64,FOP_ROW_MINB=10" "$A" 2>&1 | cut -c1-200
  $S bert_layernorm "$A" "$A,FOP_ROW_PREFETCH=2,FOP_BLOCK=128,FOP_ROW_MINB=5" "$A,FOP_ROW_PREFETCH=2,FOP_BLOCK=256,FOP_ROW_MINB=2" 2>&1 | cut -c1-200
  FOP_SWEEP_AUTOTUNE=0 timeout 600 python tools/ew_variety.py > gpurun_out/ew_def.log 2>&1
  FOP_SWEEP_AUTOTUNE=0 FOP_VEC_BYTES=32 FOP_EW_U=4 FOP_EW_MINB=1 timeout 600 python tools/ew_variety.py > gpurun_out/ew_v32.log 2>&1
  python - <<'PY'
import json
a=[json.loads(l) for l in open("gpurun_out/ew_def.log") if l.startswith("{")]
b=[json.loads(l) for l in open("gpurun_out/ew_v32.log") if l.startswith("{")]
for x,y in zip(a,b): print(x["case"][:50].ljust(50), round(x.get("GB_s",0)), round(y.get("GB_s",0)))
PY
  ;;
tune2)
  # tuner threshold 1.5 % + ROW prefetch-2 candidate: parity of every candidate, N4 ops, two bench lines
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 1500 python -m pytest tests/test_full_size_gpu.py tests/test_n4_ops.py tests/test_parity_gpu.py -q -x -m gpu > gpurun_out/pytest_tune2.log 2>&1; echo pytest=$?
  tail -1 gpurun_out/pytest_tune2.log
  for i in 1 2 3; do
  FOP_TUNE_LOG=1 timeout 900 python bench.py --no-cpu > gpurun_out/bench_tune2_$i.log 2> gpurun_out/bench_tune2_$i.err; echo bench=$?
  grep "fop tune" gpurun_out/bench_tune2_$i.err
  tail -1 gpurun_out/bench_tune2_$i.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"
  done
  ;;
rowhoist)
  # cfg4a: bias reloaded per row (FOP_ROW_HOIST=0) to fit 64 registers and 32 warps/SM
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  S="timeout 300 python tools/sweep.py"
  A="opt:autotune=0"
  $S cfg4a "$A" "$A,FOP_ROW_HOIST=0" "$A,FOP_ROW_HOIST=0,FOP_ROW_MINB=4" "$A,FOP_ROW_HOIST=0,FOP_ROW_MINB=5,FOP_BLOCK=192" "$A,FOP_ROW_HOIST=0,FOP_ROW_MINB=8,FOP_BLOCK=128" "$A,FOP_ROW_HOIST=0,FOP_ROW_MINB=16,FOP_BLOCK=64" "$A,FOP_ROW_HOIST=0,FOP_ROW_MINB=4,FOP_ROW_PREFETCH=0" "$A" 2>&1 | cut -c1-220
  $S bert_layernorm "$A" "$A,FOP_ROW_HOIST=0,FOP_ROW_MINB=4" 2>&1 | cut -c1-220
  ;;
suite_fuzz)
  # full GPU suite + fuzz campaigns on HEAD (compute-sanitizer is closed on this pool)
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu_sf.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_gpu_sf.log
  SEEDS="41 42 43 44 45" COUNT=300 bash tools/gpu_fuzz.sh
  ;;
tma_misalign)
  # the misaligned-TMA tests and the rest of the GPU suite after them
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_tm.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_gpu_tm.log
  ;;
closing)
  # closing evidence on HEAD: smoke, bench line (twice), reference arm, ncu launch list + --set full
  set -x
  python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_closing.log 2>&1; echo smoke=$?
  tail -8 gpurun_out/smoke_closing.log
  for i in 1 2; do
  timeout 900 python bench.py > gpurun_out/bench_closing_$i.log 2>&1; echo bench=$?
  tail -1 gpurun_out/bench_closing_$i.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),d['clocks'],{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"
  done
  timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_closing_ref.log 2>&1; echo ref=$?
  tail -1 gpurun_out/bench_closing_ref.log | cut -c1-300
  bash tools/gpu_profile.sh r02d
  SEEDS="46 47 48 49 50 51" COUNT=300 bash tools/gpu_fuzz.sh
  ;;
rowtma)
  # cfg4a-shaped ROW probe: generated register kernel vs a TMA-fed shared-memory row ring
  set -x
  cd tools/probes && nvcc -gencode arch=compute_100a,code=sm_100a -O3 -fmad=false -I ../../paper_conf_cgo_bastoulzrlsjfjc22_b200/csrc/device -o /tmp/row_tma_probe row_tma_probe.cu && /tmp/row_tma_probe
  ;;
final2)
  # after the seed-51 fixes: full GPU suite, fuzz seeds 51-56, smoke, bench x2, ncu evidence
  set -x
  python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_final2.log 2>&1; echo smoke=$?
  tail -2 gpurun_out/smoke_final2.log
  timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_final2.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_gpu_final2.log
  for i in 1 2; do
  timeout 900 python bench.py > gpurun_out/bench_final2_$i.log 2>&1; echo bench=$?
  tail -1 gpurun_out/bench_final2_$i.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),d['clocks'],{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"
  done
  bash tools/gpu_profile.sh r02e
  SEEDS="51 52 53 54 55 56" COUNT=300 bash tools/gpu_fuzz.sh
  ;;
tiebreak)
  # tuner tie-break (cold ties ranked back to back): three bench lines with the tuner log
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  for i in 1 2 3; do
  FOP_TUNE_LOG=1 timeout 900 python bench.py --no-cpu > gpurun_out/bench_tb_$i.log 2> gpurun_out/bench_tb_$i.err; echo bench=$?
  grep "fop tune" gpurun_out/bench_tb_$i.err
  tail -1 gpurun_out/bench_tb_$i.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"
  done
  timeout 900 python -m pytest tests/test_full_size_gpu.py tests/test_repeat_runs.py -q -m gpu > gpurun_out/pytest_tb.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_tb.log
  ;;
rowcs)
  # ROW stores evict-first (st.global.cs): does cfg4a's y write-back move out of cfg4b's window?
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  b() { timeout 900 python bench.py --no-cpu "$@" 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),round(d['roofline']['frac'],3),{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"; }
  for i in 1 2; do
  echo default; b
  echo row_cs; FOP_ROW_ST_STREAM=1 b
  done
  timeout 300 python tools/sweep.py cfg4a opt:autotune=0 opt:autotune=0,FOP_ROW_ST_STREAM=1 2>&1 | cut -c1-200
  ;;
multirank)
  # functional check of the N > 1 bench path on one GPU (weak + strong; exchange self-test + in-bench parity), final code
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  for mode in weak strong; do
  for n in 2 4; do
  FOP_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 2958$n bench.py --gpus $n --steps 5 --warmup 3 --scaling $mode --no-cpu --no-steady > gpurun_out/bench_onegpu${n}_$mode.log 2>&1; echo $mode$n=$?
  tail -1 gpurun_out/bench_onegpu${n}_$mode.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),d['n_gpus'],d['scaling'],d['config']['global_batch_scale'],d['config']['exchange_check'],d['config'].get('exchange_note'),d['config']['parallelism'])"
  done
  done
  timeout 900 python bench.py --steps 5 --warmup 3 --scaling strong --no-cpu --no-steady > gpurun_out/bench_strong1_final.log 2>&1; echo strong1=$?
  tail -1 gpurun_out/bench_strong1_final.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),d['scaling'],d['config']['global_batch_scale'],d['ms_per_step'])"
  ;;
carveout)
  # one shared-memory carveout for every kernel (FOP_CARVEOUT) vs the driver's per-kernel choice
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  b() { timeout 900 python bench.py --no-cpu "$@" 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),round(d['roofline']['frac'],3),{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"; }
  for i in 1 2; do
  echo default; b
  echo carveout100; FOP_CARVEOUT=100 b
  echo carveout60; FOP_CARVEOUT=60 b
  done
  ;;
carveout_tma)
  # max shared-memory carveout for the TMA transposes only
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  b() { timeout 900 python bench.py --no-cpu "$@" 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),round(d['roofline']['frac'],3),{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"; }
  for i in 1 2; do
  echo default; b
  echo tma100; FOP_CARVEOUT_TMA=100 b
  done
  ;;
final3)
  # closing validation of HEAD: smoke, whole GPU suite, bench line, launch list
  set -x
  python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_final3.log 2>&1; echo smoke=$?
  tail -2 gpurun_out/smoke_final3.log
  timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_final3.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_gpu_final3.log
  timeout 900 python bench.py > gpurun_out/bench_final3.log 2>&1; echo bench=$?
  tail -1 gpurun_out/bench_final3.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),d['clocks'],round(d['e2e']['value'],1),{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"
  timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_final3_ref.log 2>&1; echo ref=$?
  ;;
order2)
  # op-order sweep with the TMA transpose default (each order twice)
  set -x
  python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
  for o in cfg2,cfg3,cfg4a,cfg4b cfg2,cfg3,cfg4b,cfg4a cfg3,cfg2,cfg4a,cfg4b cfg2,cfg4a,cfg3,cfg4b cfg2,cfg4b,cfg3,cfg4a cfg3,cfg4a,cfg2,cfg4b; do
  for i in 1 2; do
  echo $o
  timeout 900 python bench.py --no-cpu --no-steady --op-order $o 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),{k:round(v['GB_s']) for k,v in d['config']['per_op'].items()})"
  done
  done
  ;;
final4)
  # after the fold workspace-offset fix: smoke, whole GPU suite, fuzz 62-65 (variants every 4th), bench line
  set -x
  python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_final4.log 2>&1; echo smoke=$?
  tail -1 gpurun_out/smoke_final4.log
  timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_final4.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_gpu_final4.log
  timeout 900 python bench.py > gpurun_out/bench_final4.log 2>&1; echo bench=$?
  tail -1 gpurun_out/bench_final4.log | python -c "import json,sys;d=json.loads(sys.stdin.read());print(round(d['value']),round(d['ms_per_step']*1e3,1),d['roofline']['kernel'],round(d['roofline']['frac'],3),d['clocks'],round(d['e2e']['value'],1),{k:(v['kernel'],round(v['GB_s']),v['steady'] and round(v['steady']['GB_s'])) for k,v in d['config']['per_op'].items()})"
  SEEDS="62 63 64 65" COUNT=300 VARIANTS_EVERY=4 bash tools/gpu_fuzz.sh
  ;;
final5)
  # the COL workspace-address helper (refactor): COL/odd/int/repeat/fuzz-regression GPU tests, fuzz 66-69, smoke
  set -x
  python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_final5.log 2>&1; echo smoke=$?
  tail -1 gpurun_out/smoke_final5.log
  timeout 2400 python -m pytest tests/test_odd_gpu.py tests/test_int_gpu.py tests/test_repeat_runs.py tests/test_fuzz.py tests/test_full_size_gpu.py tests/test_peer.py tests/test_parity_gpu.py -q -m gpu > gpurun_out/pytest_gpu_final5.log 2>&1; echo pytest=$?
  tail -3 gpurun_out/pytest_gpu_final5.log
  SEEDS="66 67 68 69" COUNT=300 VARIANTS_EVERY=4 bash tools/gpu_fuzz.sh
  ;;
*)
  echo "usage: $0 <name>  (see the names list at the top)"; exit 2
  ;;
esac
