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
