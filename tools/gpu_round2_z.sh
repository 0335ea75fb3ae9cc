# TMA transpose: DRAM bytes read vs L2 promotion and stages (is the 7 % over-fetch promotion?)
python -m paper_conf_cgo_bastoulzrlsjfjc22_b200.build >/dev/null
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,smsp__inst_executed_op_shared_ld.sum,smsp__inst_executed_op_shared_st.sum,lts__t_sectors_srcunit_tex_op_read.sum
export FOP_TR_TMA=1
for cfg in "FOP_TR_TMA_STAGES=2" "FOP_TR_TMA_STAGES=2 FOP_TMA_L2PROMO=0" "FOP_TR_TMA_STAGES=2 FOP_TMA_L2PROMO=2" "FOP_TR_TMA_STAGES=4"; do
  env $cfg timeout 300 ncu --metrics $M --clock-control none --profile-from-start off -k regex:fop_transpose -c 1 --csv python tools/profile_ops.py --reps 1 --ops cfg3 2>/dev/null | grep -E "dram__bytes|time_duration|conflicts|shared_ld|shared_st|lts__t" | awk -F'","' -v c="$cfg" '{print c" | "$(NF-2)" "$NF}'
done
