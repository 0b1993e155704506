mkdir -p gpurun_out
L=paper_conf_sc_gundaboluvt21_b200/libfastz.so
cp $L /tmp/cur.so
for v in head prof_m1 prof_m6; do
  cp ab_libs/$v.so $L
  timeout 900 ncu --metrics gpu__time_duration.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,smsp__inst_executed.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,launch__occupancy_limit_shared_mem,launch__occupancy_limit_registers,launch__shared_mem_config_size,launch__registers_per_thread,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:k_inspect -c 1 --csv python bench.py --profile --no-cpu-baseline > gpurun_out/conf_$v.csv 2>/dev/null
done
cp /tmp/cur.so $L
VARIANTS="head prof_m6" bash tools/ab.sh
