M=smsp__inst_executed.sum,smsp__thread_inst_executed.sum,gpu__time_duration.sum,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,smsp__thread_inst_executed_per_inst_executed.ratio
for lib in ${LIBS:-libv_base.so libv_theta.so}; do
  echo "== $lib"
  AUTOPIPE_LIB=$PWD/paper_conf_icpp_hulww24_b200/$lib python tools/one_shard.py ${ARGS:-b 8 0}
  AUTOPIPE_LIB=$PWD/paper_conf_icpp_hulww24_b200/$lib ncu --clock-control none --kernel-name regex:k_search_r1 --launch-skip 2 --launch-count 1 --metrics $M python tools/one_shard.py ${ARGS:-b 8 0} 2>&1 | grep -E "inst|duration|pipe_alu|ratio"
done
