cd $GRAFT_REPO_ROOT
# SASS-attributed shared-memory wavefronts (per instruction, address-derived) vs the bytes the
# instructions require: ideal wavefronts = bytes / 128.  Unlike l1tex__data_bank_conflicts_*,
# these are not charged with data-pipe cycles taken by concurrent global traffic.
M=sm__sass_l1tex_data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,sm__sass_l1tex_data_pipe_lsu_wavefronts_mem_shared_op_st.sum,sm__sass_l1tex_data_pipe_lsu_wavefronts_mem_shared_op_ldsm.sum,sm__sass_l1tex_data_pipe_lsu_wavefronts_mem_shared_op_stsm.sum,sm__sass_data_bytes_mem_shared_op_ld.sum,sm__sass_data_bytes_mem_shared_op_st.sum,sm__sass_data_bytes_mem_shared_op_ldsm.sum,sm__sass_data_bytes_mem_shared_op_stsm.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,gpu__time_duration.sum
for c in c3 c3b c5T n1 c1bsmem c2smem c3f; do
  echo "== $c"
  timeout 300 ncu --metrics $M -k regex:ll_ -s 1 -c 1 --csv python tools/profile_one.py --case $c --iters 2 2>&1 | grep -E '"(l1tex|gpu__|sm__|smsp)' | awk -F'","' '{print $(NF-2), $NF}'
done > gpurun_out/sass_wavefronts59.txt 2>&1
cat gpurun_out/sass_wavefronts59.txt | head -120
timeout 900 python tools/sweep.py --only generic > gpurun_out/sweep_linear_balance59.jsonl 2> gpurun_out/sweep59.err; cat gpurun_out/sweep_linear_balance59.jsonl; tail -3 gpurun_out/sweep59.err
