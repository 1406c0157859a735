cd $GRAFT_REPO_ROOT
M=l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,gpu__time_duration.sum,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread
for o in '{}' '{"thread_bytes": 128}' '{"thread_bytes": 64}' '{"tile_bytes": 32768}' '{"tile_bytes": 32768, "thread_bytes": 128}'; do
  echo "== c3 $o"
  timeout 300 ncu --metrics $M -k regex:ll_ -s 1 -c 1 --csv python tools/profile_one.py --case c3 --iters 2 --opts "$o" 2>&1 | grep -E '"(l1tex|gpu__|sm__|launch__|smsp)' | awk -F'","' '{print $(NF-2), $NF}'
done
for c in c5T c3b; do
  echo "== $c"
  timeout 300 ncu --metrics $M -k regex:ll_ -s 1 -c 1 --csv python tools/profile_one.py --case $c --iters 2 2>&1 | grep -E '"(l1tex|gpu__|sm__|launch__|smsp)' | awk -F'","' '{print $(NF-2), $NF}'
done
