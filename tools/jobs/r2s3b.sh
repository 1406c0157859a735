cd $GRAFT_REPO_ROOT
# control experiment for ncu's smem bank-conflict counter (tools/smem_counter_control.cu)
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o gpurun_out/smem_ctl tools/smem_counter_control.cu
for m in 0 1 2; do ./gpurun_out/smem_ctl $m 20; done > gpurun_out/r2s3b_ctl_timing.jsonl 2>&1
cat gpurun_out/r2s3b_ctl_timing.jsonl
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,sm__sass_l1tex_data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,sm__sass_l1tex_data_pipe_lsu_wavefronts_mem_shared_op_st.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum
for m in 0 1 2; do
  timeout 300 ncu --metrics $M --clock-control none -c 1 --csv ./gpurun_out/smem_ctl $m 1 > gpurun_out/r2s3b_ncu_ctl_mode$m.csv 2>&1
done
rm -f gpurun_out/smem_ctl
