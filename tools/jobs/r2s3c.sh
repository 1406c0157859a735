cd $GRAFT_REPO_ROOT
# control experiment for ncu's smem bank-conflict counter (tools/smem_counter_control.cu):
# conflict-free lane-linear STS/LDS exchange, varying loads in flight per thread (vpt),
# the load's L1 policy and the grid shape (persistent vs one tile per CTA as the product)
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o gpurun_out/smem_ctl tools/smem_counter_control.cu
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,sm__sass_l1tex_data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,sm__sass_l1tex_data_pipe_lsu_wavefronts_mem_shared_op_st.sum,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active
for vpt in 8 16; do for na in 0 1; do for one in 0 1; do for m in 0 1 2; do
  ./gpurun_out/smem_ctl $m 20 $vpt $na $one >> gpurun_out/r2s3c_ctl_timing.jsonl 2>&1
  timeout 300 ncu --metrics $M --clock-control none -c 1 --csv ./gpurun_out/smem_ctl $m 1 $vpt $na $one > gpurun_out/r2s3c_ncu_ctl_m${m}_v${vpt}_na${na}_one${one}.csv 2>&1
done; done; done; done
# the product's config-3 kernel in the same session for comparison
timeout 300 ncu --metrics $M --clock-control none -k regex:ll_ -c 1 --csv python tools/profile_one.py --case c3 --iters 1 > gpurun_out/r2s3c_ncu_c3.csv 2>&1
timeout 300 ncu --metrics $M --clock-control none -k regex:ll_ -c 1 --csv python tools/profile_one.py --case c3 --iters 1 --opts '{"thread_bytes": 128}' > gpurun_out/r2s3c_ncu_c3_tb128.csv 2>&1
rm -f gpurun_out/smem_ctl
