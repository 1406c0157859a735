cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu3.txt 2>&1
tail -3 gpurun_out/pytest_gpu3.txt
timeout 600 python tools/sweep.py --only gather,reduce > gpurun_out/sweep3.txt 2>&1
for c in c3 c2smem c1bsmem; do
LL_ISOLATE_SMEM=1 timeout 300 ncu --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum -k regex:ll_ -c 1 python tools/profile_one.py --case $c --iters 1 > gpurun_out/ncu_isolate_$c.txt 2>&1
done
timeout 300 ncu --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum -k regex:ll_ -c 1 python tools/profile_one.py --case reduce_mma --iters 1 > gpurun_out/ncu_reduce_l1.txt 2>&1
