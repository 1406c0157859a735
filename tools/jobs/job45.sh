cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_matrix.py -m gpu -q > gpurun_out/pytest45_matrix.txt 2>&1; tail -3 gpurun_out/pytest45_matrix.txt
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu45.txt 2>&1; tail -3 gpurun_out/pytest_gpu45.txt
timeout 600 python tools/sweep.py --only matrix > gpurun_out/sweep45_matrix.jsonl 2>&1; cat gpurun_out/sweep45_matrix.jsonl | cut -c1-220
M=l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,smsp__sass_inst_executed_op_ldsm.sum,smsp__sass_inst_executed_op_shared_stsm.sum,gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for c in c3b c3bvec c2fsmem c2fsmemvec c3f c3fvec; do
  timeout 300 ncu --metrics $M -k regex:ll_ -s 1 -c 1 --csv python tools/profile_one.py --case $c --iters 2 > gpurun_out/ncu45_$c.csv 2>&1
  LL_ISOLATE_SMEM=1 timeout 300 ncu --metrics $M -k regex:ll_ -c 1 --csv python tools/profile_one.py --case $c --iters 1 > gpurun_out/ncu45_iso_$c.csv 2>&1
done
for c in c3b c2fsmem; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 1 -c 1 -o gpurun_out/prof45_$c python tools/profile_one.py --case $c --iters 2 > /dev/null 2>&1
done
ls gpurun_out | grep 45
