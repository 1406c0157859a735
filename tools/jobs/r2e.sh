cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2e_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "broadcast or bulk" > gpurun_out/r2e_pytest.txt 2>&1
tail -3 gpurun_out/r2e_pytest.txt
timeout 600 python tools/sweep.py --only broadcast > gpurun_out/r2e_sweep_broadcast.jsonl 2>&1
timeout 600 python tools/sweep.py --only bulk > gpurun_out/r2e_sweep_bulk.jsonl 2>&1
cat gpurun_out/r2e_sweep_bulk.jsonl
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__sass_inst_executed_op_shared_ld.sum,smsp__sass_inst_executed_op_shared_st.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_st.sum
for c in c3 c3b; do for pipe in default bulk bulkst; do
  if [ $pipe = default ]; then O='{}'; else O="{\"pipe\":\"$pipe\"}"; fi
  timeout 300 ncu --metrics $M --clock-control none -k regex:ll_ -c 1 -o gpurun_out/r2e_ncu_${c}_${pipe} python tools/profile_one.py --case $c --iters 1 --opts "$O" > gpurun_out/r2e_ncu_${c}_${pipe}.log 2>&1
done; done
ls gpurun_out/*.ncu-rep | head
