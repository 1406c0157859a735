cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2h_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "table3 or device_loopback" > gpurun_out/r2h_pytest.txt 2>&1
tail -3 gpurun_out/r2h_pytest.txt
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r2h_bench.txt 2>&1
tail -c 300 gpurun_out/r2h_bench.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:ll_ -c 60 --csv --log-file gpurun_out/r2h_launches_bench.csv python bench.py --steps 20 --warmup 3 --no-configs --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2h_bench_under_ncu.txt 2>&1
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed_op_shfl.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum
for c in reduce_mma reduce_blocked gather_mma gather_blocked; do
timeout 300 ncu --metrics $M --clock-control none -k regex:ll_ -s 2 -c 1 -o gpurun_out/r2h_ncu_$c python tools/profile_one.py --case $c --iters 4 > gpurun_out/r2h_ncu_$c.log 2>&1
done
