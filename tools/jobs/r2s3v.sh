cd $GRAFT_REPO_ROOT
# config-4 reduce / scan / gather at the config size vs 1 GiB: ncu launch statistics
# (waves per SM, SM active cycles vs elapsed) for the small-problem ceiling
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__waves_per_multiprocessor,launch__grid_size,launch__block_size,launch__registers_per_thread,launch__occupancy_limit_registers,launch__occupancy_limit_shared_mem,launch__occupancy_limit_warps,sm__cycles_active.avg,sm__cycles_active.max,sm__cycles_elapsed.avg,sm__warps_active.avg.pct_of_peak_sustained_active,dram__throughput.avg.pct_of_peak_sustained_elapsed
for c in reduce_mma reduce_blocked gather_mma gather_blocked; do
  timeout 300 ncu --metrics $M --clock-control none -k regex:ll_ -s 3 -c 1 --csv python tools/profile_one.py --case $c --iters 5 > gpurun_out/r2s3v_ncu_$c.csv 2>&1
done
