cd $GRAFT_REPO_ROOT
# sustained: the headline step back to back for ~13 s (20000 steps), clocks sampled
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap --format=csv -lms 200 > gpurun_out/r2s3w_clocks.csv &
SMI=$!
timeout 600 python bench.py --steps 20000 --warmup 10 --no-configs --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2s3w_bench_sustained.txt 2>&1
kill $SMI
tail -c 400 gpurun_out/r2s3w_bench_sustained.txt
