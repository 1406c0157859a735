cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2g_build.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r2g_pytest_gpu.txt 2>&1
tail -3 gpurun_out/r2g_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2g_smoke.txt 2>&1
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap --format=csv -lms 200 > gpurun_out/r2g_clocks.csv &
SMI=$!
timeout 900 python bench.py > gpurun_out/r2g_bench.txt 2>&1
kill $SMI
tail -c 400 gpurun_out/r2g_bench.txt
timeout 300 python bench.py --impl reference --steps 20 --warmup 3 > gpurun_out/r2g_ref.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2g_launches.csv python bench.py --steps 20 --warmup 3 --no-configs --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2g_bench_under_ncu.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ll_tile -s 5 -c 1 -o gpurun_out/r2g_prof_c2 python tools/profile_one.py --case c2 --iters 7 > gpurun_out/r2g_prof_c2.log 2>&1
ls -la gpurun_out | tail -5
