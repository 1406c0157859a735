cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s4a_build.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r2s4a_pytest_gpu.txt 2>&1
tail -3 gpurun_out/r2s4a_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s4a_smoke.txt 2>&1
tail -1 gpurun_out/r2s4a_smoke.txt
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap --format=csv -lms 200 > gpurun_out/r2s4a_clocks.csv &
SMI=$!
timeout 900 python bench.py > gpurun_out/r2s4a_bench.txt 2>&1
kill $SMI
tail -c 300 gpurun_out/r2s4a_bench.txt
timeout 300 python bench.py --impl reference --steps 20 --warmup 3 > gpurun_out/r2s4a_ref.txt 2>&1
timeout 600 python tools/oracle_rates.py --cpp > gpurun_out/r2s4a_oracle_rates_cpp.jsonl 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:ll_ -c 60 --csv --log-file gpurun_out/r2s4a_launches.csv python bench.py --steps 20 --warmup 3 --no-configs --no-cpu-baseline --e2e-steps 1 > gpurun_out/r2s4a_bench_under_ncu.txt 2>&1
