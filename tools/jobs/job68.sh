cd $GRAFT_REPO_ROOT
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu68.txt 2>&1; tail -3 gpurun_out/pytest_gpu68.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke68.txt 2>&1; tail -2 gpurun_out/smoke68.txt
timeout 900 python bench.py > gpurun_out/bench68.json 2> gpurun_out/bench68.err; tail -c 400 gpurun_out/bench68.json
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench68_ref.json 2>&1; tail -c 300 gpurun_out/bench68_ref.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 80 --csv --log-file gpurun_out/launches68_bench.csv python bench.py --steps 5 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-configs > /dev/null 2>&1; wc -l gpurun_out/launches68_bench.csv
