cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s3z_build.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -q -k "scan or graph" > gpurun_out/r2s3z_pytest_scan.txt 2>&1
tail -2 gpurun_out/r2s3z_pytest_scan.txt
timeout 600 python tools/sweep.py --only c4rows > gpurun_out/r2s3z_c4rows.jsonl 2>&1
LL_AUX_MIN_BLOCKS=0 timeout 600 python tools/sweep.py --only c4rows > gpurun_out/r2s3z_c4rows_nohint.jsonl 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s3z_smoke.txt 2>&1
tail -1 gpurun_out/r2s3z_smoke.txt
