cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2m_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "gather" > gpurun_out/r2m_pytest.txt 2>&1
tail -3 gpurun_out/r2m_pytest.txt
timeout 600 python tools/sweep.py --only gtma > gpurun_out/r2m_sweep_gather.jsonl 2>&1
cat gpurun_out/r2m_sweep_gather.jsonl
