cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2ac_build.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x -k "fuzz" > gpurun_out/r2ac_pytest.txt 2>&1
tail -3 gpurun_out/r2ac_pytest.txt
