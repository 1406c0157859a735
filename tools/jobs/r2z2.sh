cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2z2_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "reduce or gather or table4" > gpurun_out/r2z2_pytest.txt 2>&1
tail -2 gpurun_out/r2z2_pytest.txt
