cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2ab_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "collective_stages or device" > gpurun_out/r2ab_pytest.txt 2>&1
tail -3 gpurun_out/r2ab_pytest.txt
