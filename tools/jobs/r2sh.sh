cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2sh_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "split_tiles or more_warps" > gpurun_out/r2sh_pytest.txt 2>&1
tail -2 gpurun_out/r2sh_pytest.txt
timeout 900 python tools/sweep.py --only split > gpurun_out/r2sh_split.jsonl 2> gpurun_out/r2sh_split.err
cat gpurun_out/r2sh_split.jsonl
tail -3 gpurun_out/r2sh_split.err
