cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2ad_build.txt 2>&1
timeout 900 python bench.py > gpurun_out/r2ad_bench.txt 2>&1
echo "rc=$?" >> gpurun_out/r2ad_bench.txt
tail -c 400 gpurun_out/r2ad_bench.txt
