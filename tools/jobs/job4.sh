cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu4.txt 2>&1
tail -3 gpurun_out/pytest_gpu4.txt
timeout 600 python tools/sweep.py --only gather,reduce > gpurun_out/sweep4.txt 2>&1
timeout 300 compute-sanitizer --tool racecheck python tools/profile_one.py --case c1bsmem_small --iters 1 > gpurun_out/san_racecheck.txt 2>&1
timeout 300 compute-sanitizer --tool memcheck python tools/profile_one.py --case c3_small --iters 1 > gpurun_out/san_memcheck.txt 2>&1
timeout 300 compute-sanitizer --tool synccheck python tools/profile_one.py --case c3_small --iters 1 > gpurun_out/san_synccheck.txt 2>&1
timeout 300 compute-sanitizer --tool initcheck python tools/profile_one.py --case c2_small --iters 1 > gpurun_out/san_initcheck.txt 2>&1
for c in gather_mma gather_blocked reduce_mma reduce_blocked; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 2 -c 1 -o gpurun_out/prof4_$c python tools/profile_one.py --case $c > gpurun_out/ncu4_$c.log 2>&1
done
