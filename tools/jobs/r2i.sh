cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2i_build.txt 2>&1
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in racecheck memcheck synccheck; do
  for c in "bcastS901" "c3_small" ; do
    for o in '{}' '{"pipe":"bulk"}' '{"pipe":"bulkst"}'; do
      if [ "$c" = "bcastS901" ] && [ "$o" != '{}' ]; then continue; fi
      echo "== $tool $c $o" >> gpurun_out/r2i_sanitizer.txt
      timeout 600 $CS --tool $tool --error-exitcode 9 python tools/profile_one.py --case $c --iters 1 --opts "$o" >> gpurun_out/r2i_sanitizer.txt 2>&1
      echo "rc=$?" >> gpurun_out/r2i_sanitizer.txt
    done
  done
  echo "== $tool reduce_mma_small" >> gpurun_out/r2i_sanitizer.txt
  timeout 600 $CS --tool $tool --error-exitcode 9 python tools/profile_one.py --case reduce_mma_small --iters 1 >> gpurun_out/r2i_sanitizer.txt 2>&1
  echo "rc=$?" >> gpurun_out/r2i_sanitizer.txt
done
grep -E "^==|rc=|ERROR SUMMARY" gpurun_out/r2i_sanitizer.txt | head -60
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ll_tile -s 2 -c 1 -o gpurun_out/r2i_prof_bcast python tools/profile_one.py --case bcast908 --iters 4 > gpurun_out/r2i_prof_bcast.log 2>&1
tail -2 gpurun_out/r2i_prof_bcast.log
