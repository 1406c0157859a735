cd $GRAFT_REPO_ROOT
for c in c3b_small c2fsmem_small c3f_small; do
  for tool in racecheck synccheck memcheck initcheck; do
    timeout 300 compute-sanitizer --tool $tool python tools/profile_one.py --case $c --iters 2 > gpurun_out/san47_${tool}_$c.txt 2>&1
    echo "$c $tool: $(grep -E 'SUMMARY|ERROR SUMMARY' gpurun_out/san47_${tool}_$c.txt | tail -1)"
  done
done
