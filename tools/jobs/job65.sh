cd $GRAFT_REPO_ROOT
# compute-sanitizer on the pipelined linear-tile kernels (several tiles per CTA: LL_GRID_PER_SM=1)
for w in 2 4; do
  for o in '{}' '{"min_blocks": -1}' '{"pipe": "off", "min_blocks": 2}'; do
    for tool in racecheck memcheck synccheck; do
      echo "== w=$w opts=$o tool=$tool"
      LL_GRID_PER_SM=1 timeout 600 compute-sanitizer --tool $tool --error-exitcode 9 python tools/profile_one.py --case r2small_$w --iters 2 --opts "$o" 2>&1 | grep -E "ERROR SUMMARY|linear_tile|rror" | head -4
      echo "rc=${PIPESTATUS[0]}"
    done
  done
done > gpurun_out/sanitizer65.txt 2>&1
cat gpurun_out/sanitizer65.txt
