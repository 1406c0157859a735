cd $GRAFT_REPO_ROOT
# final linear-tile defaults (unpipelined, 2 CTAs/SM, NOHOIST), several tiles per CTA
for c in r2mid_2 r2mid_4; do
  for tool in racecheck memcheck synccheck initcheck; do
    echo "== $c tool=$tool"
    LL_GRID_PER_SM=1 timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/profile_one.py --case $c --iters 1 2>&1 | grep -E "ERROR SUMMARY|RACECHECK SUMMARY|linear_tile|rror" | head -4
    echo "rc=${PIPESTATUS[0]}"
  done
done > gpurun_out/sanitizer75.txt 2>&1
cat gpurun_out/sanitizer75.txt
