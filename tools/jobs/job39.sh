cd $GRAFT_REPO_ROOT
for g in 0 2 4 8 16; do
  echo "== LL_GRID_PER_SM=$g"
  LL_GRID_PER_SM=$g timeout 300 python tools/sweep.py --only small 2>&1 | grep case
done
