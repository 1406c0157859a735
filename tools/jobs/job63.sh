cd $GRAFT_REPO_ROOT
nproc > gpurun_out/nproc63.txt
timeout 600 python tools/oracle_rates.py > gpurun_out/oracle_rates63.jsonl 2>&1; cat gpurun_out/oracle_rates63.jsonl
for c in r2_2_0 r2_4_2; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 1 -c 1 -o gpurun_out/prof63_$c python tools/profile_one.py --case $c --iters 2 > gpurun_out/prof63_$c.log 2>&1
  tail -1 gpurun_out/prof63_$c.log
done
