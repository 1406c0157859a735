cd $GRAFT_REPO_ROOT
for c in c2 c3 c3b c5T; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 2 -c 1 -o gpurun_out/prof54_$c python tools/profile_one.py --case $c > gpurun_out/ncu54_$c.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 80 --csv --log-file gpurun_out/launches54_bench.csv python bench.py --steps 5 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-configs > /dev/null 2>&1
ls -la gpurun_out/ | grep 54
