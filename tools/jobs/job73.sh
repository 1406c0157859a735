cd $GRAFT_REPO_ROOT
for nh in 0 1; do
  LL_NOHOIST=$nh timeout 900 python tools/sweep.py --only invec > gpurun_out/sweep_invec73_$nh.jsonl 2>> gpurun_out/sweep73.err
  LL_NOHOIST=$nh timeout 600 python -c "
import sys; sys.argv=['sweep.py']; sys.path.insert(0, 'tools')
import sweep; sweep.swizzle_case()" >> gpurun_out/sweep_invec73_$nh.jsonl 2>> gpurun_out/sweep73.err
done
tail -3 gpurun_out/sweep73.err
paste -d'\n' gpurun_out/sweep_invec73_0.jsonl gpurun_out/sweep_invec73_1.jsonl | cut -c1-200
