cd $GRAFT_REPO_ROOT
timeout 300 ncu --metrics dram__bytes.min.per_second,dram__bytes.max.per_second,dram__bytes.sum.per_second,dram__cycles_active.min.pct_of_peak_sustained_elapsed,dram__cycles_active.max.pct_of_peak_sustained_elapsed,gpu__time_duration.sum --clock-control none -c 3 python -c "
import torch
a=torch.empty(1<<30,dtype=torch.int16,device='cuda'); b=torch.empty_like(a)
for _ in range(3): torch.bitwise_not(a, out=b)
torch.cuda.synchronize()
" > gpurun_out/r2p_ncu_copy.txt 2>&1
cat gpurun_out/r2p_ncu_copy.txt | grep -E "dram|gpu__time|copy|Kernel|elementwise" | head -30
