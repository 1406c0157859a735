cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2l_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "scan" > gpurun_out/r2l_pytest.txt 2>&1
tail -3 gpurun_out/r2l_pytest.txt
timeout 600 python tools/sweep.py --only scan > gpurun_out/r2l_sweep_scan.jsonl 2>&1
cat gpurun_out/r2l_sweep_scan.jsonl
timeout 600 /usr/local/cuda/bin/compute-sanitizer --tool racecheck python -c "
import torch, paper_conf_asplos_0001cgrnls0trm26_b200 as ll
from workloads import configs as W
L=ll.Layout.from_spec(W.c4('reduce','mma',n_i=9,n_j=9)); p=ll.ll_plan_scan(L,1)
s=torch.rand(1<<L.d_in,device='cuda'); o=torch.empty_like(s); ll.ll_scan(s,o,p); torch.cuda.synchronize(); print(p.describe()['tma_store'])
" > gpurun_out/r2l_racecheck_scan.txt 2>&1
tail -3 gpurun_out/r2l_racecheck_scan.txt
