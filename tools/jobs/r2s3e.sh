cd $GRAFT_REPO_ROOT
# NOOP streaming copy kernel (parity + timing), small-CTA tile / thread sweeps
timeout 600 python -m pytest tests -m gpu -q -k "noop" > gpurun_out/r2s3e_pytest_noop.txt 2>&1
tail -2 gpurun_out/r2s3e_pytest_noop.txt
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o gpurun_out/smem_ctl tools/smem_counter_control.cu
./gpurun_out/smem_ctl 0 20 8 1 1 > gpurun_out/r2s3e_ctl.jsonl
timeout 600 python tools/sweep.py --only ceiling > gpurun_out/r2s3e_ceiling.jsonl 2>&1
timeout 900 python tools/sweep.py --only smallcta > gpurun_out/r2s3e_smallcta.jsonl 2>&1
./gpurun_out/smem_ctl 0 20 8 1 1 >> gpurun_out/r2s3e_ctl.jsonl
rm -f gpurun_out/smem_ctl
