cd $GRAFT_REPO_ROOT
# where do the 1-2 GiB smem / CTA kernels lose against the plain streaming ceiling?
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -o gpurun_out/smem_ctl tools/smem_counter_control.cu
for v in 8 16; do ./gpurun_out/smem_ctl 0 20 $v 1 1; done > gpurun_out/r2s3d_ctl.jsonl
timeout 600 python tools/sweep.py --only ceiling > gpurun_out/r2s3d_default.jsonl 2>&1
LL_PDL=0 timeout 600 python tools/sweep.py --only ceiling > gpurun_out/r2s3d_nopdl.jsonl 2>&1
LL_ST_HINT=wb timeout 600 python tools/sweep.py --only ceiling > gpurun_out/r2s3d_wb.jsonl 2>&1
LL_SWEEP_OPTS='{"thread_bytes": 128}' timeout 600 python tools/sweep.py --only ceiling > gpurun_out/r2s3d_tb128.jsonl 2>&1
LL_SWEEP_OPTS='{"thread_bytes": 64}' timeout 600 python tools/sweep.py --only ceiling > gpurun_out/r2s3d_tb64.jsonl 2>&1
for v in 8 16; do ./gpurun_out/smem_ctl 0 20 $v 1 1; done >> gpurun_out/r2s3d_ctl.jsonl
rm -f gpurun_out/smem_ctl
