cd $GRAFT_REPO_ROOT
timeout 900 python tools/sweep.py --only hints > gpurun_out/sweep5.txt 2>&1
timeout 300 python tools/bench_device.py --loopback 8 --n 15 > gpurun_out/bench_device_lb8.txt 2>&1
timeout 300 python tools/bench_device.py --n 15 > gpurun_out/bench_device_p1.txt 2>&1
