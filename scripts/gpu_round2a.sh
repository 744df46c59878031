nproc > gpurun_out/host.txt; free -g >> gpurun_out/host.txt; nvidia-smi -L >> gpurun_out/host.txt
timeout 1500 python -m pytest tests -m gpu -x -q -rs > gpurun_out/gpu_tests_r2a.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests_r2a.log
timeout 300 python __graft_entry__.py > gpurun_out/smoke_r2a.log 2>&1; echo "rc=$?" >> gpurun_out/smoke_r2a.log
