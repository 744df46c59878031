timeout 1500 python -m pytest tests -m gpu -x -q -rs > gpurun_out/gpu_tests_r2c.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests_r2c.log
bash scripts/profile_r02.sh r02b
