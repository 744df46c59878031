timeout 1500 python -m pytest tests -m gpu -x -q -rs > gpurun_out/gpu_tests_r2d.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests_r2d.log
timeout 300 python __graft_entry__.py > gpurun_out/smoke_r2d.log 2>&1; echo "rc=$?" >> gpurun_out/smoke_r2d.log
bash scripts/profile_r02.sh r02c
timeout 600 python bench.py --workload cfg4 --steps 10 --warmup 3 --no-extras --no-cpu-baseline > gpurun_out/prof/r02c_bench_cfg4.json 2>/dev/null
timeout 600 python bench.py --workload cfg3v8 --steps 20 --warmup 5 --no-extras --no-cpu-baseline > gpurun_out/prof/r02c_bench_cfg3v8.json 2>/dev/null
