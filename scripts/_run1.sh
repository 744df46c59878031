set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
timeout 300 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -c 3000 gpurun_out/bench.json
timeout 300 python scripts/cufft_baseline.py > gpurun_out/cufft.jsonl 2>&1; cat gpurun_out/cufft.jsonl
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_tree_pq -c 1 -o gpurun_out/tree_full python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_tree.log 2>&1; tail -3 gpurun_out/ncu_tree.log
