timeout 1500 python -m pytest tests -m gpu -x -q -rs > gpurun_out/gpu_tests_r2b.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests_r2b.log
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_r2b.json 2> gpurun_out/bench_r2b.err; echo "rc=$?" >> gpurun_out/bench_r2b.err
timeout 300 python scripts/diag/err_vs_n.py 20 26 > gpurun_out/err_vs_n_b.log 2>&1
