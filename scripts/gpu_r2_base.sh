# round-2 re-entry baseline: the GPU test suite, the default bench line and cfg3/cfg4 launch lists
mkdir -p gpurun_out/b
timeout 1500 python -m pytest tests -m gpu -x -q -rs > gpurun_out/b/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/b/gpu_tests.log
timeout 600 python bench.py > gpurun_out/b/bench_default.json 2> gpurun_out/b/bench_default.err
bash scripts/quick_perf.sh base "" cfg3 cfg4
cp -r gpurun_out/q/base_* gpurun_out/b/ 2>/dev/null
