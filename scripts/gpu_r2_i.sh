mkdir -p gpurun_out/i
timeout 1200 python -m pytest tests -m gpu -x -q -k "end_to_end or stages or alternative or cfg3_full or virtual or smoke or real" > gpurun_out/i/tests.log 2>&1; echo "rc=$?" >> gpurun_out/i/tests.log
bash scripts/quick_perf.sh i "" cfg3 cfg2 cfg3v8
cp gpurun_out/q/i_* gpurun_out/i/
timeout 300 python scripts/timeline.py --workload cfg3 --out gpurun_out/i/timeline > gpurun_out/i/timeline.log 2>&1
