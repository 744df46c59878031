# round-2 closing evidence: the GPU suite, smoke, the default bench line, launch lists and ncu
# full captures of cfg3 / cfg3v8 / cfg2 / cfg4, and the CUPTI timelines (copied to profiles/)
mkdir -p gpurun_out/prof
timeout 1800 python -m pytest tests -m gpu -q -rs > gpurun_out/prof/r02_gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/prof/r02_gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/prof/r02_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/prof/r02_smoke.log
bash scripts/profile_r02.sh r02 cfg3 cfg3v8 cfg2 cfg4 > gpurun_out/prof/profile.log 2>&1
for w in cfg3 cfg3v8 cfg2; do timeout 300 python scripts/timeline.py --workload $w --out gpurun_out/prof/r02_timeline > /dev/null 2>&1; done
rm -f gpurun_out/prof/*.full.json
