timeout 1500 python -m pytest tests -m gpu -x -q -rs > gpurun_out/gpu_tests_r2e.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests_r2e.log
bash scripts/variants_r2.sh e "ppr2 nf" cfg3 cfg3v8 cfg2
