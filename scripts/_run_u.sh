timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.log; tail -4 gpurun_out/pytest_gpu.log
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -o /tmp/btp scripts/micro/bench_tree_pc.cu && /tmp/btp 8 2 64
bash scripts/variants.sh cfg2 "X=0" "FMMFFT_PMAJ=0"
