timeout 900 python -m pytest tests -m gpu -x -q -k "end_to_end or stages or alternative or virtual or full_size" 2>&1 | tail -4
bash scripts/variants.sh cfg2 "X=0"
bash scripts/variants.sh cfg3 "X=0"
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/bs scripts/micro/bench_s2t_tc.cu && /tmp/bs 65536 16 57 && /tmp/bs 256 64 1
