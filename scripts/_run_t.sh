nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include -o /tmp/btp scripts/micro/bench_tree_pc.cu && /tmp/btp 8 2 64 && /tmp/btp 7 2 128
