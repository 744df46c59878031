timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_fft_pass|k_m2l_lvl|k_s2t_tc|k_post_pfft|k_s2m|k_up" -c 8 -o gpurun_out/cfg3_full python bench.py --workload cfg3 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_cfg3_full.log 2>&1
tail -3 gpurun_out/ncu_cfg3_full.log
