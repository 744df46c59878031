timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_s2m|k_post_pfft|k_fft_col|k_fft_rowt" --launch-skip 8 -c 4 -o /tmp/c2 python bench.py --workload cfg2 --steps 1 --warmup 3 --no-cpu-baseline --no-extras > /dev/null 2>&1
ncu -i /tmp/c2.ncu-rep --page source --csv --print-source sass > gpurun_out/c2_src.csv 2>&1
ncu -i /tmp/c2.ncu-rep --page raw --csv > gpurun_out/c2_raw.csv 2>&1
ls -la gpurun_out/c2_*
