timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_fft_col|k_fft_rowt|k_post_pfft|k_s2m|k_up|k_s2t_tc" --launch-skip 6 -c 6 -o /tmp/cfg3_full2 python bench.py --workload cfg3 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_cfg3_full2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_m2l_lvl" --launch-skip 21 -c 1 -o /tmp/cfg3_m2l python bench.py --workload cfg3 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_cfg3_m2l.log 2>&1
for f in cfg3_full2 cfg3_m2l; do
  ncu -i /tmp/$f.ncu-rep --page details --csv > gpurun_out/${f}_details.csv 2>&1
  ncu -i /tmp/$f.ncu-rep --page raw --csv > gpurun_out/${f}_raw.csv 2>&1
  ncu -i /tmp/$f.ncu-rep --page source --csv --print-source sass > gpurun_out/${f}_src.csv 2>&1
done
ls -la gpurun_out/
tail -n 2 gpurun_out/ncu_cfg3_full2.log
