mkdir -p gpurun_out/prof
for w in cfg2 cfg3; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_" --launch-skip 60 -c 40 \
      -o /tmp/full_$w python bench.py --workload $w --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/prof/ncu_$w.log 2>&1
  python scripts/ncu_traffic.py /tmp/full_$w.ncu-rep ${w}_G1 gpurun_out/prof/r01_ncu_full_$w.txt > /dev/null
  ncu -i /tmp/full_$w.ncu-rep --page details --csv > gpurun_out/prof/r01_ncu_details_$w.csv 2>/dev/null
done
cp profiles/ncu_traffic.json gpurun_out/prof/ncu_traffic.json
tail -3 gpurun_out/prof/ncu_cfg2.log
