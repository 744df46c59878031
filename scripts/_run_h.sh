for w in cfg2 cfg3; do timeout 300 python bench.py --workload $w --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err; python -c "
import json
d=json.loads(open('gpurun_out/bench_$w.json').read().strip().splitlines()[-1])
print('$w', round(d['value'],1), round(d['ms_per_step']*1e3,2), {k: round(v*1e3,1) for k,v in d['stages_ms'].items()})"; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_tree_pc|k_s2m|k_post_pfft|k_fft_row|k_s2t_tc" --launch-skip 10 -c 5 -o /tmp/cfg2_full python bench.py --workload cfg2 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_cfg2_full.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:"k_post_pfft|k_s2m" --launch-skip 4 -c 2 -o /tmp/cfg3_pp python bench.py --workload cfg3 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_cfg3_pp.log 2>&1
for f in cfg2_full cfg3_pp; do
  ncu -i /tmp/$f.ncu-rep --page details --csv > gpurun_out/${f}_details.csv 2>&1
  ncu -i /tmp/$f.ncu-rep --page raw --csv > gpurun_out/${f}_raw.csv 2>&1
done
ncu -i /tmp/cfg2_full.ncu-rep --page source --csv --print-source sass > gpurun_out/cfg2_full_src.csv 2>&1
