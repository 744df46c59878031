timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.log; tail -5 gpurun_out/pytest_gpu.log
for w in cfg2 cfg3; do timeout 300 python bench.py --workload $w --steps 50 --warmup 5 --no-cpu-baseline > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err; python -c "
import json
d=json.loads(open('gpurun_out/bench_$w.json').read().strip().splitlines()[-1])
print('$w', round(d['value'],1), round(d['ms_per_step']*1e3,2), d.get('comparator'), {k: round(v*1e3,1) for k,v in d['stages_ms'].items()})"; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_cfg2.csv python bench.py --workload cfg2 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_cfg2.log 2>&1
python scripts/summarize_launches.py gpurun_out/launches_cfg2.csv
