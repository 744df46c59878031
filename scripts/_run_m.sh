timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.log; tail -5 gpurun_out/pytest_gpu.log
bash scripts/variants.sh cfg3 "X=0" "FMMFFT_FS_MAXBITS=10" "FMMFFT_FS_MAXBITS=9" "FMMFFT_PP_MS=32"
timeout 300 python bench.py --workload cfg2 --steps 50 --warmup 5 --no-cpu-baseline > gpurun_out/bench_cfg2.json 2> gpurun_out/bench_cfg2.err; python -c "
import json
d=json.loads(open('gpurun_out/bench_cfg2.json').read().strip().splitlines()[-1])
print(round(d['value'],1), d['roofline']['kernel'], round(d['roofline']['frac'],3), d['comparator'])"
python -c "
from paper_conf_sc_cecka17_b200 import autotune
for N in (1<<20, 1<<24, 1<<26):
    print(N, autotune(N, 1, 'c64', 1e-5, True), autotune(N, 1, 'c64', 1e-5, False))
"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_cfg3.csv python bench.py --workload cfg3 --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
python scripts/summarize_launches.py gpurun_out/launches_cfg3.csv
