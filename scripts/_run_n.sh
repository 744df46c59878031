timeout 1500 python scripts/check_configs.py 20 > gpurun_out/check_configs.log 2>&1; tail -15 gpurun_out/check_configs.log
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.log; tail -5 gpurun_out/pytest_gpu.log
bash scripts/variants.sh cfg3 "X=0" "FMMFFT_FS_MAXBITS=10"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_cfg3.csv python bench.py --workload cfg3 --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
python scripts/summarize_launches.py gpurun_out/launches_cfg3.csv
python -c "
from paper_conf_sc_cecka17_b200 import autotune
for N in (1<<20, 1<<24, 1<<26):
    print(N, autotune(N, 1, 'c64', 1e-5, True), autotune(N, 1, 'c64', 1e-5, False))
"
