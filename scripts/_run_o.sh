timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.log; tail -5 gpurun_out/pytest_gpu.log
bash scripts/variants.sh cfg3 "X=0" "FMMFFT_PP=tile"
bash scripts/variants.sh cfg2 "X=0"
bash scripts/variants.sh cfg4 "X=0" "FMMFFT_FS_MAXBITS=9"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_cfg3.csv python bench.py --workload cfg3 --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
python scripts/summarize_launches.py gpurun_out/launches_cfg3.csv
