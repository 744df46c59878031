for w in cfg2 cfg3; do
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/launches_$w.csv python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_$w.log 2>&1
python scripts/summarize_launches.py gpurun_out/launches_$w.csv > gpurun_out/launches_$w.txt 2>&1; cat gpurun_out/launches_$w.txt
done
