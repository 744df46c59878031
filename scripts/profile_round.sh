# One GPU call that regenerates this round's evidence under gpurun_out/prof/ (copied to profiles/ by hand):
# bench lines (cfg2 = the N=1 headline, cfg3 at G=1), ncu launch lists of the same commands,
# and one `ncu --set full` capture per workload (one launch of every kernel) summarised with
# scripts/ncu_traffic.py (duration, DRAM bytes, SM/issue/occupancy).  usage: bash scripts/profile_round.sh TAG
tag=${1:-r01}
mkdir -p gpurun_out/prof
timeout 600 python bench.py > gpurun_out/prof/${tag}_bench_cfg2.json 2> gpurun_out/prof/${tag}_bench_cfg2.err
timeout 600 python bench.py --workload cfg3 --steps 50 --warmup 5 > gpurun_out/prof/${tag}_bench_cfg3.json 2> gpurun_out/prof/${tag}_bench_cfg3.err
for w in cfg2 cfg3; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/prof/launches_$w.csv \
      python bench.py --workload $w --steps 2 --warmup 3 --no-cpu-baseline --no-extras > /dev/null 2>&1
  python scripts/summarize_launches.py gpurun_out/prof/launches_$w.csv > gpurun_out/prof/${tag}_launches_$w.txt
  # skip the 3 warm-up executes' launches: capture the kernels of one execute of the timed plan
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_" --launch-skip 60 -c 40 \
      -o /tmp/full_$w python bench.py --workload $w --steps 1 --warmup 3 --no-cpu-baseline --no-extras > /dev/null 2>&1
  python scripts/ncu_traffic.py /tmp/full_$w.ncu-rep ${w}_G1 gpurun_out/prof/${tag}_ncu_full_$w.txt > /dev/null
  ncu -i /tmp/full_$w.ncu-rep --page details --csv > gpurun_out/prof/${tag}_ncu_details_$w.csv 2>/dev/null
done
cp profiles/ncu_traffic.json gpurun_out/prof/ncu_traffic.json
rm -f gpurun_out/prof/launches_*.csv
ls -la gpurun_out/prof
