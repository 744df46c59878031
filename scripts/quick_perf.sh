# Quick iteration loop under gpurun: a parity subset, the bench lines of the given workloads
# (no comparators), and their ncu launch lists.  usage: bash scripts/quick_perf.sh TAG "pytest -k expr" wl...
tag=$1; kexpr=$2; shift 2
mkdir -p gpurun_out/q
if [ -n "$kexpr" ]; then timeout 900 python -m pytest tests -m gpu -x -q -k "$kexpr" > gpurun_out/q/${tag}_tests.log 2>&1; echo "rc=$?" >> gpurun_out/q/${tag}_tests.log; fi
for w in "$@"; do
  timeout 300 python bench.py --workload $w --steps 20 --warmup 5 --no-extras --no-cpu-baseline > gpurun_out/q/${tag}_bench_$w.json 2> gpurun_out/q/${tag}_bench_$w.err
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file /tmp/l_$w.csv \
      python bench.py --workload $w --steps 2 --warmup 3 --no-cpu-baseline --no-extras > /dev/null 2>&1
  python scripts/summarize_launches.py /tmp/l_$w.csv > gpurun_out/q/${tag}_launches_$w.txt
done
