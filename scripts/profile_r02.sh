# One GPU call that regenerates this round's evidence under gpurun_out/prof/ (copied to profiles/):
# the bench line (cfg3, the N = 1 headline, with cfg2 in configs_extra), ncu launch lists of
# cfg3 / cfg3v8 / cfg2, one `ncu --set full` (+ tensor / fma pipe metrics) capture per workload
# summarised with scripts/ncu_traffic.py, and the SASS evidence of the tcgen05 kernel.
# usage: bash scripts/profile_r02.sh TAG [workloads...]
tag=${1:-r02}; shift
wl=${@:-cfg3 cfg3v8 cfg2}
mkdir -p gpurun_out/prof
EXTRA=$(python -c "import sys; sys.path.insert(0,'scripts'); import ncu_traffic as n; print(n.EXTRA)")
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/prof/${tag}_bench_cfg3.json 2> gpurun_out/prof/${tag}_bench_cfg3.err
for w in $wl; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/prof/launches_$w.csv \
      python bench.py --workload $w --steps 2 --warmup 3 --no-cpu-baseline --no-extras > /dev/null 2>&1
  python scripts/summarize_launches.py gpurun_out/prof/launches_$w.csv > gpurun_out/prof/${tag}_launches_$w.txt
  n=$(python - "$w" <<'PY'
import csv, sys
rows = [r for r in csv.reader(open(f"gpurun_out/prof/launches_{sys.argv[1]}.csv")) if r]
print(sum(1 for r in rows if len(r) > 5 and "fmmfft::" in ",".join(r)))
PY
)
  per=$(( n / 15 ))  # --steps 2 --warmup 3: 5 executes each of the timed, profiled and e2e plans; capture the 3rd
  timeout 1200 ncu --set full --metrics $EXTRA --clock-control none --import-source on -k regex:"k_" --launch-skip $(( 2 * per )) -c $per \
      -o /tmp/full_$w python bench.py --workload $w --steps 1 --warmup 3 --no-cpu-baseline --no-extras > /dev/null 2>&1
  key=${w}_G1; [ "$w" = cfg3v8 ] && key=cfg3v8_G8
  python scripts/ncu_traffic.py /tmp/full_$w.ncu-rep $key gpurun_out/prof/${tag}_ncu_full_$w.txt > /dev/null
  ncu -i /tmp/full_$w.ncu-rep --page details --csv 2>/dev/null | gzip > gpurun_out/prof/${tag}_details_$w.csv.gz
done
python scripts/sass_evidence.py paper_conf_sc_cecka17_b200/libfmmfft.so > gpurun_out/prof/${tag}_sass_tcgen05.txt
cp profiles/ncu_traffic.json gpurun_out/prof/ncu_traffic.json
rm -f gpurun_out/prof/launches_*.csv
ls -la gpurun_out/prof
