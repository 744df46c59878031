# Profile ONE kernel (regex) of one bench workload with --set full + source counters; export the
# summary, details and per-line source table (stall reasons) as text under gpurun_out/k/.
# usage: bash scripts/ncu_kernel.sh TAG WORKLOAD REGEX [SKIP]
tag=$1; w=$2; rx=$3; skip=${4:-3}
mkdir -p gpurun_out/k
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"$rx" --launch-skip $skip -c 1 \
    -o /tmp/k_$tag python bench.py --workload $w --steps 1 --warmup 3 --no-cpu-baseline --no-extras > /dev/null 2>&1
ncu -i /tmp/k_$tag.ncu-rep --page details --csv 2>/dev/null > gpurun_out/k/${tag}_details.csv
ncu -i /tmp/k_$tag.ncu-rep --page source --csv --print-source sass 2>/dev/null | gzip > gpurun_out/k/${tag}_source_sass.csv.gz
ncu -i /tmp/k_$tag.ncu-rep --page source --csv --print-source cuda 2>/dev/null | gzip > gpurun_out/k/${tag}_source.csv.gz
ls -la gpurun_out/k
