# Bench the tuning builds (FMMFFT_LIB) against the default library on the given workloads.
# usage: bash scripts/variants_r2.sh TAG "name1 name2 ..." wl...
tag=$1; names=$2; shift 2
mkdir -p gpurun_out/v
for n in base $names; do
  lib=""; [ "$n" != base ] && lib=$PWD/paper_conf_sc_cecka17_b200/libfmmfft_$n.so
  for w in "$@"; do
    FMMFFT_LIB=$lib timeout 300 python bench.py --workload $w --steps 20 --warmup 5 --no-extras --no-cpu-baseline \
        > gpurun_out/v/${tag}_${n}_$w.json 2> gpurun_out/v/${tag}_${n}_$w.err
  done
done
