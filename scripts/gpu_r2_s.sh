mkdir -p gpurun_out/s3
timeout 1200 python -m pytest tests -m gpu -x -q -k "end_to_end or stages or alternative or cfg3_full or cfg4_shape or virtual or s2t" > gpurun_out/s3/tests.log 2>&1; echo "rc=$?" >> gpurun_out/s3/tests.log
for i in 1 2; do
  timeout 300 python bench.py --workload cfg3 --steps 20 --warmup 5 --no-extras --no-cpu-baseline > gpurun_out/s3/sym_cfg3_$i.json 2>/dev/null
  FMMFFT_S2M_NOSYM=1 timeout 300 python bench.py --workload cfg3 --steps 20 --warmup 5 --no-extras --no-cpu-baseline > gpurun_out/s3/nosym_cfg3_$i.json 2>/dev/null
done
timeout 300 python bench.py --workload cfg4 --steps 5 --warmup 3 --no-extras --no-cpu-baseline > gpurun_out/s3/sym_cfg4.json 2>/dev/null
FMMFFT_S2M_OLD=1 timeout 300 python bench.py --workload cfg4 --steps 5 --warmup 3 --no-extras --no-cpu-baseline > gpurun_out/s3/old_cfg4.json 2>/dev/null
