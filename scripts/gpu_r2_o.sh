mkdir -p gpurun_out/o
timeout 900 python -m pytest tests -m gpu -x -q -k "end_to_end or post_pfft or cfg3_full or virtual or stages" > gpurun_out/o/tests.log 2>&1; echo "rc=$?" >> gpurun_out/o/tests.log
bash scripts/variants_r2.sh o "old ppp3" cfg3
bash scripts/variants_r2.sh o2 "old" cfg3
