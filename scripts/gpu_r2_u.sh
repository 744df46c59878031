mkdir -p gpurun_out/u
bash scripts/variants_r2.sh w "bw12 bw16" cfg3 cfg3v8 cfg2
bash scripts/variants_r2.sh w2 "bw12 bw16" cfg3
timeout 900 python -m pytest tests -m gpu -x -q -k "end_to_end or stages or alternative or cfg3_full or virtual or smoke" > gpurun_out/u/tests_bw8_default.log 2>&1; echo "rc=$?" >> gpurun_out/u/tests_bw8_default.log
