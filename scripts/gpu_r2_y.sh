mkdir -p gpurun_out/y
FMMFFT_LIB=$PWD/paper_conf_sc_cecka17_b200/libfmmfft_ew8.so timeout 600 python -m pytest tests -m gpu -x -q -k "end_to_end or stages or alternative or cfg3_full" > gpurun_out/y/tests_ew8.log 2>&1; echo "rc=$?" >> gpurun_out/y/tests_ew8.log
bash scripts/variants_r2.sh y "ew8" cfg3 cfg2 cfg3v8
bash scripts/variants_r2.sh y2 "ew8" cfg3
