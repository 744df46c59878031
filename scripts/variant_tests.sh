# run a pytest selection against a tuning build: bash scripts/variant_tests.sh NAME "expr"
FMMFFT_LIB=$PWD/paper_conf_sc_cecka17_b200/libfmmfft_$1.so timeout 900 python -m pytest tests -m gpu -x -q -k "$2" > gpurun_out/v/tests_$1.log 2>&1; echo "rc=$?" >> gpurun_out/v/tests_$1.log
