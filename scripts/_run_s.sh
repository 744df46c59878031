timeout 900 python -m pytest tests -m gpu -x -q -k "post_pfft or end_to_end or virtual or stages or inverse" 2>&1 | tail -4
bash scripts/variants.sh cfg2 "X=0" "FMMFFT_PP=tile"
bash scripts/variants.sh cfg4 "X=0"
