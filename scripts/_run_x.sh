bash scripts/variants.sh cfg2 "X=0" "FMMFFT_PDL=1" "X=0" "FMMFFT_PDL=1"
bash scripts/variants.sh cfg3 "X=0" "FMMFFT_PDL=1"
