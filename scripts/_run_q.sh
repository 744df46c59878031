bash scripts/variants.sh cfg2 "X=0" "FMMFFT_S2T_TPC=2" "FMMFFT_S2T_TPC=2 FMMFFT_PDL=1" "FMMFFT_PDL=1"
bash scripts/variants.sh cfg3 "X=0" "FMMFFT_FS_NARROW=1"
