mkdir -p gpurun_out/x
md5sum paper_conf_sc_cecka17_b200/libfmmfft*.so > gpurun_out/x/md5_before.txt
python -c "import sys; sys.path.insert(0,'paper_conf_sc_cecka17_b200'); import build as b; print('needs_build', b.needs_build())" > gpurun_out/x/nb.txt 2>&1
bash scripts/variants_r2.sh x "copy bw12" cfg3
md5sum paper_conf_sc_cecka17_b200/libfmmfft*.so > gpurun_out/x/md5_after.txt
