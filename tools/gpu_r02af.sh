OUT=gpurun_out; mkdir -p $OUT
ncu --set full --clock-control none --import-source on -k 'regex:^(sweep_tile_kernel)' -s 22 -c 1 -o $OUT/prof_r02af_pubmed -f \
    python bench.py --config pubmed --steps 20 --warmup 3 --no-cpu-baseline > $OUT/prof_r02af_pubmed.log 2>&1
python tools/profile_md.py $OUT/prof_r02af_pubmed.ncu-rep sweep_tile "sampling kernel, pubmed, r02af (FFMA2 walk)" > $OUT/r02af_pubmed_profile.md 2>&1
head -60 $OUT/r02af_pubmed_profile.md
