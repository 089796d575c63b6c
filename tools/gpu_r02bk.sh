OUT=gpurun_out
bash tools/ncu_configs.sh r02bk pubmed pubmed_x5 > $OUT/r02bk_ncu.log 2>&1
cp profiles/traffic.json $OUT/traffic_r02bk.json
python tools/profile_md.py $OUT/prof_r02bk_pubmed.ncu-rep sweep_tile "sampling kernel, pubmed, r02bk (final code)" > $OUT/r02bk_pubmed_profile.md 2>&1
python tools/profile_md.py $OUT/prof_r02bk_pubmed_x5.ncu-rep sweep_tile "sampling kernel, pubmed_x5, r02bk (final code)" > $OUT/r02bk_pubmed_x5_profile.md 2>&1
head -28 $OUT/r02bk_pubmed_profile.md | tail -20
