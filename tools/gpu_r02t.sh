bash tools/ncu_configs.sh r02t pubmed
python tools/profile_md.py gpurun_out/prof_r02t_pubmed.ncu-rep sweep_tile "sweep_tile_kernel, PubMed-shaped K=1024, r02t" > gpurun_out/r02t_pubmed_profile.md 2>&1
head -5 gpurun_out/r02t_pubmed_profile.md
