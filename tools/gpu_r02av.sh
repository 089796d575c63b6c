bash tools/gpu_variants.sh r02av pubmed nc1 nc0 nc1 nc0
bash tools/gpu_variants.sh r02av1 nytimes nc1 nc0
