bash tools/gpu_variants.sh r02an pubmed d4 d2 d4 d2
bash tools/gpu_variants.sh r02an1 nytimes d4 d2
