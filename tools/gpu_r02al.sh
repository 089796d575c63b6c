bash tools/gpu_variants.sh r02al pubmed d4 d2
bash tools/gpu_variants.sh r02al1 nytimes d4 d2
