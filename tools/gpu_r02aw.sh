bash tools/gpu_variants.sh r02aw pubmed bsc1 bsc0 bsc1 bsc0
bash tools/gpu_variants.sh r02aw1 nytimes bsc1 bsc0
