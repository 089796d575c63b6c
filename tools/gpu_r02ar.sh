bash tools/gpu_variants.sh r02ar pubmed bs1 bs0 bs1 bs0
bash tools/gpu_variants.sh r02ar1 nytimes bs1 bs0
