bash tools/gpu_variants.sh r02aj pubmed base w9 w10
