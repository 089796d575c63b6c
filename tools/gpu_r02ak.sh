bash tools/gpu_variants.sh r02ak pubmed base w9r112 w10r96
