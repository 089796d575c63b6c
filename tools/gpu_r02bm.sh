bash tools/gpu_variants.sh r02bm pubmed rc4 rc8 rc6 rc4 rc8
