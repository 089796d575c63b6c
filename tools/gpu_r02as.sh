bash tools/gpu_variants.sh r02as pubmed ls1 ls0 ls1 ls0
bash tools/gpu_variants.sh r02as1 nytimes ls1 ls0
