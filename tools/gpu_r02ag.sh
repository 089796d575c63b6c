bash tools/gpu_variants.sh r02ag pubmed base tring4
bash tools/gpu_variants.sh r02ag8 nytimes_k8192 base tring4
