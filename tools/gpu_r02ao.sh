bash tools/gpu_variants.sh r02ao pubmed lc1 lc0 lc1 lc0
bash tools/gpu_variants.sh r02ao1 nytimes lc1 lc0
bash tools/gpu_variants.sh r02ao8 nytimes_k8192 lc1 lc0
