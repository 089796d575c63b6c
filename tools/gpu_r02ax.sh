bash tools/gpu_variants.sh r02ax pubmed le1 le0 le1 le0
bash tools/gpu_variants.sh r02ax1 nytimes le1 le0
bash tools/gpu_variants.sh r02ax8 nytimes_k8192 le1 le0
