bash tools/gpu_variants.sh r02ap pubmed split nosplit split nosplit
bash tools/gpu_variants.sh r02ap1 nytimes split nosplit
bash tools/gpu_variants.sh r02ap8 nytimes_k8192 split nosplit
