bash tools/gpu_variants.sh r02ba8 nytimes_k8192 g4 g3 old g4 g3 old
