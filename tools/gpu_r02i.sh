bash tools/gpu_variants.sh r02i nytimes_k8192 ctapf0 ctapf1
