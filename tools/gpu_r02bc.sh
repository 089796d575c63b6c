bash tools/gpu_variants.sh r02bc8 nytimes_k8192 nb4 nb3 nb2 nb4 nb3 nb2
