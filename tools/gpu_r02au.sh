bash tools/gpu_variants.sh r02au pubmed pf1 pf0 pf1 pf0
