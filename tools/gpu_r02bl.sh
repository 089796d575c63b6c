bash tools/gpu_variants.sh r02bl pubmed g16 g8 g16 g8
