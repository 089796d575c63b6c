bash tools/gpu_variants.sh r02at pubmed su1 su0 su1 su0
bash tools/gpu_variants.sh r02at1 nytimes su1 su0
