bash tools/gpu_variants.sh r02aq pubmed pe1 pe0 pe1 pe0
bash tools/gpu_variants.sh r02aq1 nytimes pe1 pe0
