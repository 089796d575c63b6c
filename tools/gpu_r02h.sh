timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -m gpu -q -x -p no:cacheprovider > gpurun_out/r02h_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02h_pytest.log
bash tools/gpu_variants.sh r02h nytimes_k8192 prmt redraw
bash tools/gpu_variants.sh r02h2 pubmed redraw
tail -3 gpurun_out/r02h_pytest.log
