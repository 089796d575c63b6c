bash tools/gpu_variants.sh r02am pubmed d4 d2
bash tools/gpu_variants.sh r02am8 nytimes_k8192 d4 d2
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "k_variants or k8192 or exact_redraw or tiny or decomposition" > gpurun_out/r02am_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02am_pytest.log; tail -2 gpurun_out/r02am_pytest.log
