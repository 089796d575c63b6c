timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "wide or k_variants or edge" > gpurun_out/r02d_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02d_pytest.log
bash tools/gpu_variants.sh r02d pubmed w0h0 w2h0 w2h1 w0h1 w2h0r4
tail -3 gpurun_out/r02d_pytest.log
