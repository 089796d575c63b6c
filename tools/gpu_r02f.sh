timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "lockstep or redraw or decomposition or k8192" > gpurun_out/r02f_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02f_pytest.log
bash tools/gpu_variants.sh r02f pubmed w0h1 i2fp prmt
tail -3 gpurun_out/r02f_pytest.log
