timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_stream.py -m gpu -q -p no:cacheprovider > gpurun_out/r02e_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02e_pytest.log
LDA_LIBRARY=variants/liblda_stats.so timeout 300 python tools/tile_stats.py pubmed 25 > gpurun_out/r02e_stats.log 2>&1
LDA_LIBRARY=variants/liblda_stats.so timeout 300 python tools/tile_stats.py nytimes 25 >> gpurun_out/r02e_stats.log 2>&1
tail -3 gpurun_out/r02e_pytest.log; cat gpurun_out/r02e_stats.log | tail -4
