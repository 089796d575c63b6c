nproc > gpurun_out/r02k_nproc.txt
LDA_TIMING=1 timeout 600 python tools/exp_options.py --config pubmed --sweeps 1 --warmup 1 > gpurun_out/r02k_loadtiming.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/r02k_bench.json 2> gpurun_out/r02k_bench.err
timeout 900 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_stream.py -m gpu -q -x -p no:cacheprovider > gpurun_out/r02k_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02k_pytest.log
cat gpurun_out/r02k_nproc.txt; grep "\[lda\]" gpurun_out/r02k_loadtiming.log; tail -2 gpurun_out/r02k_pytest.log
