timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "midsize or lockstep" > gpurun_out/r02m_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02m_pytest.log
LDA_TIMING=1 timeout 900 python tools/exp_options.py --config pubmed --sweeps 10 --warmup 25 --set zdoc=0 --set zdoc=1 --set zdoc=0 --set zdoc=1 > gpurun_out/r02m_zdoc.log 2>&1
grep -v "^\[lda\]   copier" gpurun_out/r02m_zdoc.log | grep "Gtok\|\[lda\]" | head -40; grep copier gpurun_out/r02m_zdoc.log; tail -2 gpurun_out/r02m_pytest.log
