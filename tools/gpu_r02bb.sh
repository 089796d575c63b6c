OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "theta_in_sampler" > $OUT/r02bb_pytest.log 2>&1; echo "pytest exit $?" >> $OUT/r02bb_pytest.log; tail -3 $OUT/r02bb_pytest.log
timeout 900 python tools/exp_options.py --config pubmed --sweeps 10 --warmup 20 --set "" --set theta_in_sampler=1 --set "" --set theta_in_sampler=1 2>&1 | cut -c1-160
timeout 900 python tools/exp_options.py --config nytimes --sweeps 10 --warmup 20 --set "" --set theta_in_sampler=1 2>&1 | cut -c1-160
