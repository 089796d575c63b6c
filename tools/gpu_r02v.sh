timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "midsize or edge" > gpurun_out/r02v_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02v_pytest.log
timeout 900 python tools/exp_options.py --config pubmed --sweeps 10 --warmup 25 --set theta_fused=0 --set theta_fused=1 --set theta_fused=0 --set theta_fused=1 2>&1 | grep Gtok
timeout 900 python tools/exp_options.py --config nytimes --sweeps 10 --warmup 25 --set theta_fused=0 --set theta_fused=1 2>&1 | grep Gtok
tail -2 gpurun_out/r02v_pytest.log
