timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "midsize or tiny or edge" > gpurun_out/r02o_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02o_pytest.log
LDA_TIMING=1 timeout 900 python tools/exp_options.py --config pubmed --sweeps 3 --warmup 1 --set "" --set "" > gpurun_out/r02o_load.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/r02o_bench.json 2> gpurun_out/r02o_bench.err
grep "\[lda\]\|Gtok" gpurun_out/r02o_load.log; tail -2 gpurun_out/r02o_pytest.log
python -c "
import json; d=json.loads(open('gpurun_out/r02o_bench.json').read().strip().splitlines()[-1]); print(d['value']/1e9, d['e2e'])"
