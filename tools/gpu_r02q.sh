timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r02q_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02q_pytest.log
LDA_TIMING=1 timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/r02q_bench.json 2> gpurun_out/r02q_bench.err
grep "\[lda\]" gpurun_out/r02q_bench.err | head -20; tail -3 gpurun_out/r02q_pytest.log
python -c "
import json
d=json.loads(open('gpurun_out/r02q_bench.json').read().strip().splitlines()[-1]); print(d['value']/1e9, d['e2e']['value']/1e9, d['e2e']['breakdown'], d['cpu_baseline'])"
