timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "radix" > gpurun_out/r02w_pytest0.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02w_pytest0.log
tail -3 gpurun_out/r02w_pytest0.log
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/r02w_pytest.log 2>&1; echo "pytest exit $?" >> gpurun_out/r02w_pytest.log
tail -3 gpurun_out/r02w_pytest.log
for i in 1 2; do
LDA_TIMING=1 timeout 900 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/r02w_bench$i.json 2> gpurun_out/r02w_bench$i.err
grep "\[lda\]" gpurun_out/r02w_bench$i.err | head -20
python -c "
import json
d=json.loads(open('gpurun_out/r02w_bench$i.json').read().strip().splitlines()[-1]); print(d['value']/1e9, d['e2e']['value']/1e9, d['e2e']['breakdown'])"
done
