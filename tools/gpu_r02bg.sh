OUT=gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py tests/test_gpu_stream.py -m gpu -q -x -p no:cacheprovider -k "8192 or sparse or exact_redraw or midsize" > $OUT/r02bg_pytest.log 2>&1; tail -2 $OUT/r02bg_pytest.log
for c in nytimes_k8192 nytimes pubmed; do
timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline > $OUT/r02bg_$c.json 2>/dev/null
python -c "
import json
d=json.loads(open('$OUT/r02bg_$c.json').read().strip().splitlines()[-1]); print('$c', d['value']/1e9, d['roofline']['frac'], d['config'].get('tiles'), d['e2e']['value']/1e9)"
done
