# f2 sparse word rows: parity at K = 8192, then NYTimes K = 8192 bench with the rows on / off
OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py tests/test_gpu_stream.py -m gpu -q -x -p no:cacheprovider -k "8192 or sparse" > $OUT/r02x_pytest.log 2>&1; echo "pytest exit $?" >> $OUT/r02x_pytest.log
tail -3 $OUT/r02x_pytest.log
for o in "sparse_words=0" "sparse_words=-1" "sparse_words=8192" "sparse_words=512"; do
  timeout 900 python bench.py --config nytimes_k8192 --steps 20 --warmup 3 --no-cpu-baseline --opt $o > $OUT/r02x_k8192_$o.json 2> $OUT/r02x_k8192_$o.err
  python -c "
import json
d=json.loads(open('$OUT/r02x_k8192_$o.json').read().strip().splitlines()[-1])
print('$o', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['phases_ms_per_step'].items()})" 2>&1 | tail -1
done
