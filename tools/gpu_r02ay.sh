OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -p no:cacheprovider > $OUT/r02ay_pytest.log 2>&1; tail -1 $OUT/r02ay_pytest.log
free -g | head -2
for i in 1 2; do
LDA_TIMING=1 timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $OUT/r02ay_bench$i.json 2> $OUT/r02ay_bench$i.err
grep "\[lda\]" $OUT/r02ay_bench$i.err | grep -v "layout:" | head -14
python -c "
import json
d=json.loads(open('$OUT/r02ay_bench$i.json').read().strip().splitlines()[-1]); print(d['e2e']['breakdown'])"
done
