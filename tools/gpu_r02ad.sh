OUT=gpurun_out; mkdir -p $OUT
for i in 1 2 3; do
LDA_TIMING=1 timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > $OUT/r02ad_bench$i.json 2> $OUT/r02ad_bench$i.err
grep "\[lda\]" $OUT/r02ad_bench$i.err | grep -v "layout:" | head -14
python -c "
import json
d=json.loads(open('$OUT/r02ad_bench$i.json').read().strip().splitlines()[-1]); print(d['e2e']['breakdown'])"
done
