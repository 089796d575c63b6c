OUT=gpurun_out; mkdir -p $OUT
LDA_TIMING=1 python tools/load_only.py --config pubmed --reps 3 --pinned > $OUT/r02ac_load_pinned.log 2>&1
grep -E "sorter|copiers|load [0-9]|layout done|init" $OUT/r02ac_load_pinned.log
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/r02ac_pytest.log 2>&1; echo "pytest exit $?" >> $OUT/r02ac_pytest.log
tail -3 $OUT/r02ac_pytest.log
for i in 1 2; do
timeout 900 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > $OUT/r02ac_bench$i.json 2> $OUT/r02ac_bench$i.err
python -c "
import json
d=json.loads(open('$OUT/r02ac_bench$i.json').read().strip().splitlines()[-1]); print(d['value']/1e9, d['roofline']['frac'], d['e2e']['value']/1e9, d['e2e']['breakdown'])"
done
