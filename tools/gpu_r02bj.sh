OUT=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/r02bj_pytest.log 2>&1; echo "pytest exit $?" >> $OUT/r02bj_pytest.log; tail -2 $OUT/r02bj_pytest.log
python -c "import __graft_entry__ as g; g.smoke()" > $OUT/r02bj_smoke.log 2>&1; tail -1 $OUT/r02bj_smoke.log
for c in pubmed nytimes nytimes_k128 nytimes_k8192 pubmed_x5; do
  timeout 900 python bench.py --config $c --steps 20 --warmup 3 > $OUT/bench_r02bj_$c.json 2> $OUT/bench_r02bj_$c.err
  python -c "
import json
d=json.loads(open('$OUT/bench_r02bj_$c.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$c', round(d['value']/1e9,3), round(d['ms_per_step'],2), round(r['frac'],3), round(r['sweep_frac'],3), round(d['e2e']['value']/1e9,3), d['e2e']['breakdown'], d['clocks']['reasons'])" 2>&1 | tail -1
done
