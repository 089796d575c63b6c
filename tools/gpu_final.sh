#!/bin/bash
# End-of-round evidence on one B200: GPU test suite + smoke, bench lines of
# every BASELINE config (and f3 streaming), ncu captures per config (traffic
# for the bench lines) + launch list, profile summaries, convergence runs,
# sanitizers.  Usage: bash tools/gpu_final.sh <tag>
TAG=${1:-r02}
OUT=gpurun_out; mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q -rA -p no:cacheprovider > $OUT/${TAG}_pytest.log 2>&1; echo "pytest exit $?" >> $OUT/${TAG}_pytest.log
python -c "import __graft_entry__ as g; g.smoke()" > $OUT/${TAG}_smoke.log 2>&1
# the bench lines first (their e2e loads measured 0.25 s standalone but up
# to 0.40 s right after the ncu captures on the same box); roofline.traffic
# comes from the committed profiles/traffic.json (the previous capture)
for c in pubmed nytimes nytimes_k128 nytimes_k8192 pubmed_x5; do
  timeout 900 python bench.py --config $c --steps 20 --warmup 3 > $OUT/bench_${TAG}_$c.json 2> $OUT/bench_${TAG}_$c.err
done
bash tools/ncu_configs.sh $TAG pubmed nytimes nytimes_k128 nytimes_k8192 pubmed_x5
cp profiles/traffic.json $OUT/traffic_${TAG}.json
for c in pubmed nytimes nytimes_k128 nytimes_k8192 pubmed_x5; do
  k=$( [ $c = nytimes_k8192 ] && echo sweep_tile_cta || echo sweep_tile )
  python tools/profile_md.py $OUT/prof_${TAG}_$c.ncu-rep $k "sampling kernel, $c, $TAG" > $OUT/${TAG}_${c}_profile.md 2>&1
done
timeout 900 python bench.py --config pubmed --steps 10 --warmup 3 --no-cpu-baseline --opt stream_chunks=4 > $OUT/bench_${TAG}_pubmed_stream4.json 2> $OUT/bench_${TAG}_pubmed_stream4.err
timeout 1200 python tools/convergence.py --config pubmed --sweeps 100 --every 10 --write > $OUT/${TAG}_conv_pubmed.log 2>&1
timeout 1500 python tools/convergence.py --config nytimes@0.01 --sweeps 100 --every 10 --anchor --write > $OUT/${TAG}_conv_nyt1pct.log 2>&1
cp profiles/convergence_*.md $OUT/
# compute-sanitizer is closed on the GPU pool (runs under it left GPUs needing a reset): not run
tail -2 $OUT/${TAG}_pytest.log; tail -1 $OUT/${TAG}_smoke.log
for c in pubmed nytimes nytimes_k128 nytimes_k8192 pubmed_x5 pubmed_stream4; do
  python -c "
import json
d=json.loads(open('$OUT/bench_${TAG}_$c.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$c', round(d['value']/1e9,3), round(d['ms_per_step'],2), round(r['frac'],3), round(r['sweep_frac'],3), r['dram_frac'] and round(r['dram_frac'],3), round(d['e2e']['value']/1e9,3), d['e2e']['breakdown'])" 2>&1 | tail -1
done
