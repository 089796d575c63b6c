LDA_TIMING=1 timeout 900 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/r02p_bench.json 2> gpurun_out/r02p_bench.err
LDA_TIMING=1 timeout 900 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/r02p_bench2.json 2> gpurun_out/r02p_bench2.err
grep "\[lda\]" gpurun_out/r02p_bench.err | head -20
python -c "
import json
for f in ['gpurun_out/r02p_bench.json','gpurun_out/r02p_bench2.json']:
    d=json.loads(open(f).read().strip().splitlines()[-1]); print(d['value']/1e9, d['e2e']['value']/1e9, d['e2e']['breakdown'])"
