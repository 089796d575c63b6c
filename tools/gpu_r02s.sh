for i in 1 2 3; do
LDA_TIMING=1 timeout 900 python bench.py --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/r02s_bench$i.json 2> gpurun_out/r02s_bench$i.err
grep "\[lda\]" gpurun_out/r02s_bench$i.err | head -20
python -c "
import json
d=json.loads(open('gpurun_out/r02s_bench$i.json').read().strip().splitlines()[-1]); print(d['value']/1e9, d['e2e']['value']/1e9, d['e2e']['breakdown'])"
done
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -p no:cacheprovider -k "tiny or invalid or midsize" 2>&1 | tail -2
