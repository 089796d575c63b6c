# bench lines of the other BASELINE configs (1 GPU): tools/bench_configs.sh <tag>
TAG=${1:-r01}
mkdir -p gpurun_out
for c in nytimes nytimes_k128 nytimes_k8192 pubmed_x5; do
  timeout 900 python bench.py --config $c --steps 20 --warmup 3 > gpurun_out/bench_${TAG}_$c.json 2> gpurun_out/bench_${TAG}_$c.err
  tail -c 300 gpurun_out/bench_${TAG}_$c.json
done
