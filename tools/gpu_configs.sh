mkdir -p gpurun_out
for c in nytimes nytimes_k128 nytimes_k8192; do
  timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_r01g_$c.json 2> gpurun_out/bench_r01g_$c.err
  tail -c 400 gpurun_out/bench_r01g_$c.json; echo
done
timeout 1200 python bench.py --config pubmed_x5 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_r01g_pubmed_x5.json 2> gpurun_out/bench_r01g_pubmed_x5.err
tail -c 600 gpurun_out/bench_r01g_pubmed_x5.json; tail -3 gpurun_out/bench_r01g_pubmed_x5.err
nvidia-smi --query-gpu=memory.used,memory.total --format=csv
