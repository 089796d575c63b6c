# full bench line (pubmed) + other configs + load phase timing
timeout 900 python bench.py --steps 20 --warmup 3 > gpurun_out/r02j_bench.json 2> gpurun_out/r02j_bench.err
bash tools/bench_configs.sh r02j
LDA_TIMING=1 timeout 600 python tools/exp_options.py --config pubmed --sweeps 1 --warmup 1 > gpurun_out/r02j_loadtiming.log 2>&1
tail -30 gpurun_out/r02j_loadtiming.log
