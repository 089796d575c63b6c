mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "convergence or tiny_config or nytimes_shaped or tile_sampler" > gpurun_out/gpu_tests12.log 2>&1; tail -2 gpurun_out/gpu_tests12.log
timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#"
timeout 600 python tools/convergence.py --config pubmed --sweeps 100 --every 10 --write > gpurun_out/conv_pubmed.log 2>&1; tail -3 gpurun_out/conv_pubmed.log
timeout 600 python tools/convergence.py --config nytimes --sweeps 100 --every 10 --write > gpurun_out/conv_nyt.log 2>&1; tail -2 gpurun_out/conv_nyt.log
mkdir -p gpurun_out/prof; cp profiles/convergence_*.md gpurun_out/prof/ 2>/dev/null
