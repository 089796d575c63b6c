set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "k_variants or edge or tile_sampler or appendix or tiny_config_lockstep" > gpurun_out/gpu_tests2.log 2>&1; tail -15 gpurun_out/gpu_tests2.log
timeout 600 python tools/exp_options.py --sweeps 5 --set "sampler=2" --set "sampler=2,tile_tokens=8000000" --set "sampler=2,tile_tokens=32000000" --set "sampler=2,chunk_tokens=1024" --set "sampler=0" > gpurun_out/exp2.log 2>&1; cat gpurun_out/exp2.log
