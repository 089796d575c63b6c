mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "k_variants or edge or tile_sampler or appendix or tiny_config_lockstep or k8192 or exact_redraw" > gpurun_out/gpu_tests11.log 2>&1; tail -2 gpurun_out/gpu_tests11.log
timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#"
for v in tr3; do LDA_LIBRARY=$PWD/variants/$v.so timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#" | sed "s/^/$v /"; done
