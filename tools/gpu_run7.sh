mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "k_variants or edge or tile_sampler or appendix or tiny_config_lockstep or k8192" > gpurun_out/gpu_tests9.log 2>&1; tail -2 gpurun_out/gpu_tests9.log
timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#"
for v in w6 tr3; do LDA_LIBRARY=$PWD/variants/$v.so timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#" | sed "s/^/$v /"; done
