timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "k_variants or edge or tile_sampler or appendix or tiny_config_lockstep or k8192 or exact_redraw" 2>&1 | tail -2
timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#"
