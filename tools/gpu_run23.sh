timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "k_variants or edge or tile_sampler or k8192 or exact_redraw" 2>&1 | tail -2
timeout 300 python tools/exp_options.py --config nytimes_k8192 --sweeps 5 2>&1 | grep -v "^#" | cut -c 1-200
timeout 300 python tools/exp_options.py --config nytimes --sweeps 5 --set "sampler=3" 2>&1 | grep -v "^#" | cut -c 1-200
timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=3" 2>&1 | grep -v "^#" | cut -c 1-200
