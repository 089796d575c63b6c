timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
LDA_TIMING=1 timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" 2>&1 | grep -v "^#" | cut -c 1-200
timeout 300 python tools/exp_options.py --config nytimes_k8192 --sweeps 5 2>&1 | grep -v "^#" | cut -c 1-200
