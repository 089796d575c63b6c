timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
LDA_TIMING=1 timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2" --set "sampler=0" 2>&1 | grep -v "^#"
