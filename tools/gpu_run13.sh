nproc; lscpu | grep "Model name"; free -g | head -2
LDA_TIMING=1 timeout 300 python tools/exp_options.py --sweeps 2 --set "sampler=2" 2>&1 | grep -v "^#"
