timeout 300 python tools/exp_options.py --sweeps 5 --set "sampler=2,theta_mode=1" --set "sampler=2,theta_mode=0" 2>&1 | grep -v "^#"
