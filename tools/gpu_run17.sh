timeout 600 python bench.py --no-cpu-baseline --steps 5 2>&1 | python -c "import sys,json; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d['value'], d['e2e'])"
timeout 600 ncu --set full --clock-control none --import-source on -k 'regex:sweep_tile_kernel' -s 3 -c 1 \
    -o gpurun_out/prof_tile7 -f python tools/exp_options.py --sweeps 1 --warmup 3 --set "sampler=2" > gpurun_out/prof_tile7.log 2>&1
tail -1 gpurun_out/prof_tile7.log
