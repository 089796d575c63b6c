set -x
mkdir -p gpurun_out
python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; tail -5 gpurun_out/gpu_tests.log
python tools/exp_options.py --sweeps 5 --set "sampler=0" --set "sampler=1" --set "sampler=1,chunk_tokens=8192" > gpurun_out/exp.log 2>&1; cat gpurun_out/exp.log
python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -c 3000 gpurun_out/bench.json; tail -5 gpurun_out/bench.err
bash tools/ncu_capture.sh r01b pubmed
