# full GPU round: tests, bench, launch list + ncu full capture
TAG=${1:-r01c}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests_full.log 2>&1; tail -3 gpurun_out/gpu_tests_full.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -c 1500 gpurun_out/bench_$TAG.json; tail -3 gpurun_out/bench_$TAG.err
timeout 1200 bash tools/ncu_capture.sh $TAG pubmed
python tools/write_traffic.py gpurun_out/prof_${TAG}_pubmed.ncu-rep pubmed $TAG
