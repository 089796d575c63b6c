timeout 1500 compute-sanitizer --tool memcheck --print-limit 5 python tools/sanitize.py > gpurun_out/memcheck.log 2>&1; tail -4 gpurun_out/memcheck.log
timeout 1500 compute-sanitizer --tool racecheck --racecheck-report analysis --print-limit 5 python tools/sanitize.py > gpurun_out/racecheck.log 2>&1; tail -6 gpurun_out/racecheck.log
