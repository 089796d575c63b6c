# compute-sanitizer over tools/sanitize.py: memcheck, racecheck, synccheck (logs in gpurun_out/)
TAG=${1:-r02}
timeout 1500 compute-sanitizer --tool memcheck --print-limit 5 python tools/sanitize.py > gpurun_out/memcheck_${TAG}.log 2>&1; tail -3 gpurun_out/memcheck_${TAG}.log
timeout 1500 compute-sanitizer --tool racecheck --racecheck-report analysis --print-limit 5 python tools/sanitize.py > gpurun_out/racecheck_${TAG}.log 2>&1; tail -6 gpurun_out/racecheck_${TAG}.log
timeout 1500 compute-sanitizer --tool synccheck --print-limit 5 python tools/sanitize.py > gpurun_out/synccheck_${TAG}.log 2>&1; tail -3 gpurun_out/synccheck_${TAG}.log
