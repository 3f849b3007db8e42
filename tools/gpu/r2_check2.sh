set -x
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 300 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 4 > gpurun_out/eat_C2.log 2>&1
timeout 300 python tools/prof_query.py --config C2 --problem reach --k 64 --reps 4 > gpurun_out/reach_C2.log 2>&1
timeout 300 python tools/prof_query.py --config C2 --problem reach --k 64 --reps 1 --stats 1 > gpurun_out/reach_C2_stats.log 2>&1
timeout 300 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 --stats 1 > gpurun_out/eat_C2_stats.log 2>&1
timeout 300 python tools/prof_query.py --config C1 --problem eat --k 1 --reps 5 > gpurun_out/eat_C1.log 2>&1
timeout 600 python tools/prof_query.py --config C4 --problem eat --k 64 --reps 3 > gpurun_out/eat_C4.log 2>&1
timeout 900 python tools/prof_query.py --config C5 --problem eat --k 1 --reps 4 > gpurun_out/eat_C5.log 2>&1
grep rep gpurun_out/*.log | tail -30
