timeout 600 python -m pytest tests -m "gpu and not slow" -x -q -k "reach or insert or stream" > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
timeout 300 python tools/prof_query.py --config C2 --problem reach --k 64 --reps 4 > gpurun_out/reach_C2.log 2>&1
timeout 300 python tools/prof_query.py --config C4 --problem reach --k 64 --reps 2 > gpurun_out/reach_C4.log 2>&1
grep rep gpurun_out/reach_C2.log gpurun_out/reach_C4.log; tail -2 gpurun_out/pytest_gpu.log
