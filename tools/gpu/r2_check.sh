# quick check: parity subset + timings of the EAT engine (C2, C4) and the bit-lane reach engine
set -x
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_gpu.log
timeout 600 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 4 > gpurun_out/eat_C2.log 2>&1
timeout 600 python tools/prof_query.py --config C2 --problem reach --k 64 --reps 4 > gpurun_out/reach_C2.log 2>&1
timeout 600 python tools/prof_query.py --config C4 --problem eat --k 64 --reps 3 > gpurun_out/eat_C4.log 2>&1
timeout 600 python tools/prof_query.py --config C4 --problem reach --k 64 --reps 2 > gpurun_out/reach_C4.log 2>&1
tail -3 gpurun_out/eat_C2.log gpurun_out/reach_C2.log gpurun_out/eat_C4.log gpurun_out/reach_C4.log
