timeout 300 python tools/prof_query.py --config C2 --problem reach --k 64 --reps 4 > gpurun_out/reach_C2.log 2>&1
timeout 300 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 3 > gpurun_out/eat_C2.log 2>&1
timeout 300 python tools/prof_query.py --config C4 --problem reach --k 64 --reps 2 > gpurun_out/reach_C4.log 2>&1
timeout 300 python tools/prof_query.py --config C4 --problem eat --k 64 --reps 2 > gpurun_out/eat_C4.log 2>&1
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q -k "reach or exchange or stream" > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name regex:"k_reach_(scan|big)" --launch-skip 8 --launch-count 2 -o gpurun_out/ncu_reach_c2 -f python tools/prof_query.py --config C2 --problem reach --k 64 --reps 1 > gpurun_out/ncu_reach.log 2>&1
grep rep gpurun_out/reach_C2.log gpurun_out/reach_C4.log gpurun_out/eat_C2.log gpurun_out/eat_C4.log; tail -2 gpurun_out/pytest_gpu.log
