# round 2: reach tests, engine diag counters (pairs per union edge), ncu on the relax kernels
set -x
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q -k "reach or exchange" > gpurun_out/pytest_reach.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_reach.log
for c in C2 C4; do
  TG_TRACE=1 timeout 600 python tools/prof_query.py --config $c --problem eat --k 64 --reps 1 --stats 1 --relabel 0 > gpurun_out/trace_$c.log 2>&1
done
timeout 600 python tools/prof_query.py --config C2 --problem reach --k 64 --reps 3 > gpurun_out/reach_C2.log 2>&1
timeout 600 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 3 > gpurun_out/eat_C2.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name regex:"k_eat_(activate|big)" --launch-skip 6 --launch-count 2 -o gpurun_out/ncu_c2_r4 -f python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 --relabel 0 > gpurun_out/ncu_c2.log 2>&1
echo done
