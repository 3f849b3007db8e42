mkdir -p gpurun_out/r3e
TG_TRACE=1 timeout 600 python tools/prof_query.py --config C4 --problem eat --k 64 --reps 1 --stats 1 > gpurun_out/r3e/c4_stats.log 2>&1; echo a=$?
TG_TRACE=1 timeout 600 python tools/prof_query.py --config C4 --problem eat --k 64 --reps 1 > gpurun_out/r3e/c4_trace.log 2>&1; echo b=$?
TG_TRACE=1 timeout 600 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 --stats 1 > gpurun_out/r3e/c2_stats.log 2>&1; echo c=$?
TG_TRACE=1 timeout 600 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 > gpurun_out/r3e/c2_trace.log 2>&1; echo d=$?
grep diag gpurun_out/r3e/*stats.log
