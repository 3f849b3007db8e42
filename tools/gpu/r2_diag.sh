mkdir -p gpurun_out/r16
TG_TRACE=1 timeout 900 python tools/prof_query.py --config C4 --problem eat --k 1024 --reps 1 --stats 1 > gpurun_out/r16/trace_C4_1024.log 2>&1
grep "diag" gpurun_out/r16/trace_C4_1024.log | head -20; grep rep gpurun_out/r16/trace_C4_1024.log
