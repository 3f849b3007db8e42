mkdir -p gpurun_out/r13
TG_TRACE=1 timeout 300 python tools/prof_query.py --config C3 --problem fp --k 16 --reps 1 > gpurun_out/r13/trace_C3_fp.log 2>&1
TG_TRACE=1 timeout 300 python tools/prof_query.py --config C2 --problem sp --k 32 --reps 1 > gpurun_out/r13/trace_C2_sp.log 2>&1
timeout 300 python tools/prof_query.py --config C2 --problem sp --k 32 --reps 2 > gpurun_out/r13/C2_sp.log 2>&1
tail -30 gpurun_out/r13/trace_C3_fp.log; grep "round\|rep" gpurun_out/r13/trace_C2_sp.log | tail -30; cat gpurun_out/r13/C2_sp.log | tail -3
