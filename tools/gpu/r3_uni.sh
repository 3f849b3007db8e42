TG_TRACE=1 timeout 600 python tools/prof_query.py --config C4 --problem eat --k 64 --reps 1 --stats 1 2>&1 | grep diag
TG_TRACE=1 timeout 600 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 --stats 1 2>&1 | grep diag
