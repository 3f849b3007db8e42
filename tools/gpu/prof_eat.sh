python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
TG_TRACE=1 timeout 300 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 2 --stats 1 2>&1 | grep -v Warn | tail -32 > gpurun_out/trace_eat.log
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name regex:"k_eat_(activate|big)" --launch-skip 6 --launch-count 2 -o gpurun_out/eat_r4 -f python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 > gpurun_out/ncu_eat.log 2>&1
