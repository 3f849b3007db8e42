mkdir -p gpurun_out/r3a
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r3a/smoke.log 2>&1; echo smoke=$?
timeout 600 python tools/prof_query.py --config C4 --problem eat --k 64 --reps 3 --stats 1 > gpurun_out/r3a/stats_c4.log 2>&1; echo stats=$?
timeout 600 python tools/prof_query.py --config C4 --problem eat --k 64 --reps 3 > gpurun_out/r3a/time_c4.log 2>&1; echo time=$?
timeout 1800 ncu --set full --import-source on --clock-control none --kernel-name regex:"k_eat_(activate|big)" --launch-skip 8 --launch-count 4 -o gpurun_out/r3a/ncu_c4 -f python tools/prof_query.py --config C4 --problem eat --k 64 --reps 1 > gpurun_out/r3a/ncu.log 2>&1; echo ncu=$?
tail -3 gpurun_out/r3a/ncu.log; cat gpurun_out/r3a/stats_c4.log gpurun_out/r3a/time_c4.log
