mkdir -p gpurun_out/r20
timeout 1800 ncu --set full --import-source on --clock-control none --kernel-name regex:"k_eat_(activate|big)" --launch-skip 6 --launch-count 2 -o gpurun_out/r20/ncu_c4_r4 -f python tools/prof_query.py --config C4 --problem eat --k 1024 --reps 1 > gpurun_out/r20/ncu.log 2>&1; echo ncu=$?
tail -3 gpurun_out/r20/ncu.log
