python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name regex:"k_eat_(activate|big)" --launch-skip 6 --launch-count 2 -o gpurun_out/eat_r4c -f python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 > gpurun_out/ncu_eat.log 2>&1
