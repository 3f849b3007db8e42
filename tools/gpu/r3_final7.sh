mkdir -p gpurun_out/final7
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/final7/smoke.log 2>&1; echo smoke=$?
timeout 3000 python -m pytest tests -m gpu -x -q > gpurun_out/final7/pytest_gpu.log 2>&1; echo pytest=$?
tail -1 gpurun_out/final7/pytest_gpu.log
timeout 2400 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --kernel-name regex:"k_eat_(activate|big|chain)" --csv --log-file gpurun_out/final7/relax_traffic_C4_job.csv python tools/prof_query.py --config C4 --problem eat --k 1024 --reps 1 > gpurun_out/final7/ncu.log 2>&1; echo ncu=$?
grep -c gpu__time gpurun_out/final7/relax_traffic_C4_job.csv
