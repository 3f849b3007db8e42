mkdir -p gpurun_out/r3v
timeout 3000 python -m pytest tests -m gpu -x -q > gpurun_out/r3v/pytest_gpu.log 2>&1; echo pytest=$?; tail -1 gpurun_out/r3v/pytest_gpu.log
timeout 2400 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --kernel-name regex:"k_eat_(activate|big|chain)" --csv --log-file gpurun_out/r3v/relax_traffic_C4_job.csv python tools/prof_query.py --config C4 --problem eat --k 1024 --reps 1 > gpurun_out/r3v/ncu.log 2>&1; echo ncu=$?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --kernel-name regex:"k_eat_(activate|big|chain)" --csv --log-file gpurun_out/r3v/relax_traffic_C2.csv python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 > gpurun_out/r3v/ncu2.log 2>&1; echo ncu2=$?
tail -2 gpurun_out/r3v/ncu.log; grep -c gpu__time gpurun_out/r3v/relax_traffic_C4_job.csv
