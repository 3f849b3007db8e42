mkdir -p gpurun_out/last2
timeout 2400 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --kernel-name regex:"k_eat_(activate|big|chain)" --csv --log-file gpurun_out/last2/relax_traffic_C4_job.csv python tools/prof_query.py --config C4 --problem eat --k 1024 --reps 1 > gpurun_out/last2/ncu.log 2>&1; echo ncu=$?
grep -c gpu__time gpurun_out/last2/relax_traffic_C4_job.csv
