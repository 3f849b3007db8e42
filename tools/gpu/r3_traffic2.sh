mkdir -p gpurun_out/r3w
timeout 1500 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r3w/pytest_gpu.log 2>&1; echo pytest=$?; tail -1 gpurun_out/r3w/pytest_gpu.log
timeout 2400 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --kernel-name regex:"k_eat_(activate|big|chain)" --csv --log-file gpurun_out/r3w/relax_traffic_C4_job.csv python tools/prof_query.py --config C4 --problem eat --k 1024 --reps 1 > gpurun_out/r3w/ncu.log 2>&1; echo ncu=$?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --kernel-name regex:"k_eat_(activate|big|chain)" --csv --log-file gpurun_out/r3w/relax_traffic_C2.csv python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 > gpurun_out/r3w/ncu2.log 2>&1; echo ncu2=$?
tail -2 gpurun_out/r3w/ncu.log; grep -c gpu__time gpurun_out/r3w/relax_traffic_C4_job.csv
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r3w/launches_bench_C4.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/r3w/ncu_launches.log 2>&1; echo ncu3=$?
