mkdir -p gpurun_out/r2b
# per-kernel DRAM traffic of one 64-source C4 sub-batch (every relax launch of the query)
timeout 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__warps_active.avg.pct_of_peak_sustained_active --clock-control none --kernel-name regex:"k_eat_(activate|big|chain)" --csv --log-file gpurun_out/r2b/relax_traffic_C4.csv python tools/prof_query.py --config C4 --problem eat --k 64 --reps 1 > gpurun_out/r2b/ncu_traffic_c4.log 2>&1; echo ncu1=$?
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --kernel-name regex:"k_eat_(activate|big|chain)" --csv --log-file gpurun_out/r2b/relax_traffic_C2.csv python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 > gpurun_out/r2b/ncu_traffic_c2.log 2>&1; echo ncu2=$?
# launch list of the bench command (our kernels), serialised cold-cache replay
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name regex:"^(k_|void .*k_)" -c 400 --csv --log-file gpurun_out/r2b/launches_bench_C4.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/r2b/ncu_launches.log 2>&1; echo ncu3=$?
for sb in 32 96 128; do timeout 300 python tools/variant_bench.py paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so C4 $sb --problems=eat --opt=mirror:0 --opt=sub_batch:$sb >> gpurun_out/r2b/subbatch.log 2>&1; done
timeout 600 python bench.py --config C5 --partitions 8 --query-only --k 1 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r2b/bench_C5_k1.json 2> gpurun_out/r2b/bench_C5_k1.err; echo c5=$?
timeout 600 python tools/dynamic_bench.py C2 100000 5 > gpurun_out/r2b/dynamic_C2.json 2> gpurun_out/r2b/dynamic_C2.err; echo dyn=$?
timeout 3000 python -m pytest tests/test_gpu_parity_fullsize.py -x -q > gpurun_out/r2b/pytest_fullsize.log 2>&1; echo full=$?
tail -3 gpurun_out/r2b/pytest_fullsize.log; grep median gpurun_out/r2b/subbatch.log; cat gpurun_out/r2b/dynamic_C2.json
