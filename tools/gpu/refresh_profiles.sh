# Round profile refresh: ncu relax traffic (EAT + LD batch), launch list of a bench
# step, one full capture of the round-4 activate/big kernels, then the bench lines.
set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
mkdir -p gpurun_out/prof
timeout 600 python bench.py > gpurun_out/prof/bench_C2.json 2> gpurun_out/prof/bench_C2.err
timeout 600 python bench.py --config C3 > gpurun_out/prof/bench_C3.json 2> gpurun_out/prof/bench_C3.err
O=gpurun_out/prof
mkdir -p $O
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum
timeout 600 ncu --metrics $M --clock-control none -k regex:"k_eat_(activate|big|chain)" --csv --log-file $O/relax_eat.csv python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 > /dev/null 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:"k_eat_(activate|big|chain)" --csv --log-file $O/relax_ld.csv python tools/prof_query.py --config C2 --problem ld --k 64 --reps 1 > /dev/null 2>&1
python tools/relax_traffic.py C2 $O/relax_eat.csv $O/relax_ld.csv $O
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_bench_step.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python tools/launches.py $O/launches_bench_step.csv 1000 > $O/launches_bench_step_summary.txt
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name regex:"k_eat_(activate|big)" --launch-skip 6 --launch-count 2 -o $O/eat_round4_activate_big_full -f python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 > /dev/null 2>&1
cp $O/relax_traffic_C2.json profiles/round1/relax_traffic_C2.json
