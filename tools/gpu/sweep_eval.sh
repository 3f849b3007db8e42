python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
L=paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so
for p in 0 262144 1048576 4194304; do
timeout 300 python tools/variant_bench.py $L C2 64 --opt=sweep_struct:1 --opt=engine:2 --opt=sweep_part:$p 2>&1 | grep -v Warn | tail -2
done
timeout 300 python tools/variant_bench.py $L C2 64 --pred --opt=engine:1 2>&1 | grep -v Warn | tail -2
timeout 300 python tools/variant_bench.py $L C2 64 --pred --opt=sweep_struct:1 --opt=engine:2 2>&1 | grep -v Warn | tail -2
TG_TRACE=1 timeout 300 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 2 --relabel 0 --stats 1 --engine 2 2>&1 | grep -v Warn | tail -12
