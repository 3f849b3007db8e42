python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
L=paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so
for part in 65536 262144 1048576 4194304 16777216; do
timeout 300 python tools/variant_bench.py $L C2 64 --opt=sweep_part:$part --opt=exp:1 2>&1 | grep -v Warn
TG_TRACE=1 timeout 300 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 --relabel 0 --stats 1 --sweep-part $part 2>&1 | grep -v Warn | grep sweep
done
