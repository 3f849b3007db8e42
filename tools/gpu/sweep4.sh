python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for part in 1048576 16777216; do
TG_TRACE=1 timeout 300 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 2 --relabel 0 --stats 1 --sweep-part $part 2>&1 | grep -v Warn | grep sweep
done
TG_TRACE=1 timeout 300 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 2 --relabel 0 --stats 1 --sweep-part 16777216 --exp 1 2>&1 | grep -v Warn | grep sweep
