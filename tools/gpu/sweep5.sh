python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for ex in 1 2 3; do
TG_TRACE=1 timeout 300 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 2 --relabel 0 --stats 1 --sweep-part 16777216 --exp $ex 2>&1 | grep -v Warn | grep sweep
done
