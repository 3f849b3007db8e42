python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for sb in 64 32 16; do
TG_TRACE=1 timeout 300 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1 --sub-batch $sb --relabel 0 --stats 1 2>&1 | grep -v Warn | tail -30
done
python - <<'PY'
import subprocess
PY
for sb in 64 32 16 8; do
timeout 300 python tools/prof_query.py --config C2 --problem eat --k 64 --reps 3 --sub-batch $sb --relabel 0 2>&1 | grep -v Warn | tail -1
done
