mkdir -p gpurun_out/r3t
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r3t/smoke.log 2>&1; echo smoke=$?
timeout 1500 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r3t/pytest_gpu.log 2>&1; echo pytest=$?
tail -1 gpurun_out/r3t/pytest_gpu.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r3t/bench_C4.json 2> gpurun_out/r3t/bench_C4.err; echo c4=$?
for c in C1 C2 C3; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/r3t/bench_$c.json 2> gpurun_out/r3t/bench_$c.err; echo $c=$?
done
timeout 600 python bench.py --config C5 --partitions 2 --query-only --k 1 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r3t/bench_C5_single_source.json 2> gpurun_out/r3t/bench_C5.err; echo c5=$?
python - <<'PY'
import json, glob
for f in sorted(glob.glob('gpurun_out/r3t/bench_*.json')):
    try:
        d=json.load(open(f)); r=d.get('roofline') or {}
        print(f.split('/')[-1], round(d['value'],2), round(d['ms_per_step'],2), d.get('rounds'), r.get('frac') and round(r['frac'],4), r.get('relax_ms_per_step'), r.get('relax_share_of_step'), (d.get('e2e') or {}).get('value'), d.get('clocks'), d.get('gpu_launches'))
    except Exception as e: print(f, 'ERR', e)
PY
