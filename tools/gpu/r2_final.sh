# round 2 final: smoke, the whole -m gpu suite (incl. slow), bench lines of every config
mkdir -p gpurun_out/final2
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/final2/smi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/final2/smoke.log 2>&1; echo smoke=$?
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/final2/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/final2/pytest_gpu.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/final2/bench_C4.json 2> gpurun_out/final2/bench_C4.err; echo c4=$?
for c in C1 C2 C3; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/final2/bench_$c.json 2> gpurun_out/final2/bench_$c.err; echo $c=$?
done
timeout 600 python bench.py --config C5 --partitions 8 --query-only --k 1 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/final2/bench_C5_single_source.json 2> gpurun_out/final2/bench_C5.err; echo c5=$?
timeout 900 python bench.py --config C2 --problems sp,fp --k 32 --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/final2/bench_C2_spfp.json 2> gpurun_out/final2/bench_C2_spfp.err; echo spfp=$?
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/final2/bench_ref_C4.json 2> gpurun_out/final2/bench_ref_C4.err; echo ref=$?
python - <<'PY'
import json, glob
for f in sorted(glob.glob('gpurun_out/final2/bench_*.json')):
    try:
        d=json.load(open(f)); r=d.get('roofline') or {}
        print(f.split('/')[-1], round(d['value'],2), round(d['ms_per_step'],2), d.get('rounds'), r.get('frac') and round(r['frac'],4), (d.get('e2e') or {}).get('value'), d.get('clocks'))
    except Exception as e: print(f, 'ERR', e)
PY
