mkdir -p gpurun_out/r3
timeout 1200 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r3/pytest_gpu.log 2>&1; echo pytest=$?
tail -2 gpurun_out/r3/pytest_gpu.log
timeout 900 python bench.py --config C2 --problems sp,fp --k 32 --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/r3/bench_C2_spfp.json 2> gpurun_out/r3/bench_C2_spfp.err; echo spfp=$?
timeout 600 python bench.py --config C2 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r3/bench_C2.json 2> gpurun_out/r3/bench_C2.err; echo c2=$?
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r3/bench_C4.json 2> gpurun_out/r3/bench_C4.err; echo c4=$?
python - <<'PY'
import json
for f in ['bench_C2_spfp','bench_C2','bench_C4']:
    try:
        d=json.load(open(f'gpurun_out/r3/{f}.json')); r=d['roofline']
        print(f, round(d['value'],1), round(d['ms_per_step'],2), d['rounds'], round(r['frac'],4), r.get('spfp_relax_and_wait_steps_per_step'), r['kernels_ms_per_step'])
    except Exception as e: print(f, 'ERR', e)
PY
