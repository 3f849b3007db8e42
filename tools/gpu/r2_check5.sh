mkdir -p gpurun_out/r5
timeout 1200 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r5/pytest_gpu.log 2>&1; echo pytest=$?
tail -2 gpurun_out/r5/pytest_gpu.log
timeout 900 python tools/order_exp.py C4 1024 > gpurun_out/r5/order_exp.log 2>&1
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/r5/bench_C4.json 2> gpurun_out/r5/bench_C4.err; echo c4=$?
timeout 600 python bench.py --config C2 --steps 10 --warmup 3 > gpurun_out/r5/bench_C2.json 2> gpurun_out/r5/bench_C2.err; echo c2=$?
timeout 900 python bench.py --config C2 --problems sp,fp --k 32 --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/r5/bench_C2_spfp.json 2> gpurun_out/r5/bench_C2_spfp.err; echo spfp=$?
cat gpurun_out/r5/order_exp.log | grep order
python - <<'PY'
import json
for f in ['bench_C4','bench_C2','bench_C2_spfp']:
    try:
        d=json.load(open(f'gpurun_out/r5/{f}.json')); r=d['roofline']
        print(f, round(d['value'],1), round(d['ms_per_step'],2), d['rounds'], round(r['frac'],4), (d.get('e2e') or {}).get('value'), r['kernels_ms_per_step'])
    except Exception as e: print(f, 'ERR', e)
PY
