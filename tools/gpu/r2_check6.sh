mkdir -p gpurun_out/r8
timeout 1200 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r8/pytest_gpu.log 2>&1; echo pytest=$?
tail -2 gpurun_out/r8/pytest_gpu.log
timeout 900 python bench.py --config C2 --problems sp,fp --k 32 --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/r8/bench_C2_spfp.json 2> gpurun_out/r8/bench_C2_spfp.err; echo spfp=$?
timeout 900 python bench.py --config C2 --problems sp,fp --k 128 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/r8/bench_C2_spfp128.json 2> gpurun_out/r8/bench_C2_spfp128.err; echo spfp128=$?
timeout 600 python bench.py --config C3 --steps 10 --warmup 3 > gpurun_out/r8/bench_C3.json 2> gpurun_out/r8/bench_C3.err; echo c3=$?
python - <<'PY'
import json
for f in ['bench_C2_spfp','bench_C2_spfp128','bench_C3']:
    try:
        d=json.load(open(f'gpurun_out/r8/{f}.json')); r=d['roofline']
        print(f, round(d['value'],1), round(d['ms_per_step'],2), d['rounds'], round(r['frac'],4), r['kernels_ms_per_step'])
    except Exception as e: print(f, 'ERR', e)
PY
