mkdir -p gpurun_out/r12
timeout 1200 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r12/pytest_gpu.log 2>&1; echo pytest=$?
tail -15 gpurun_out/r12/pytest_gpu.log | grep -v "^$" | tail -8
timeout 900 python bench.py --config C2 --problems sp,fp --k 32 --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/r12/bench_C2_spfp.json 2> gpurun_out/r12/bench_C2_spfp.err; echo spfp=$?
timeout 600 python bench.py --config C3 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r12/bench_C3.json 2> gpurun_out/r12/bench_C3.err; echo c3=$?
timeout 600 python bench.py --config C1 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r12/bench_C1.json 2> gpurun_out/r12/bench_C1.err; echo c1=$?
python - <<'PY'
import json
for f in ['bench_C2_spfp','bench_C3','bench_C1']:
    try:
        d=json.load(open(f'gpurun_out/r12/{f}.json')); r=d['roofline']
        print(f, round(d['value'],1), round(d['ms_per_step'],3), d['rounds'], round(r['frac'],4), r.get('spfp_relax_and_wait_steps_per_step'), r['kernels_ms_per_step'])
    except Exception as e: print(f, 'ERR', e)
PY
tail -3 gpurun_out/r12/bench_C2_spfp.err
