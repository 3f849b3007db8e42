mkdir -p gpurun_out/r18
for P in 2 4; do
timeout 900 python bench.py --config C5 --partitions $P --query-only --k 1 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r18/bench_C5_p$P.json 2> gpurun_out/r18/bench_C5_p$P.err; echo p$P=$?
tail -2 gpurun_out/r18/bench_C5_p$P.err
done
python - <<'PY'
import json
for P in (2, 4):
    try:
        d=json.load(open(f'gpurun_out/r18/bench_C5_p{P}.json')); r=d['roofline']
        print(P, round(d['value'],2), round(d['ms_per_step'],2), d['rounds'], round(r['frac'],4), d['graph']['device_bytes'], r['kernels_ms_per_step'])
    except Exception as e: print(P, 'ERR', e)
PY
