mkdir -p gpurun_out/final6
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -k "lanes or loop or bound" > gpurun_out/final6/pytest.log 2>&1; echo pytest=$?; tail -1 gpurun_out/final6/pytest.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/final6/bench_C4.json 2> gpurun_out/final6/bench_C4.err; echo c4=$?
timeout 600 python bench.py --config C2 --steps 10 --warmup 3 > gpurun_out/final6/bench_C2.json 2> gpurun_out/final6/bench_C2.err; echo c2=$?
python - <<'PY'
import json
for c in ['C4','C2']:
    d=json.load(open(f'gpurun_out/final6/bench_{c}.json')); r=d['roofline']
    print(c, round(d['value'],1), round(d['ms_per_step'],2), r['frac'], d['e2e']['value'], d['e2e']['ms_per_step'], d['step_ms'])
PY
