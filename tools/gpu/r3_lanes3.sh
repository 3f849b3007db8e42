mkdir -p gpurun_out/r3u
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
L=$D/libtempgraph.so
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r3u/pytest.log 2>&1; echo pytest=$?; tail -1 gpurun_out/r3u/pytest.log
timeout 900 python tools/job_exp.py C4 1024 $L:lanes=1 $L:lanes=2 $L:lanes=4 > gpurun_out/r3u/job_c4.log 2>&1; echo c4=$?
cat gpurun_out/r3u/job_c4.log
timeout 900 python bench.py --steps 6 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r3u/bench_C4.json 2> gpurun_out/r3u/bench_C4.err; echo b4=$?
timeout 600 python bench.py --config C2 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r3u/bench_C2.json 2> gpurun_out/r3u/bench_C2.err; echo b2=$?
python - <<'PY'
import json
for c in ['C4','C2']:
    d=json.load(open(f'gpurun_out/r3u/bench_{c}.json')); r=d['roofline']
    print(c, round(d['value'],1), round(d['ms_per_step'],1), d['step_ms'], r['relax_ms_per_step'], r['frac'], d['graph']['build_ms'])
PY
