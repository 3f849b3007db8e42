mkdir -p gpurun_out/final10
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/final10/bench_C4.json 2> gpurun_out/final10/bench_C4.err; echo c4=$?
python -c "
import json; d=json.load(open('gpurun_out/final10/bench_C4.json')); r=d['roofline']; print(round(d['value'],1), round(d['ms_per_step'],1), r['frac'], r['traffic_vs_algorithmic'], d['e2e']['value'], d['cpu_baseline']['value'], d['clocks'], d['step_ms'])"
