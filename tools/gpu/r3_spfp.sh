mkdir -p gpurun_out/r3za
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
timeout 1500 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r3za/pytest.log 2>&1; echo pytest=$?; tail -1 gpurun_out/r3za/pytest.log
for c in C1 C3 C2; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r3za/bench_$c.json 2> gpurun_out/r3za/bench_$c.err; echo $c=$?; done
timeout 900 python bench.py --config C2 --problems sp,fp --k 32 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r3za/bench_C2_spfp.json 2> gpurun_out/r3za/bench_C2_spfp.err; echo spfp=$?
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name regex:"^(k_|void .*k_)" -c 400 --csv --log-file gpurun_out/r3za/launches_bench_C4.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/r3za/ncu_launches.log 2>&1; echo ncu3=$?
python - <<'PY'
import json, glob
for f in sorted(glob.glob('gpurun_out/r3za/bench_*.json')):
    d=json.load(open(f)); r=d.get('roofline') or {}
    print(f.split('/')[-1], round(d['value'],2), round(d['ms_per_step'],3), r.get('frac'), r.get('kernels_ms_per_step'))
PY
