mkdir -p gpurun_out/final11
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/final11/smoke.log 2>&1; echo smoke=$?
timeout 3000 python -m pytest tests -m gpu -x -q > gpurun_out/final11/pytest_gpu.log 2>&1; echo pytest=$?
tail -1 gpurun_out/final11/pytest_gpu.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/final11/bench_C4.json 2> gpurun_out/final11/bench_C4.err; echo c4=$?
for c in C1 C2 C3; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/final11/bench_$c.json 2> gpurun_out/final11/bench_$c.err; echo $c=$?
done
timeout 600 python bench.py --config C5 --partitions 2 --query-only --k 1 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/final11/bench_C5_single_source.json 2> gpurun_out/final11/bench_C5.err; echo c5=$?
timeout 900 python bench.py --config C5 --partitions 8 --query-only --k 4 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/final11/bench_C5.json 2> gpurun_out/final11/bench_C5b.err; echo c5b=$?
timeout 900 python bench.py --config C2 --problems sp,fp --k 32 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/final11/bench_C2_spfp.json 2> gpurun_out/final11/bench_C2_spfp.err; echo spfp=$?
timeout 600 python bench.py --impl reference --steps 1 --warmup 3 > gpurun_out/final11/bench_reference_C4.json 2> gpurun_out/final11/bench_ref.err; echo ref=$?
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name regex:"^(k_|void .*k_)" -c 400 --csv --log-file gpurun_out/final11/launches_bench_C4.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/final11/ncu_launches.log 2>&1; echo ncu3=$?
python - <<'PY'
import json, glob
for f in sorted(glob.glob('gpurun_out/final11/bench_*.json')):
    try:
        d=json.load(open(f)); r=d.get('roofline') or {}
        print(f.split('/')[-1], round(d['value'],2), round(d.get('ms_per_step') or 0,2), r.get('frac') and round(r['frac'],4), r.get('relax_share_of_step'), (d.get('e2e') or {}).get('value'), d.get('clocks'), d.get('gpu_launches'))
    except Exception as e: print(f, 'ERR', e)
PY
