mkdir -p gpurun_out/r3d2
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
timeout 1500 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r3d2/pytest.log 2>&1; echo pytest=$?; tail -1 gpurun_out/r3d2/pytest.log
timeout 900 python tools/job_exp.py C4 1024 $D/libtg_base2.so $D/libtempgraph.so $D/libtempgraph.so 2>&1 | grep ms
timeout 900 python tools/job_exp.py C2 256 $D/libtempgraph.so 2>&1 | grep ms
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r3d2/bench_C4.json 2> gpurun_out/r3d2/bench_C4.err; echo c4=$?
python -c "
import json; d=json.load(open('gpurun_out/r3d2/bench_C4.json')); r=d['roofline']; print(round(d['value'],1), round(d['ms_per_step'],1), r['frac'], d['e2e']['value'], d['step_ms'])"
