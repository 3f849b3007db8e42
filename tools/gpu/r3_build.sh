mkdir -p gpurun_out/r3k
D=paper_conf_asplos_0003wh0dhwy0lyl25_b200
timeout 900 python tools/build_bench.py $D/libtempgraph.so C4 > gpurun_out/r3k/build_c4.log 2>&1; echo b4=$?
TG_TRACE_BUILD=1 timeout 900 python tools/build_bench.py $D/libtempgraph.so C4 2>&1 | grep build-trace | tail -12 > gpurun_out/r3k/build_trace_c4.log
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/r3k/bench_c4.json 2> gpurun_out/r3k/bench_c4.err; echo bench=$?
cat gpurun_out/r3k/build_c4.log gpurun_out/r3k/build_trace_c4.log; python -c "
import json; d=json.load(open('gpurun_out/r3k/bench_c4.json')); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['e2e']['value'], d['clocks'])"
