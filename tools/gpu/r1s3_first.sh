set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1200 python -m pytest tests -x -q -m gpu --durations=15 > gpurun_out/gpu_tests.log 2>&1; echo tests=$?
timeout 600 python bench.py > gpurun_out/bench_C2.log 2>&1; echo bench=$?
for e in 1 2; do timeout 300 python tools/variant_bench.py paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so C2 64 --opt=engine:$e 2>&1 | grep -v Warn; done > gpurun_out/engines.log 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv >> gpurun_out/engines.log
