# Bench lines of every config with the current library (no profiler).
set -x
mkdir -p gpurun_out/bl
timeout 300 python bench.py > gpurun_out/bl/bench_C2.json 2> gpurun_out/bl/bench_C2.err
timeout 300 python bench.py --config C3 > gpurun_out/bl/bench_C3.json 2> gpurun_out/bl/bench_C3.err
timeout 900 python bench.py --config C4 > gpurun_out/bl/bench_C4.json 2> gpurun_out/bl/bench_C4.err
timeout 900 python bench.py --config C5 --partitions 8 --query-only > gpurun_out/bl/bench_C5.json 2> gpurun_out/bl/bench_C5.err
