# round 2: gap-skip variant, -m gpu (not slow), bench lines for every config + f1/f2 lines
mkdir -p gpurun_out/r2
for lib in paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so variants/lib_nogap.so; do
  timeout 300 python tools/variant_bench.py $lib C2 64 >> gpurun_out/r2/variants3.log 2>&1
  timeout 300 python tools/variant_bench.py $lib C4 64 --problems=eat --opt=mirror:0 >> gpurun_out/r2/variants3.log 2>&1
done
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r2/smoke.log 2>&1; echo smoke=$?
timeout 1200 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/r2/pytest_gpu.log 2>&1; echo pytest=$?
tail -2 gpurun_out/r2/pytest_gpu.log
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/r2/bench_C4.json 2> gpurun_out/r2/bench_C4.err; echo c4=$?
for c in C1 C2 C3; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/r2/bench_$c.json 2> gpurun_out/r2/bench_$c.err; echo $c=$?
done
timeout 600 python bench.py --config C2 --problems reach --reach-bits --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r2/bench_C2_reachbits.json 2> gpurun_out/r2/bench_C2_reachbits.err; echo reach=$?
timeout 600 python bench.py --config C2 --problems eat --stream-blocks 8 --query-only --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/r2/bench_C2_streamed8.json 2> gpurun_out/r2/bench_C2_streamed8.err; echo stream=$?
timeout 900 python bench.py --config C5 --partitions 8 --query-only --k 4 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/r2/bench_C5.json 2> gpurun_out/r2/bench_C5.err; echo c5=$?
grep -h median gpurun_out/r2/variants3.log
