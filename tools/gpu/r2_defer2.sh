mkdir -p gpurun_out/r2
for lib in variants/lib_defer*.so; do
  timeout 300 python tools/variant_bench.py $lib C2 64 --check >> gpurun_out/r2/variants_defer2.log 2>&1
  timeout 300 python tools/variant_bench.py $lib C4 64 --problems=eat --opt=mirror:0 >> gpurun_out/r2/variants_defer2.log 2>&1
done
timeout 900 python bench.py --config C2 --problems sp,fp --k 32 --steps 3 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/r2/bench_C2_spfp.json 2> gpurun_out/r2/bench_C2_spfp.err; echo spfp=$?
grep -h "median\|check" gpurun_out/r2/variants_defer2.log
