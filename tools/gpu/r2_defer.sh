mkdir -p gpurun_out/r2
for lib in paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so variants/lib_defer*.so; do
  timeout 300 python tools/variant_bench.py $lib C2 64 --check >> gpurun_out/r2/variants_defer.log 2>&1
  timeout 300 python tools/variant_bench.py $lib C4 64 --problems=eat --opt=mirror:0 >> gpurun_out/r2/variants_defer.log 2>&1
done
TG_TRACE_BUILD=1 timeout 600 python tools/dynamic_bench.py C2 100000 3 > gpurun_out/r2/dyn_trace.log 2>&1
grep -h "median\|check" gpurun_out/r2/variants_defer.log; grep insert-trace gpurun_out/r2/dyn_trace.log | tail -12
