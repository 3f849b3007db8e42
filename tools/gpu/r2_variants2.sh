for lib in paper_conf_asplos_0003wh0dhwy0lyl25_b200/libtempgraph.so variants/lib_*.so; do
  timeout 300 python tools/variant_bench.py $lib C2 64 --check >> gpurun_out/variants2.log 2>&1
  timeout 300 python tools/variant_bench.py $lib C4 64 --problems=eat --opt=mirror:0 >> gpurun_out/variants2.log 2>&1
done
timeout 300 python tools/prof_query.py --config C2 --problem reach --k 64 --reps 4 > gpurun_out/reach_C2.log 2>&1
timeout 300 python tools/prof_query.py --config C4 --problem reach --k 64 --reps 2 > gpurun_out/reach_C4.log 2>&1
timeout 300 python tools/prof_query.py --config C1 --problem eat --k 1 --reps 5 > gpurun_out/eat_C1.log 2>&1
timeout 300 python -m pytest tests -m "gpu and not slow" -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
grep -h "median\|check" gpurun_out/variants2.log; grep rep gpurun_out/reach_C2.log gpurun_out/reach_C4.log gpurun_out/eat_C1.log; tail -2 gpurun_out/pytest_gpu.log
